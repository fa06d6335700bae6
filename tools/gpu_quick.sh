# Quick GPU check: build, one bench line, the GPU tests (without scale 27).
#   gpurun -- bash tools/gpu_quick.sh <tag>
O=gpurun_out/${1:-quick}
mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
tail -c 600 $O/bench.json
timeout 2400 python -m pytest tests -m "gpu and not scale27" -q -x > $O/pytest_gpu.txt 2>&1
tail -3 $O/pytest_gpu.txt
