# one bench line (N=1) on a fresh box: gpurun -- bash tools/gpu_bench.sh <tag>
O=gpurun_out/${1:-bench}; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $O/reference.json 2> $O/reference.err
tail -c 400 $O/bench.json; tail -c 300 $O/reference.json
