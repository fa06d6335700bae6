# Final evidence of the round: bench line, launch list, per-class traffic, ncu full of the
# changed kernels, GPU test tiers.   gpurun -- bash tools/gpu_final.sh <tag>
TAG=${1:-final}
O=gpurun_out/$TAG
mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build
python -c "import oracle; oracle.build()"
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
    python bench.py --profile-only --steps 1 --warmup 0 > /dev/null 2>&1
timeout 1800 python tools/ncu_traffic.py $TAG > $O/traffic.log 2>&1
NCU="ncu --set full --import-source on --clock-control none --cache-control none"
PB="python bench.py --profile-only --steps 1 --warmup 1"
timeout 900 $NCU -k regex:'^k_jp_rounds$' -s 1 -c 1 -o $O/jp $PB > /dev/null 2>&1
timeout 900 $NCU -k regex:'^k_(round0|mm_round)' -s 20 -c 4 -o $O/mm $PB > /dev/null 2>&1
timeout 900 $NCU -k regex:'^k_mis_round' -s 12 -c 4 -o $O/mis $PB > /dev/null 2>&1
timeout 1800 python -m pytest tests -m "gpu and not scale27" -q -x > $O/pytest_gpu.txt 2>&1
timeout 1500 python -m pytest tests -m scale27 -q -x > $O/pytest_s27.txt 2>&1
tail -2 $O/pytest_gpu.txt $O/pytest_s27.txt
ls -la $O
