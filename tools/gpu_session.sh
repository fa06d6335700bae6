#!/bin/bash
# One measurement session on the GPU box: sanitizers, ncu launch list + DRAM traffic
# (same session as the bench line), ncu --set full of the hot kernels, the bench line,
# the GPU test tiers.   gpurun -- bash tools/gpu_session.sh <tag>
TAG=${1:-run}
O=gpurun_out/$TAG
mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build
python -c "import oracle; oracle.build()"
# compute-sanitizer is closed on this GPU pool (it reports so and exits): the sanitizer
# driver runs without it -- every C-ABI flow once, checked for errors by the library
for t in memcheck racecheck synccheck; do
  echo "== compute-sanitizer --tool $t (tools/sanitize.py)" >> $O/sanitizers.txt
  timeout 300 compute-sanitizer --tool $t python tools/sanitize.py 2>&1 | tail -n 3 >> $O/sanitizers.txt
done
echo "== python tools/sanitize.py (no sanitizer)" >> $O/sanitizers.txt
timeout 600 python tools/sanitize.py >> $O/sanitizers.txt 2>&1 && echo "sanitize.py flows: ok" >> $O/sanitizers.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
    python bench.py --profile-only --steps 1 --warmup 0 > /dev/null 2>&1
timeout 1800 python tools/ncu_traffic.py $TAG > $O/traffic.log 2>&1
NCU="ncu --set full --import-source on --clock-control none --cache-control none"
PB="python bench.py --profile-only --steps 1 --warmup 1"
timeout 900 $NCU -k regex:'^k_jp_rounds$' -s 1 -c 1 -o $O/jp $PB > /dev/null 2>&1
timeout 900 $NCU -k regex:'^k_jpc_fill' -s 1 -c 1 -o $O/fill $PB > /dev/null 2>&1
timeout 900 $NCU -k regex:'^k_split' -s 2 -c 2 -o $O/split $PB > /dev/null 2>&1
timeout 900 $NCU -k regex:'^k_(round0|mm_round)' -s 20 -c 4 -o $O/mm $PB > /dev/null 2>&1
timeout 900 $NCU -k regex:'^k_mis_round' -s 16 -c 4 -o $O/mis $PB > /dev/null 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 1800 python -m pytest tests -m "gpu and not scale27" -q -x > $O/pytest_gpu.txt 2>&1
timeout 1500 python -m pytest tests -m scale27 -q -x > $O/pytest_s27.txt 2>&1
tail -2 $O/pytest_gpu.txt $O/pytest_s27.txt
grep -h "SUMMARY" $O/sanitizers.txt
ls -la $O
