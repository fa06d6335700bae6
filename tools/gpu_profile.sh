#!/bin/bash
# One GPU session: bench line + ncu launch list + ncu --set full of the hot kernels.
#   gpurun -- bash tools/gpu_profile.sh <tag>
set -x
TAG=${1:-run}
O=gpurun_out/$TAG
mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
tail -c 600 $O/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
    python bench.py --profile-only --steps 1 --warmup 0 > /dev/null 2>&1
NCU="ncu --set full --import-source on --clock-control none"
PB="python bench.py --profile-only --steps 1 --warmup 0"
timeout 600 $NCU -k regex:'^k_jp(_rounds|c_fill)$' -c 2 -o $O/jp $PB > /dev/null 2>&1
timeout 600 $NCU -k regex:'^k_split' -c 2 -o $O/split $PB > /dev/null 2>&1
timeout 600 $NCU -k regex:'^k_(round0|mm_round)' -c 3 -o $O/mm $PB > /dev/null 2>&1
timeout 600 $NCU -k regex:'^k_mis_round' -c 4 -o $O/mis $PB > /dev/null 2>&1
ls -la $O
