# Build-knob sweep of the whole step: for each set of -D knobs, rebuild libsym, run the
# small-graph parity tests, and a short bench (per-class ms).
#   bash tools/knob_sweep.sh <tag> "<defs 1>" "<defs 2>" ...
O=gpurun_out/$1; shift; mkdir -p $O
for defs in "$@"; do
  echo "== $defs" | tee -a $O/sweep.txt
  SYM_NVCC_DEFS="$defs" python -m paper_conf_ipps_nayyaroddeengk17_b200.build --force > /dev/null 2>&1 || { echo build failed | tee -a $O/sweep.txt; continue; }
  timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -n 1 | tee -a $O/sweep.txt
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-configs --no-e2e 2>/dev/null | tail -n 1 > $O/b.json
  python -c "
import json; d=json.loads(open('$O/b.json').read())
print(round(d['ms_per_step'],3), {k:(round(v['ms_per_launch'],3), v['launches_per_call']) for k,v in d['rooflines'].items()})" | tee -a $O/sweep.txt
done
python -m paper_conf_ipps_nayyaroddeengk17_b200.build --force > /dev/null 2>&1
