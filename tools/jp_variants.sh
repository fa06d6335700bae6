# Build-knob sweep of the JP rounds kernel: for each set of -D knobs, rebuild libsym,
# check COLOR parity (small graphs) and time COLOR-Deg2 at R-MAT s24 (tools/diag_jp_levels.py).
#   bash tools/jp_variants.sh <tag> "<defs 1>" "<defs 2>" ...
O=gpurun_out/$1; shift; mkdir -p $O
for defs in "$@"; do
  echo "== $defs" | tee -a $O/variants.txt
  SYM_NVCC_DEFS="$defs" python -m paper_conf_ipps_nayyaroddeengk17_b200.build --force > /dev/null 2>&1 || { echo build failed | tee -a $O/variants.txt; continue; }
  timeout 600 python -m pytest tests/test_gpu_parity.py -k color -q -x 2>&1 | tail -n 1 | tee -a $O/variants.txt
  timeout 300 python tools/diag_jp_levels.py 24 2>&1 | grep -E "COLOR-Deg2 ms|profile|median" | tee -a $O/variants.txt
done
python -m paper_conf_ipps_nayyaroddeengk17_b200.build --force > /dev/null 2>&1
