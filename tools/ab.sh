# A/B of build knobs on one box: for each "<defs>" rebuild libsym and run tools/exp.py.
#   bash tools/ab.sh <tag> "<exp.py args>" "<defs 1>" "<defs 2>" ...
O=gpurun_out/$1; shift; ARGS=$1; shift; mkdir -p $O
for defs in "$@"; do
  echo "== [$defs]" | tee -a $O/ab.txt
  SYM_NVCC_DEFS="$defs" python -m paper_conf_ipps_nayyaroddeengk17_b200.build --force > /dev/null 2>&1 || { echo build failed | tee -a $O/ab.txt; continue; }
  timeout 600 python tools/exp.py $ARGS 2>&1 | tee -a $O/ab.txt
done
python -m paper_conf_ipps_nayyaroddeengk17_b200.build --force > /dev/null 2>&1
