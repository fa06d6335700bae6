O=gpurun_out/r2za; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
SYM_JP_TRACE=2 timeout 300 python tools/diag_jp_levels.py 24 > $O/trace2.txt 2>&1; tail -n 20 $O/trace2.txt
timeout 300 python tools/diag_jp_levels.py 24 > $O/trace1.txt 2>&1; tail -n 20 $O/trace1.txt
