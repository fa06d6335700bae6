O=gpurun_out/r2zj; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
timeout 600 python tools/overlap_probe.py > $O/overlap.json 2> $O/overlap.err; cat $O/overlap.json; tail -3 $O/overlap.err
