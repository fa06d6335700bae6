O=gpurun_out/r2t; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 600 python tools/exp.py mis_none mis_deg2 color_deg2 > $O/exp.txt 2>&1
SYM_JP_COUNTED=1 timeout 600 python tools/exp.py color_deg2 >> $O/exp.txt 2>&1
cat $O/exp.txt
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python tools/exp.py --once mis_none color_deg2 > /dev/null 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x -k "mis or color or sharded or variants or smoke or bridge or concurrent" > $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "mis or color" >> $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
bash tools/ab.sh r2t "mis_none mis_deg2" "-DSYM_MIS_MINB=5"
