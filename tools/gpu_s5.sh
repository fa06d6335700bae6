O=gpurun_out/r2u; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "mm or sharded or smoke or bridge or variants" > $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "mm" >> $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
bash tools/ab.sh r2u "mm_none mm_rand4 mis_none mis_deg2" "" "-DSYM_MM_ALT=0" "-DSYM_MM_MINB=5"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python tools/exp.py --once mm_none mm_rand4 > /dev/null 2>&1
