O=gpurun_out/r2x; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "mm or color" > $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x -k "mm or color" >> $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
bash tools/ab.sh r2x "mm_none mm_rand4 mis_deg2 color_deg2" "" "-DSYM_MM_SMALL=16" "-DSYM_MM_SMALL=32" "-DSYM_MM_SMALL=32 -DSYM_MM_MINB=5" "-DSYM_FILL_BATCH=8" "-DSYM_POLL_BATCH=8"
timeout 1500 python tools/ncu_traffic.py r2x > $O/traffic.log 2>&1; tail -3 $O/traffic.log
