O=gpurun_out/r2y; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_sharded.py tests/test_gpu_variants.py tests/test_gpu_bridge.py -m gpu -q -x > $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x >> $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
bash tools/ab.sh r2y "split_degk mis_none mis_deg2 mm_none mm_rand4 color_deg2" "" "-DSYM_MM_MINB=6" "-DSYM_MM_MINB=4" "-DSYM_SPLIT_PREGATHER=1" "-DSYM_SPLIT_PREGATHER=2"
