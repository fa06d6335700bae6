O=gpurun_out/r2zo; mkdir -p $O
bash tools/ab.sh r2zo "color_deg2" "" "-DSYM_JP_FILTER_MIN=0" "-DSYM_JP_FILTER_MIN=512" "-DSYM_JP_FILTER_MIN=8192" "-DSYM_JP_FILTER_MIN=2000000000"
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -x -k "color" > $O/pytest.txt 2>&1; tail -2 $O/pytest.txt
