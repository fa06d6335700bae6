O=gpurun_out/r2ze; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
bash tools/ab.sh r2ze "mis_none mis_deg2 mm_none mm_rand4 color_deg2" "" "-DSYM_JP_ACT_SMEM=0"
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py tests/test_gpu_bridge.py tests/test_sharded.py -m gpu -q -x > $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "mis or color" >> $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 900 python bench.py --steps 20 --warmup 5 --no-seq > $O/bench.json 2> $O/bench.err
python -c "import json; d=json.loads(open('$O/bench.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['breakdown_ms'])"
