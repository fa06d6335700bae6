O=gpurun_out/r2z; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 600 python tools/exp.py color_deg2 mm_rand4 mis_deg2 > $O/exp.txt 2>&1; cat $O/exp.txt
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py tests/test_gpu_bridge.py tests/test_sharded.py -m gpu -q -x -k "color or smoke" > $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "color" >> $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 900 python bench.py --steps 20 --warmup 5 --no-seq > $O/bench.json 2> $O/bench.err
python -c "import json; d=json.loads(open('$O/bench.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['breakdown_ms'])"
