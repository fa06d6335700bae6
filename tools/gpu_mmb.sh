# MM validation after a change: parity, full-size MM, sharded, one bench line
O=gpurun_out/${1:-mmv}; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_sharded.py tests/test_gpu_variants.py tests/test_gpu_bridge.py -m gpu -q -x > $O/pytest.txt 2>&1
tail -2 $O/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "mm" >> $O/pytest.txt 2>&1
tail -2 $O/pytest.txt
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
python -c "import json; d=json.loads(open('$O/bench.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['value']/1e9, d['e2e']['value']/1e9, d['breakdown_ms'])"
