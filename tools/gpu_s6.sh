O=gpurun_out/r2v; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
python -c "import oracle; oracle.build()" >> $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_sharded.py -m gpu -q -x -k "mis or mm or color or smoke" > $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "mis or mm or color" >> $O/pytest.txt 2>&1
tail -3 $O/pytest.txt
bash tools/ab.sh r2v "mis_none mis_deg2 mm_none mm_rand4 color_deg2" "" "-DSYM_MIS_VEC=0 -DSYM_MM_VEC=0 -DSYM_JP_VEC=0" "-DSYM_MIS_MINB=4" "-DSYM_MM_ALT=0"
timeout 900 python bench.py --steps 20 --warmup 5 --no-seq > $O/bench.json 2> $O/bench.err
python -c "import json; d=json.loads(open('$O/bench.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['breakdown_ms'])"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python tools/exp.py --once mm_none mm_rand4 mis_none color_deg2 > /dev/null 2>&1
