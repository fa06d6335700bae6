# JP experiment: colour parity (small + s24), per-round traces, bench step
O=gpurun_out/${1:-jpx}; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build
timeout 900 python -m pytest tests/test_gpu_parity.py -k color -q -x > $O/parity.txt 2>&1; tail -n 2 $O/parity.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -k "c4 or color" -q -x > $O/full.txt 2>&1; tail -n 2 $O/full.txt
timeout 300 python tools/diag_jp_levels.py 24 > $O/trace.txt 2>&1; tail -n 14 $O/trace.txt
SYM_JP_TRACE=2 timeout 300 python tools/diag_jp_levels.py 24 > $O/trace2.txt 2>&1; tail -n 14 $O/trace2.txt
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-configs --no-e2e > $O/bench.json 2>$O/bench.err; python -c "
import json; d=json.loads(open('$O/bench.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], {k:(round(v['ms_per_launch'],3), v['launches_per_call']) for k,v in d['rooflines'].items()})"
