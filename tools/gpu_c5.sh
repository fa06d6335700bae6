# C5 (R-MAT s27 ef16) timings on one GPU: gpurun -- bash tools/gpu_c5.sh <tag>
O=gpurun_out/${1:-c5}; mkdir -p $O
python -m paper_conf_ipps_nayyaroddeengk17_b200.build > $O/build.log 2>&1
timeout 1800 python bench.py --c5 --steps 5 --warmup 3 --no-cpu --no-e2e --reps 3 > $O/bench_c5.json 2> $O/bench_c5.err
python -c "import json; d=json.loads(open('$O/bench_c5.json').read().strip().splitlines()[-1]); c=d['configs']['C5']; print(json.dumps({k:(v['ms_incl_decomp'], v['ms_problem_only'], v['rounds']) if isinstance(v,dict) and 'rounds' in v else v for k,v in c.items()}))"
