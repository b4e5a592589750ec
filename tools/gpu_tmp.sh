python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_rsbench.py tests/test_gpu_parity.py -q -x > $O/t_g23.log 2>&1; tail -1 $O/t_g23.log
timeout 900 python tools/sweep.py --what rsbench --thresholds 24,32 --unroll 12 --reps 5 > $O/sw_rs23.json 2>/dev/null
timeout 900 python tools/sweep.py --what rsbench --thresholds 16,20,24 --unroll 12 --prolog 2048 --reps 5 > $O/sw_rsf23.json 2>/dev/null
python -c "
import json
for f in ('sw_rs23','sw_rsf23'):
    d=json.load(open('$O/'+f+'.json'))['rsbench']
    print(f, [(r['mode'],r['T'],round(r['ms'],3)) for r in d])"
timeout 900 python bench.py --steps 10 --no-cpu > $O/b_g23.json 2> $O/b_g23.err; python tools/bench_summary.py $O/b_g23.json
