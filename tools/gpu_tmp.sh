python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_pathtrace.py -q -x > $O/t_g25.log 2>&1; tail -3 $O/t_g25.log
for F in 0 32 0 32; do
  timeout 900 python tools/sweep.py --what pathtrace --thresholds 8,12,16 --unroll 8 --reps 5 --flags $F > $O/sw_pt25_$F.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_pt25_$F.json'))['pathtrace']
print('flags $F', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
