python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
S="python tools/sweep.py --what pathtrace --reps 3"
for U in 4 8 16; do timeout 900 $S --thresholds 4,8,12,16,24,32 --unroll $U --flags 64 > $O/sw_ptmix_u$U.json 2>/dev/null; done
for f in $O/sw_ptmix_u*.json; do python -c "
import json;d=json.load(open('$f'))['pathtrace']
print('$f'.split('/')[-1], [(r['mode'],r['T'],round(r['ms'],2), round(r.get('region_eff',0),3)) for r in d])"; done
