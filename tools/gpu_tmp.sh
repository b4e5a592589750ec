# scratch launcher for the current gpurun experiment (see profiles/experiments.md)
python -c "import __graft_entry__ as g; g.build()"
O=gpurun_out
for U in 4 6 8 10 12 16; do
  timeout 600 python tools/sweep.py --what pathtrace --thresholds 10,12,14 --unroll $U --reps 5 --flags 32 > $O/sw_u_$U.json 2>/dev/null
  python -c "
import json;d=json.load(open('$O/sw_u_$U.json'))['pathtrace']
print('U=$U pool', [(r['mode'],r['T'],round(r['ms'],2)) for r in d])"
done
