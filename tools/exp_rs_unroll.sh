#!/bin/bash
# Run under gpurun: RSBench merged inner loop partially unrolled (U iterations per
# release): parity + schedule tests, then thresholds x U (plain and expensive-fetch).
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_rsbench.py -x -q > $O/tests_rsu.log 2>&1; tail -1 $O/tests_rsu.log
for u in ${US:-1 2 3 4}; do
  timeout 600 python tools/sweep.py --reps 5 --what rsbench --thresholds ${TS:-16,24,32} --unroll $u > $O/rsu_$u.json 2>/dev/null
  timeout 600 python tools/sweep.py --reps 5 --what rsbench --thresholds 8,12,16 --prolog 2048 --unroll $u > $O/rsfu_$u.json 2>/dev/null
  python - <<PY
import json
for f, k in (("$O/rsu_$u.json", "rsbench"), ("$O/rsfu_$u.json", "rsfetch")):
    d = json.load(open(f))[k]
    print("U=$u", k, [(r["T"], round(r["ms"], 3)) for r in d])
PY
done
