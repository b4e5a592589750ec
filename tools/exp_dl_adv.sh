#!/bin/bash
# Run under gpurun: divergent loop, run-ahead lanes taking up to V iterations per
# advance round: parity + schedule tests, then T x V (CUDA-event timing per launch).
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q -k divloop > $O/tests_dladv.log 2>&1; tail -1 $O/tests_dladv.log
for v in 1 2 4 8 16 64; do
  timeout 600 python tools/sweep.py --reps 20 --what divloop --thresholds 8,12,16,24,32 --unroll $v > $O/dlv_$v.json 2>/dev/null
  python - <<PY
import json
d = json.load(open("$O/dlv_$v.json"))["divloop"]
print("V=$v", [(r["T"], round(r["ms"] * 1000, 1)) for r in d])
PY
done
