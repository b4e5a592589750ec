#!/bin/bash
# Run under gpurun: divergent-loop kernels with the software-pipelined prolog --
# parity tests, threshold sweep (block sizes 64/128), bench microbench line.
TAG=${1:-dp}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "divloop or smoke or abi" > $O/tests_$TAG.log 2>&1; tail -1 $O/tests_$TAG.log
timeout 600 python tools/sweep.py --what divloop --thresholds 1,4,8,12,16,20,24,32 --blocks 64,128 --reps 5 > $O/sweep_dl_$TAG.json 2>/dev/null
python - <<PY
import json
d = json.load(open("$O/sweep_dl_$TAG.json"))
print(json.dumps(d)[:3000])
PY
