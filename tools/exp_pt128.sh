#!/bin/bash
# Run under gpurun: path tracer with vectorised read-only scene loads -- parity tests + timing.
TAG=${1:-pt128}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_pathtrace.py -x -q > $O/tests_$TAG.log 2>&1; tail -1 $O/tests_$TAG.log
timeout 600 python tools/sweep.py --what pathtrace --thresholds 4,8,16 --unroll 8 --reps 3 > $O/sweep_pt_$TAG.json 2>/dev/null
python -c "
import json;d=json.load(open('$O/sweep_pt_$TAG.json'))
for r in d['pathtrace']: print(r.get('mode'), r.get('T'), round(r['ms'],2))"
