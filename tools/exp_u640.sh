#!/bin/bash
# Run under gpurun: MC parity tests with the current build and the merge-unroll sweep.
TAG=${1:-u640}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "mcml or smoke or bench" > $O/tests_$TAG.log 2>&1; tail -1 $O/tests_$TAG.log
for U in 2 3 4 6 8; do
  timeout 300 python tools/sweep.py --what mcml --thresholds 32 --reps 5 --unroll $U 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('unroll $U', [(r['mode'],r['T'],round(r['ms'],3)) for r in d['mcml']])"
done
