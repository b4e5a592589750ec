#!/bin/bash
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "unrolled or deferred" 2>&1 | tail -1
for U in 1 2 4 8; do
  python tools/sweep.py --what mcml --blocks 512 --thresholds 32,24 --reps 3 --unroll $U 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('unroll $U', [(r['mode'],r['T'],round(r['ms'],2)) for r in d['mcml']])"
done
