#!/bin/bash
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k mcml 2>&1 | tail -1
for D in 0 2 4 8 16 32; do
  python tools/sweep.py --what mcml --blocks 512 --thresholds 32 --reps 3 --defer $D 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('defer $D', [(r['mode'],r['T'],round(r['ms'],2)) for r in d['mcml']])"
done
