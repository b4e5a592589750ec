#!/bin/bash
# Run under gpurun: MC parity tests + two headline bench timings (no configs, no CPU).
TAG=${1:-mcq}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "mcml or smoke or dom or hg or device_math" > $O/tests_$TAG.log 2>&1; tail -1 $O/tests_$TAG.log
for rep in 1 2; do
  timeout 300 python bench.py --no-cpu --no-configs --steps 10 > $O/mcq_${TAG}_$rep.json 2>/dev/null
  python -c "import json;d=json.load(open('$O/mcq_${TAG}_$rep.json'));print(round(d['ms_per_step'],3), round(d['pdom']['ms_per_step'],3), round(d['roofline']['frac'],3))"
done
