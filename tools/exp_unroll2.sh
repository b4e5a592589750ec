#!/bin/bash
# Run under gpurun: MC merge_unroll re-check after the domain-restricted div/sqrt step,
# plus one full bench line (configs incl. the RSBench / path-tracer roofline keys).
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
for rep in 1 2; do
for u in 3 4 5 6 8; do
  timeout 300 python bench.py --no-cpu --no-configs --steps 10 --unroll $u > $O/unr_${u}_$rep.json 2>/dev/null
  python -c "import json;d=json.load(open('$O/unr_${u}_$rep.json'));print('U=$u', round(d['ms_per_step'],3))"
done
done
timeout 600 python bench.py --no-cpu > $O/bench_cfg.json 2> $O/bench_cfg.err; tail -2 $O/bench_cfg.err
python - <<PY
import json
d=json.load(open("$O/bench_cfg.json"))
print(d["ms_per_step"], d["roofline"]["frac"])
for k in ("rsbench","pathtrace"): print(k, {kk: vv for kk, vv in d["configs"][k].items() if kk not in ("launch",)})
PY
