#!/bin/bash
# Run under gpurun: GPU parity tests + one bench line (tag $1).
TAG=${1:-q}
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tests_$TAG.log 2>&1; tail -2 gpurun_out/tests_$TAG.log
timeout 900 python bench.py --no-cpu > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
python - <<PY
import json
d = json.load(open("gpurun_out/bench_$TAG.json"))
print("mc spec", d["ms_per_step"], "pdom", d["pdom"]["ms_per_step"], "x", round(d["speedup_vs_pdom"], 3))
c = d.get("configs", {})
for k, v in c.items():
    print(k, {kk: (round(vv["ms"], 4) if isinstance(vv, dict) and "ms" in vv else vv) for kk, vv in v.items() if kk != "launch"})
PY
