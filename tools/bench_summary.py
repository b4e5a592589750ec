"""One-screen summary of a bench.py JSON line: python tools/bench_summary.py FILE"""
import json
import sys

d = json.loads([l for l in open(sys.argv[1]) if l.startswith("{")][-1])
print("mc spec ms", round(d["ms_per_step"], 3), "pdom", round(d["pdom"]["ms_per_step"], 3),
      "x", round(d["speedup_vs_pdom"], 3), "roofline", round((d.get("roofline") or {}).get("frac", 0), 3))
for k, v in (d.get("configs") or {}).items():
    row = {}
    for kk, vv in v.items():
        if isinstance(vv, dict) and "ms" in vv:
            row[kk] = round(vv["ms"], 4)
        elif isinstance(vv, float):
            row[kk] = round(vv, 3)
        elif kk == "issue_roofline":
            row["roof"] = {a: round(b, 3) for a, b in vv["frac"].items()}
    print(k, row)
