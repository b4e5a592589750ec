"""Per-region check of the warp simulator against ncu SourceCounters
("per-region counts vs ncu SourceCounters").

For each simulator-validation launch, ncu's per-instruction counts (SASS page:
Instructions Executed, Thread Instructions Executed) are summed over the
source regions tools/sass_regions.py assigns to the same instructions of the
same cubin, and set beside the simulator's prediction for that region
(cost_r x executions_r warp-instructions, cost_r x lanes_r thread-instructions).
A whole-kernel SIMT match could hide compensating errors between regions; this
cannot.

TEST/EVALUATION INFRASTRUCTURE: uses oracle/ (via simt_predict).

usage: python tools/region_check.py <tag> [--write]
  reads gpurun_out/src_<label-key>_<tag>.ncu-rep (tools/gpu_profile.sh)
  --write: profiles/region_check_<tag>.json (+ the measured region sums, so the
           test can run without the .ncu-rep files)
"""
from __future__ import annotations

import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import sass_regions  # noqa: E402
import simt_predict as sp  # noqa: E402

# label -> report key (one single-launch report each)
REPORTS = {
    "divloop_pdom": "divloop_pdom", "divloop_spec(T=16)": "divloop_spec",
    "rs_pdom": "rs_pdom", "rs_spec(T=32)": "rs_spec",
    "mcml_pdom_static": "mc_pdom", "mcml_spec_static(T=32)": "mc_spec32",
    "mcml_spec_static(T=8)": "mc_spec8", "mcml_spec_static(T=32,U=4)": "mc_spec32u4",
    "divloop_pool(T=16)": "dlpool", "divloop_pool_split4(T=16)": "dlpool4",
    "pt_pdom": "pt_pdom", "pt_spec(T=12)": "pt_spec", "pt_spec_pool(T=12)": "pt_pool",
}


def ncu_sass_counts(rep):
    """[(address, inst_executed, thread_inst_executed)] of the report's kernel."""
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source",
                          "sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
    hdr = rows[hdr_i]
    ia, ie, it = hdr.index("Address"), hdr.index("Instructions Executed"), \
        hdr.index("Thread Instructions Executed")
    out = []
    for r in rows[hdr_i + 1:]:
        if len(r) <= it or not r[ia].startswith("0x"):
            continue
        out.append((int(r[ia], 16), float(r[ie] or 0), float(r[it] or 0)))
    return out


def measured_regions(label, tag, costs_all):
    pat = sp.CASES[label][0]
    k = next(k for k in costs_all if __import__("re").search(pat, k))
    instr = costs_all[k]["instr"]
    rep = os.path.join(ROOT, "gpurun_out", f"src_{REPORTS[label]}_{tag}.ncu-rep")
    counts = ncu_sass_counts(rep)
    base = min(a for a, _, _ in counts)
    by_off = {a - base: (e, t) for a, e, t in counts}
    meas, cold_inst, unknown = {}, 0.0, 0.0
    for off, key, _ in instr:
        e, t = by_off.get(off, (0.0, 0.0))
        if key is None:
            cold_inst += e
            continue
        m = meas.setdefault(key, [0.0, 0.0])
        m[0] += e
        m[1] += t
    known = {off for off, _, _ in instr}
    unknown = sum(e for off, (e, _) in by_off.items() if off not in known)
    return meas, cold_inst, unknown


def predicted_regions(label, costs_all):
    import re
    pat, gen = sp.CASES[label]
    costs = next(v for k, v in costs_all.items() if re.search(pat, k))["regions"]
    acc = {}
    for sim, nv in gen():
        for key, c in costs.items():
            name, full = key.split(":")[0], key.endswith(":full")
            if name in ("ENTRY", "UNMAPPED"):
                x, l = 1, nv
            elif name.startswith("COLD"):
                x, l = 0, 0
            else:
                x, ln = sim[name]
                l = x * nv if full else ln
            a = acc.setdefault(key, [0.0, 0.0])
            a[0] += c * x
            a[1] += c * l
    sc = sp.inst_scale(label)   # sampled-warp cases: scale to the whole launch
    return {k: [v[0] * sc, v[1] * sc] for k, v in acc.items()}


def main():
    tag = sys.argv[1]
    costs_all = sass_regions.kernel_costs("divloop_|mcml_|rs_|pt_")
    out = {}
    for label in REPORTS:
        rep = os.path.join(ROOT, "gpurun_out", f"src_{REPORTS[label]}_{tag}.ncu-rep")
        if not os.path.exists(rep):
            continue
        meas, cold, unknown = measured_regions(label, tag, costs_all)
        pred = predicted_regions(label, costs_all)
        tot = sum(v[0] for v in meas.values())
        rows = {}
        for key in sorted(set(meas) | set(pred)):
            m, p = meas.get(key, [0.0, 0.0]), pred.get(key, [0.0, 0.0])
            rows[key] = dict(meas_inst=m[0], pred_inst=p[0], meas_thread=m[1], pred_thread=p[1])
        out[label] = dict(regions=rows, total_inst=tot, cold_inst=cold, unmatched_inst=unknown,
                          sass_sha=next(iter(sass_regions.kernel_hashes(
                              sp.CASES[label][0]).values()), None))
        print(label, file=sys.stderr)
        for key, r in sorted(rows.items(), key=lambda kv: -kv[1]["meas_inst"]):
            print(f"  {key:14s} inst meas {r['meas_inst']:.4g} pred {r['pred_inst']:.4g}   "
                  f"thread meas {r['meas_thread']:.4g} pred {r['pred_thread']:.4g}",
                  file=sys.stderr)
    js = json.dumps(out, indent=1)
    if "--write" in sys.argv:
        open(os.path.join(ROOT, "profiles", f"region_check_{tag}.json"), "w").write(js + "\n")
    print(js)


if __name__ == "__main__":
    main()
