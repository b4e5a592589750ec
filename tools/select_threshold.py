"""Simulator-guided soft-barrier threshold selection (
the paper leaves threshold discovery to future work).

For every candidate T the warp simulator (oracle part 2) replays the workload's
event streams under the SR schedule and the static SASS region costs of the
built cubin (tools/sass_regions.py) turn the replay into warp-instructions =
issue slots.  The kernels are issue-bound, so the predicted
time of a schedule is proportional to its warp-instructions; the selected T is
the argmin.  With --measured the prediction is set beside a measured threshold
sweep (tools/sweep.py JSON) and the cost of trusting the model is reported:
measured time at the predicted T over the measured best.

MC is simulated on a sample of warps (photon streams are i.i.d., so the mean
per-warp cost of a sample estimates the launch's); the other workloads are
simulated in full at their configs[] size.

TEST/EVALUATION INFRASTRUCTURE: uses oracle/ (event streams + simulator).

usage: python tools/select_threshold.py [--what divloop,rsbench,rsfetch,mcml,pathtrace]
           [--thresholds 1,2,4,8,16,24,32] [--mc-warps 512] [--mc-iters 64]
           [--unroll 4] [--measured sweep.json ...] [--write out.json]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import sass_regions  # noqa: E402
import simt_predict as sp  # noqa: E402
from paper_conf_cgo_damanijskymg20_b200 import inputs as I  # noqa: E402


def mc_sample(n_warps, iters):
    """Event streams of n_warps*32 lanes x iters photons (static layout)."""
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    n = n_warps * 32
    ev, off, ns = oracle.mcml_events_batch(p, 0, n * iters, I.PRIMARY_SEED)
    return np.ascontiguousarray(ev), off, ns, n


def mc_warps(sample, iters, mode, T, U):
    ev, off, ns, n = sample
    for w in range(0, n, 32):
        lanes = np.arange(w, w + 32)
        ids = lanes[:, None] + np.arange(iters)[None, :] * n
        yield oracle.ws_loopmerge_raw(ns[ids], ev, off[ids].ravel(), mode, T, U=U), 32


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--what", default="divloop,rsbench,rsfetch,mcml")
    ap.add_argument("--thresholds", default="1,2,4,8,16,24,32")
    ap.add_argument("--mc-warps", type=int, default=512)
    ap.add_argument("--mc-iters", type=int, default=I.C3.iters)
    ap.add_argument("--unroll", type=int, default=I.C3.merge_unroll)
    ap.add_argument("--measured", nargs="*", default=[])
    ap.add_argument("--write", default="")
    a = ap.parse_args()
    Ts = [int(x) for x in a.thresholds.split(",")]
    costs = sass_regions.kernel_costs("divloop_|mcml_|rs_|pt_")

    fams = {}
    if "divloop" in a.what:
        fams["divloop"] = (r"divloop_pdomILi125ELb0", r"divloop_specILi125ELb0",
                           lambda mode, T: sp.divloop_warps(mode, T), I.C1.n_threads * I.C1.iters)
    if "rsbench" in a.what:
        fams["rsbench"] = (r"rs_pdomILi8ELi0ELb0", r"rs_specILi8ELi0ELb0ELb1E",   # warp pool
                           lambda mode, T: sp.rsbench_warps(mode, T, pool=True),
                           I.NEXT1.n_threads * I.NEXT1.iters)
    if "rsfetch" in a.what:   # the expensive-prolog variant (trip counts are the same)
        fams["rsfetch"] = (r"rs_pdomILi8ELi256ELb0", r"rs_specILi8ELi256ELb0ELb1E",
                           lambda mode, T: sp.rsbench_warps(mode, T, pool=True),
                           I.NEXT1.n_threads * I.NEXT1.iters)
    if "pathtrace" in a.what:   # sampled warps (simt_predict.PT_SAMPLE), split merge U = 8
        fams["pathtrace"] = (r"pt_pdomILb0E", r"pt_specILb0ELb1ELb1ELb0ELb0EE",
                             lambda mode, T: sp.pt_warps(mode, T, 8),
                             sp.PT_SAMPLE * 32 * I.C4.spp)
    if "ptpool" in a.what:   # the same with the warp's paths pooled (SR_F_POOL)
        fams["ptpool"] = (r"pt_pdomILb0E", r"pt_specILb0ELb1ELb1ELb0ELb1EE",
                          lambda mode, T: sp.pt_warps(
                              oracle.SPEC_LOOP_POOL if mode == oracle.SPEC_LOOP else mode, T, 8),
                          sp.PT_SAMPLE * 32 * I.C4.spp)
    if "mcml" in a.what:
        sample = mc_sample(a.mc_warps, a.mc_iters)
        # the PDOM kernel ignores the unroll; SPEC runs U steps per release
        fams["mcml"] = (r"mcml_pdomILb0ELb0ELb1", r"mcml_specILb0ELb0ELb1",
                        lambda mode, T: mc_warps(sample, a.mc_iters, mode, T,
                                                 a.unroll if mode == oracle.SPEC_LOOP else 1),
                        sample[3] * a.mc_iters)

    measured = {}
    for path in a.measured:   # FILE, or FAMILY=FILE to file a sweep under another family
        rename = None
        if "=" in path:
            rename, path = path.split("=", 1)
        d = json.load(open(path))
        for fam, rows in d.items():
            fam = rename or fam
            measured.setdefault(fam, {})
            for r in rows:
                measured[fam][(r["mode"], r["T"])] = r["ms"]

    out = {}
    for fam, (pat_pdom, pat_spec, gen, units) in fams.items():
        base = sp.predict(sp.find(costs, pat_pdom), gen(oracle.PDOM, 0))
        rows = [dict(mode="pdom", T=0, inst=base["inst"], simt=base["simt"])]
        for T in Ts:
            p = sp.predict(sp.find(costs, pat_spec), gen(oracle.SPEC_LOOP, T))
            rows.append(dict(mode="spec", T=T, inst=p["inst"], simt=p["simt"]))
        for r in rows:
            r["inst_per_unit"] = r["inst"] / units
            r["pred_speedup"] = base["inst"] / r["inst"]
            ms = measured.get(fam, {}).get((r["mode"], r["T"]))
            if ms is not None:
                r["measured_ms"] = ms
        spec = [r for r in rows if r["mode"] == "spec"]
        t_pred = min(spec, key=lambda r: r["inst"])["T"]
        res = dict(rows=rows, T_pred=t_pred)
        have = [r for r in spec if "measured_ms" in r]
        if have:
            best = min(have, key=lambda r: r["measured_ms"])
            pdom_ms = rows[0].get("measured_ms")
            at_pred = next((r for r in have if r["T"] == t_pred), None)
            res.update(T_measured=best["T"],
                       loss_at_T_pred=(at_pred["measured_ms"] / best["measured_ms"]
                                       if at_pred else None))
            if pdom_ms:
                for r in rows:
                    if "measured_ms" in r:
                        r["meas_speedup"] = pdom_ms / r["measured_ms"]
            xs = np.array([r["pred_speedup"] for r in rows if "meas_speedup" in r])
            ys = np.array([r["meas_speedup"] for r in rows if "meas_speedup" in r])
            if len(xs) > 2:
                res["rank_corr"] = float(np.corrcoef(np.argsort(np.argsort(xs)),
                                                     np.argsort(np.argsort(ys)))[0, 1])
        out[fam] = res
        print(f"{fam}: T_pred={t_pred} " + " ".join(
            f"T={r['T']}:{r['pred_speedup']:.2f}" + (f"/{r['meas_speedup']:.2f}" if "meas_speedup" in r else "")
            for r in rows), file=sys.stderr)
    js = json.dumps(out, indent=1)
    if a.write:
        open(a.write, "w").write(js + "\n")
    print(js)


if __name__ == "__main__":
    main()
