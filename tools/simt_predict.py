"""Predict whole-kernel SIMT efficiency with the warp simulator (oracle part
2) and the static SASS region costs of the built cubin (tools/sass_regions.py),
and compare with the ncu measurement in profiles/simt_efficiency.json.

SIMT efficiency = thread-instructions / (32 x warp-instructions);
predicted = sum_r c_r L_r / (32 sum_r c_r X_r), where for each SASS region r
with cost c_r the simulator supplies X_r warp executions and L_r active lanes
over every warp of the launch ("X:full" regions run with every valid lane
whenever step X runs; ENTRY once per warp).

TEST/EVALUATION INFRASTRUCTURE: uses oracle/ (event streams + simulator).

usage: python tools/simt_predict.py  -> JSON (and profiles/simt_prediction.json with --write)
"""
from __future__ import annotations

import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import sass_regions  # noqa: E402
from paper_conf_cgo_damanijskymg20_b200 import inputs as I  # noqa: E402


def accumulate(costs, sim, n_valid, acc):
    for key, c in costs.items():
        name, full = key.split(":")[0], key.endswith(":full")
        if name in ("ENTRY", "UNMAPPED"):
            x, l = 1, n_valid
        elif name.startswith("COLD"):
            # the guarded slow branch of a domain check that the workloads never
            # take: no executions
            x, l = 0, 0
        else:
            x, ln = sim[name]
            l = x * n_valid if full else ln
        acc[0] += c * x
        acc[1] += c * l


def predict(costs, warps):
    """warps: iterable of (sim_counts_dict, n_valid)."""
    acc = [0, 0]
    for sim, nv in warps:
        accumulate(costs, sim, nv, acc)
    return dict(inst=acc[0], thread_inst=acc[1], simt=acc[1] / (32.0 * acc[0]))


def find(costs_all, pattern):
    import re
    for k, v in costs_all.items():
        if re.search(pattern, k):
            return v["regions"]
    raise KeyError(pattern)


def divloop_warps(mode, T, V=None, batch=False):
    """batch: the prolog_batch = 64 kernels -- each valid lane evaluates its
    conditions in groups of 8 draws at entry (MASKGRP, ceil(iters/8) times)"""
    c = I.C1
    V = c.advance_unroll if V is None else V
    want = oracle.divloop_wants(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.p_u32)
    groups = (min(c.iters, 64) + 7) // 8
    for w in range(0, c.n_threads, 32):
        ww = want[w:w + 32]
        s = oracle.ws_divloop(ww, mode, T, V=V if mode == oracle.SPEC_LOOP else 1)
        if batch:
            s["MASKGRP"] = (groups, groups * len(ww))
        yield s, len(ww)


def divloop_pool_warps(split=1):
    """the SR_F_POOL kernels: per window, every (valid) lane runs its prologs
    (MASKGRP: groups of 8 draws; with split > 1 each of the group's `split` warps
    takes 64 / split iterations); the window's N wanted calls then run as
    ceil(N/32) releases (STEP: N lanes in all) -- one warp's queue (split = 1) or
    the CTA's, its 32-call chunks dealt round-robin to the warps; warp 0 adds
    every thread's results in order (EPIK: per slice as many trips as the
    thread with the most calls, one lane per call).  Closed-form counts."""
    c = I.C1
    want = oracle.divloop_wants(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.p_u32)
    L = 64 // split
    for w in range(0, c.n_threads, 32):
        ww = want[w:w + 32].astype(np.int64)
        nv = len(ww)
        rel = [0] * split
        lanes = [0] * split
        groups = [0] * split
        epik_x = epik_l = 0
        for b in range(0, c.iters, 64):
            Ns = []
            for sl in range(split):
                lo, hi = b + sl * L, min(b + (sl + 1) * L, b + 64, c.iters)
                cnt = ww[:, lo:hi].sum(1) if hi > lo else np.zeros(nv, np.int64)
                Ns.append(int(cnt.sum()))
                groups[sl] += (max(hi - lo, 0) + 7) // 8
                epik_x += int(cnt.max()) if nv else 0
                epik_l += int(cnt.sum())
            N = sum(Ns)
            chunks = (N + 31) // 32
            for ch in range(chunks):       # chunk ch -> warp ch % split
                rel[ch % split] += 1
                lanes[ch % split] += min(32, N - 32 * ch)
        for sl in range(split):
            yield {"MASKGRP": (groups[sl], groups[sl] * nv), "RELEASE": (rel[sl], 32 * rel[sl]),
                   "STEP": (rel[sl], lanes[sl]),
                   "EPIK": (epik_x, epik_l) if sl == 0 else (0, 0), "rounds": rel[sl]}, nv


def commoncall_warps(mode):
    c = I.C2
    _, arm = oracle.commoncall(0, c.n_threads, 1, I.PRIMARY_SEED, c.split_u32, fma_count=0)
    for w in range(0, c.n_threads, 32):
        a = arm[w:w + 32]
        yield oracle.ws_commoncall(a, mode), len(a)


MC_VALIDATION = dict(n_threads=16384, iters=8)   # static launch the oracle can replay


def mcml_warps(mode, T, n_threads=MC_VALIDATION["n_threads"], iters=MC_VALIDATION["iters"], U=1):
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    ev, off, ns = oracle.mcml_events_batch(p, 0, n_threads * iters, I.PRIMARY_SEED)
    ev = np.ascontiguousarray(ev)
    for w in range(0, n_threads, 32):
        lanes = np.arange(w, min(w + 32, n_threads))
        ids = lanes[:, None] + np.arange(iters)[None, :] * n_threads   # static assignment
        yield oracle.ws_loopmerge_raw(ns[ids], ev, off[ids].ravel(), mode, T, U=U), len(lanes)


def rsbench_warps(mode, T, U=None, pool=False):
    """pool: the default warp task pool (SPEC); else lane l runs thread l's lookups"""
    c = I.NEXT1
    U = c.merge_unroll if U is None else U
    _, _, trips = oracle.rsbench(0, c.n_threads, c.iters, I.PRIMARY_SEED, fma_count=0, trips=True)
    for w in range(0, c.n_threads, 32):
        tr = trips[w:w + 32]
        if pool and mode == oracle.SPEC_LOOP:
            s = oracle.ws_loopmerge_pool(tr, T, U=U)
            s["PERK"] = (c.iters, c.iters * len(tr))   # the in-order per-thread sum
            yield s, len(tr)
        else:
            yield oracle.ws_loopmerge(tr, mode, T, U=U if mode == oracle.SPEC_LOOP else 1), len(tr)


# configs[3]: the path tracer's warps are 8 x 4 pixel tiles (inputs.pt_lane_pixels); the
# work-item streams come from oracle.pt_trace (the oracle's BVH traversal over
# the scene image sr_scene_build writes), sampled over PT_SAMPLE warps spread
# over the frame
PT_SAMPLE = 48
_pt_cache = {}


def _pt_streams():
    if "ops" not in _pt_cache:
        from paper_conf_cgo_damanijskymg20_b200 import sr
        c = I.C4
        tris, mat, mats, cam = I.cornell_scene(c)
        img = sr.scene_image_host(tris, mat, mats, cam)
        n_warps = c.n_pixels // 32
        picks = np.linspace(0, n_warps - 1, PT_SAMPLE).astype(np.int64)
        lanes = I.pt_lane_pixels(c.width, c.height)
        pix = lanes[(picks[:, None] * 32 + np.arange(32)[None, :]).ravel()]
        ops, off, _ = oracle.pt_trace(img, c.width, c.height, c.spp, c.max_depth,
                                      I.PRIMARY_SEED, pixels=pix)
        _pt_cache.update(ops=ops, off=off)
    return _pt_cache["ops"], _pt_cache["off"]


def pt_warps(mode, T=0, U=8):
    ops, off = _pt_streams()
    for w in range(PT_SAMPLE):
        o = off[32 * w:32 * w + 33]
        yield oracle.ws_pt(ops[o[0]:o[-1]], o - o[0], mode, T, U), 32


# the bench launch of configs[2] (dynamic claiming): a persistent grid of
# 2 x 148 CTAs of 640 threads = 5920 warps, each taking ~10^7 / 5920 photons in
# chunks from one counter.  Which photons a warp gets depends on timing; their
# step counts are i.i.d., so each sampled warp replays a stream of consecutive
# photon ids of the same length (one drain at the end, as on the GPU).
MC_DYN = dict(warps=5920, sample_warps=48)


def mcml_dyn_warps(mode, T, U=None, photons=None, sample=None):
    m = I.C3
    U = m.merge_unroll if U is None else U
    photons = photons or m.n_photons
    sample = sample or MC_DYN["sample_warps"]
    q = photons // MC_DYN["warps"]
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    ev, off, ns = oracle.mcml_events_batch(p, 0, q * sample, I.PRIMARY_SEED)
    ev = np.ascontiguousarray(ev)
    for w in range(sample):
        sl = slice(w * q, (w + 1) * q)
        yield oracle.ws_loopmerge_stream(ns[sl], mode, T, U=U if mode == oracle.SPEC_LOOP else 1,
                                         ev=ev, ev_off=off[sl]), 32


CASES = {
    "divloop_pdom": (r"divloop_pdomILi125ELb0", lambda: divloop_warps(oracle.PDOM, 0)),
    "divloop_spec(T=16)": (r"divloop_specILi125ELb0", lambda: divloop_warps(oracle.SPEC_LOOP, 16)),
    "commoncall_pdom": (r"commoncall_pdomILi250ELb0", lambda: commoncall_warps(oracle.PDOM)),
    "commoncall_spec": (r"commoncall_specILi250ELb0", lambda: commoncall_warps(oracle.SPEC_CALL)),
    "mcml_pdom_static": (r"mcml_pdomILb0ELb0ELb1", lambda: mcml_warps(oracle.PDOM, 0)),
    "mcml_spec_static(T=32)": (r"mcml_specILb0ELb0ELb1", lambda: mcml_warps(oracle.SPEC_LOOP, 32)),
    "mcml_spec_static(T=8)": (r"mcml_specILb0ELb0ELb1", lambda: mcml_warps(oracle.SPEC_LOOP, 8)),
    "mcml_spec_static(T=32,U=4)": (r"mcml_specILb0ELb0ELb1",
                                   lambda: mcml_warps(oracle.SPEC_LOOP, 32, U=4)),
    "rs_pdom": (r"rs_pdomILi8ELi0ELb0", lambda: rsbench_warps(oracle.PDOM, 0)),
    f"rs_spec(T={I.NEXT1.threshold})": (
        r"rs_specILi8ELi0ELb0ELb1E",
        lambda: rsbench_warps(oracle.SPEC_LOOP, I.NEXT1.threshold, pool=True)),
    f"rs_spec_static(T={I.NEXT1.threshold})": (
        r"rs_specILi8ELi0ELb0ELb0E", lambda: rsbench_warps(oracle.SPEC_LOOP, I.NEXT1.threshold)),
    "divloop_pdom_batch": (r"divloop_pdom_batchILi125ELb0",
                           lambda: divloop_warps(oracle.PDOM, 0, batch=True)),
    "divloop_spec_batch(T=16)": (r"divloop_spec_batchILi125ELb0",
                                 lambda: divloop_warps(oracle.SPEC_LOOP, 16, batch=True)),
    "divloop_pool(T=16)": (r"divloop_poolILi125ELb0", lambda: divloop_pool_warps(1)),
    "divloop_pool_split4(T=16)": (r"divloop_pool_splitILi125ELb0ELi4",
                                  lambda: divloop_pool_warps(4)),
    "pt_pdom": (r"pt_pdomILb0E", lambda: pt_warps(oracle.PDOM)),
    f"pt_spec(T={I.C4.threshold})": (r"pt_specILb0ELb1ELb1ELb0ELb0EE",
                                      lambda: pt_warps(oracle.SPEC_LOOP, I.C4.threshold, 8)),
    f"pt_spec_pool(T={I.C4.threshold})": (r"pt_specILb0ELb1ELb1ELb0ELb1EE",
                                           lambda: pt_warps(oracle.SPEC_LOOP_POOL,
                                                            I.C4.threshold, 8)),
    "mcml_pdom": (r"mcml_pdomILb1ELb0ELb1", lambda: mcml_dyn_warps(oracle.PDOM, 0)),
    "mcml_spec(T=32)": (r"mcml_specILb1ELb0ELb1", lambda: mcml_dyn_warps(oracle.SPEC_LOOP, 32)),
}


def inst_scale(label):
    """the sampled-warp cases predict instructions for sample_warps of the launch"""
    if label in ("mcml_pdom", "mcml_spec(T=32)"):
        return MC_DYN["warps"] / MC_DYN["sample_warps"]
    if label.startswith("pt_"):
        return I.C4.n_pixels / 32 / PT_SAMPLE
    return 1.0


def main():
    costs = sass_regions.kernel_costs("divloop_|commoncall_|mcml_|rs_|pt_")
    measured = json.load(open(os.path.join(ROOT, "profiles", "simt_efficiency.json")))
    rows = {}
    cases = [(k, v[0], v[1]) for k, v in CASES.items()]
    for label, pat, gen in cases:
        p = predict(find(costs, pat), gen())
        m = measured.get(label, {})
        rows[label] = dict(predicted=p["simt"], measured=m.get("simt_efficiency"),
                           predicted_inst=p["inst"] * inst_scale(label),
                           measured_inst=m.get("inst"),
                           predicted_thread_inst=p["thread_inst"] * inst_scale(label),
                           measured_thread_inst=m.get("thread_inst"),
                           costs=find(costs, pat))
        if m.get("simt_efficiency") is not None:
            rows[label]["abs_err_points"] = 100 * abs(p["simt"] - m["simt_efficiency"])
    out = json.dumps(rows, indent=1)
    if "--write" in sys.argv:
        open(os.path.join(ROOT, "profiles", "simt_prediction.json"), "w").write(out + "\n")
    print(out)


if __name__ == "__main__":
    main()
