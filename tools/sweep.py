"""Soft-barrier threshold sweep (paper Fig. 9, Sec. 5.3) and launch
tuning on one B200.  Prints one JSON object.

usage: python tools/sweep.py [--what mcml,divloop] [--thresholds 1,2,4,8,16,24,32]
                             [--blocks 512] [--photons N] [--reps 5]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_cgo_damanijskymg20_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_damanijskymg20_b200 import sr  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--what", default="mcml,divloop")
ap.add_argument("--thresholds", default="1,2,4,8,16,24,32")
ap.add_argument("--blocks", default="0")
ap.add_argument("--photons", type=int, default=I.C3.n_photons)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--flags", type=int, default=0, help="extra sr_workload.flags (e.g. 4 = F_COARSE)")
ap.add_argument("--unroll", type=int, default=0, help="merge partial unroll (MC steps, PT node visits, RSBench inner iterations per release)")
ap.add_argument("--defer", type=int, default=0, help="MCML boundary defer threshold T_b")
ap.add_argument("--static", action="store_true", help="MCML static photon assignment (F_STATIC)")
ap.add_argument("--iters", type=int, default=0, help="MCML photons per lane (default configs[2])")
ap.add_argument("--prolog", type=int, default=0, help="RSBench prolog FMAs (expensive task fetch)")
ap.add_argument("--batch", type=int, default=0, help="divloop prolog_batch (0 or 64)")
ap.add_argument("--split", type=int, default=0, help="divloop pool_split (with --flags 32)")
ap.add_argument("--unrolls", default="", help="comma list: sweep the merge unroll too")
a = ap.parse_args()
Ts = [int(x) for x in a.thresholds.split(",")]
blocks = [int(x) for x in a.blocks.split(",")]
stream = torch.cuda.Stream()
ctx = sr.Context.create(0, 1 << 20, stream)
seed = I.PRIMARY_SEED
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timed(fn, reps):
    ms = []
    for i in range(reps + 2):
        with torch.cuda.stream(stream):
            flush.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(stream)
        fn()
        e.record(stream)
        e.synchronize()
        if i >= 2:
            ms.append(s.elapsed_time(e))
    return statistics.median(ms)


def eff(w, n, iters, mode, T):
    wi = sr.Workload.from_buffer_copy(w)
    wi.flags |= sr.F_SCHED
    ctx.ensure(sr.sr_workspace_bytes(wi, n))
    sr.sr_run(wi, n, iters, seed, mode, T)
    s = ctx.region(wi, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    s = s.astype("int64")
    return dict(rounds=int(s[:, 0].sum()), releases=int(s[:, 1].sum()),
                common_lanes=int(s[:, 2].sum()), advances=int(s[:, 3].sum()),
                region_eff=float(s[:, 2].sum() / (32.0 * max(1, s[:, 1].sum()))))


out = {}
if "mcml" in a.what:
    m = I.C3
    iters = a.iters or m.iters
    nt = a.photons // iters
    res = []
    for b in blocks:
        w = sr.mcml_workload(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap,
                             block=b, defer=a.defer, unroll=a.unroll,
                             flags=sr.F_STATIC if a.static else 0)
        ctx.ensure(sr.sr_workspace_bytes(w, nt))
        for mode, T in [(sr.PDOM, 0)] + [(sr.SPEC_LOOP, t) for t in Ts]:
            t = timed(lambda: sr.sr_run(w, nt, iters, seed, mode, T), a.reps)
            r = dict(block=b, mode="pdom" if mode == sr.PDOM else "spec", T=T, ms=t,
                     photons_per_s=nt * iters / (t * 1e-3), launch=sr.sr_last_launch(),
                     unroll=a.unroll, static=a.static, photons=nt * iters)
            r.update(eff(w, min(nt, 65536), iters, mode, T))
            res.append(r)
            print(json.dumps(r), file=sys.stderr, flush=True)
    out["mcml"] = res
if "divloop" in a.what:
    c = I.C1
    res = []
    for b in blocks:
        w = sr.divloop_workload(c.p_u32, c.fma_count, block=b, advance=a.unroll, batch=a.batch,
                                flags=a.flags, split=a.split)
        ctx.ensure(sr.sr_workspace_bytes(w, c.n_threads))
        for mode, T in [(sr.PDOM, 0)] + [(sr.SPEC_LOOP, t) for t in Ts]:
            def run():
                for _ in range(20):
                    sr.sr_run(w, c.n_threads, c.iters, seed, mode, T)
            t = timed(run, a.reps) / 20
            r = dict(block=b, mode="pdom" if mode == sr.PDOM else "spec", T=T, ms=t,
                     thread_iters_per_s=c.n_threads * c.iters / (t * 1e-3))
            r.update(eff(w, c.n_threads, c.iters, mode, T))
            res.append(r)
            print(json.dumps(r), file=sys.stderr, flush=True)
    out["divloop"] = res
if "rsbench" in a.what:
    c = I.NEXT1
    res = []
    Us = [int(x) for x in a.unrolls.split(",")] if a.unrolls else [a.unroll]
    for b, U in [(b, U) for b in blocks for U in Us]:
        w = sr.rsbench_workload(c.fma_count, block=b, prolog_fma=a.prolog, unroll=U, flags=a.flags)
        ctx.ensure(sr.sr_workspace_bytes(w, c.n_threads))
        for mode, T in ([(sr.PDOM, 0)] if U == Us[0] else []) + [(sr.SPEC_LOOP, t) for t in Ts]:
            t = timed(lambda: sr.sr_run(w, c.n_threads, c.iters, seed, mode, T), a.reps)
            r = dict(block=b, mode="pdom" if mode == sr.PDOM else "spec", T=T, ms=t, unroll=U,
                     flags=a.flags,
                     lookups_per_s=c.n_threads * c.iters / (t * 1e-3), launch=sr.sr_last_launch())
            r.update(eff(w, c.n_threads, c.iters, mode, T))
            res.append(r)
            print(json.dumps(r), file=sys.stderr, flush=True)
    out["rsfetch" if a.prolog else "rsbench"] = res
if "pathtrace" in a.what:
    c = I.C4
    tris, mat, mats, cam = I.cornell_scene(c)
    buf, used = sr.upload_scene(tris, mat, mats, cam)
    res = []
    for b in blocks:
        w = sr.pathtrace_workload(buf.data_ptr(), used, c.width, c.height, c.max_depth, block=b,
                                  flags=a.flags, unroll=a.unroll,
                                  pool_spp=c.spp if a.flags & sr.F_POOL else 0)
        ctx.ensure(sr.sr_workspace_bytes(w, c.n_pixels))
        for mode, T in [(sr.PDOM, 0)] + [(sr.SPEC_LOOP, t) for t in Ts]:
            t = timed(lambda: sr.sr_run(w, c.n_pixels, c.spp, seed, mode, T), a.reps)
            r = dict(block=b, mode="pdom" if mode == sr.PDOM else "spec", T=T, ms=t,
                     paths_per_s=c.n_pixels * c.spp / (t * 1e-3), launch=sr.sr_last_launch())
            r.update(eff(w, c.n_pixels, c.spp, mode, T))
            res.append(r)
            print(json.dumps(r), file=sys.stderr, flush=True)
    out["pathtrace"] = res
print(json.dumps(out))
sr.sr_finalize()
