"""Launch each hot-path kernel once (for ncu); no timing, no oracle.

usage: python tools/one_launch.py [divloop] [commoncall] [mcml] [--photons N] [--sched]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_cgo_damanijskymg20_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_damanijskymg20_b200 import sr  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("what", nargs="*", default=["divloop", "commoncall", "mcml", "pathtrace",
                                             "rsbench"])
ap.add_argument("--photons", type=int, default=I.C3.n_photons)
ap.add_argument("--modes", default="pdom,spec")
ap.add_argument("--threshold", type=int, default=32)
ap.add_argument("--static", action="store_true")
ap.add_argument("--iters", type=int, default=0, help="MCML photons per lane (default configs[2]: 64)")
ap.add_argument("--unroll", type=int, default=I.C3.merge_unroll,
                help="MCML merge unroll (default: the bench's, configs[2])")
ap.add_argument("--pt-flags", type=int, default=0, help="extra PATHTRACE flags (F_NOSPLIT = 8)")
ap.add_argument("--dl-batch", type=int, default=0, help="divloop prolog_batch (0 or 64)")
ap.add_argument("--dl-threads", type=int, default=0, help="divloop threads (default configs[0])")
ap.add_argument("--dl-fma", type=int, default=-1, help="divloop FMAs per Expensive (default configs[0])")
ap.add_argument("--dl-flags", type=int, default=0, help="divloop flags (F_POOL = 32)")
ap.add_argument("--dl-split", type=int, default=0, help="divloop pool_split")
ap.add_argument("--rs-flags", type=int, default=0, help="extra RSBENCH flags (F_STATIC = 2)")
a = ap.parse_args()
modes = a.modes.split(",")
ctx = sr.Context.create(0, 1 << 20)
seed = I.PRIMARY_SEED
if "divloop" in a.what:
    c = I.C1
    nth = a.dl_threads or c.n_threads
    w = sr.divloop_workload(c.p_u32, c.fma_count if a.dl_fma < 0 else a.dl_fma,
                            advance=c.advance_unroll, batch=a.dl_batch, flags=a.dl_flags,
                            split=a.dl_split)
    ctx.ensure(sr.sr_workspace_bytes(w, nth))
    for md in modes:
        sr.sr_run(w, nth, c.iters, seed, sr.PDOM if md == "pdom" else sr.SPEC_LOOP,
                  0 if md == "pdom" else c.threshold)
if "commoncall" in a.what:
    c = I.C2
    w = sr.commoncall_workload(c.fma_count, c.split_u32)
    ctx.ensure(sr.sr_workspace_bytes(w, c.n_threads))
    for md in modes:
        sr.sr_run(w, c.n_threads, c.iters, seed, sr.PDOM if md == "pdom" else sr.SPEC_CALL, 0)
if "mcml" in a.what:
    m = I.C3
    iters = a.iters or m.iters
    nt = a.photons // iters
    w = sr.mcml_workload(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap,
                         flags=sr.F_STATIC if a.static else 0, unroll=a.unroll)
    ctx.ensure(sr.sr_workspace_bytes(w, nt))
    for md in modes:
        sr.sr_run(w, nt, iters, seed, sr.PDOM if md == "pdom" else sr.SPEC_LOOP,
                  0 if md == "pdom" else a.threshold)
if "rsbench" in a.what:
    c = I.NEXT1
    w = sr.rsbench_workload(c.fma_count, unroll=c.merge_unroll, flags=a.rs_flags)
    ctx.ensure(sr.sr_workspace_bytes(w, c.n_threads))
    for md in modes:
        sr.sr_run(w, c.n_threads, c.iters, seed, sr.PDOM if md == "pdom" else sr.SPEC_LOOP,
                  0 if md == "pdom" else c.threshold)
if "pathtrace" in a.what:
    c = I.C4
    tris, mat, mats, cam = I.cornell_scene(c)
    buf, used = sr.upload_scene(tris, mat, mats, cam)
    w = sr.pathtrace_workload(buf.data_ptr(), used, c.width, c.height, c.max_depth,
                              flags=a.pt_flags, pool_spp=c.spp if a.pt_flags & sr.F_POOL else 0)
    ctx.ensure(sr.sr_workspace_bytes(w, c.n_pixels))
    for md in modes:
        sr.sr_run(w, c.n_pixels, c.spp, seed, sr.PDOM if md == "pdom" else sr.SPEC_LOOP,
                  0 if md == "pdom" else c.threshold)   # the path tracer's best threshold
torch.cuda.synchronize()
sr.sr_finalize()
print("ok")
