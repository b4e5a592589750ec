"""Every *_pdom / *_spec kernel variant once, at small sizes, for compute-sanitizer
(tests/test_gpu_sanitizer.py runs this under --tool memcheck / racecheck / synccheck).

The warp-synchronous kernels use computed masks (`__syncwarp(P)` inside
`if (parked)`, `__ballot_sync` over the full warp with invalid lanes taking
part, shared-memory tally staging and traversal stacks): the constructs the
paper warns need explicit masks (Sec. 6).  Sizes are small and
ragged (a partial last warp and CTA) so that the invalid-lane paths run too.

usage: python tools/sanitize_run.py [family ...]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_cgo_damanijskymg20_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_damanijskymg20_b200 import sr  # noqa: E402

what = sys.argv[1:] or ["divloop", "commoncall", "mcml", "rsbench", "pathtrace"]
seed = I.PRIMARY_SEED
ctx = sr.Context.create(0, 1 << 22)
launches = 0


def run(w, n, iters, mode, thr):
    global launches
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, iters, seed, mode, thr)
    launches += 1


if "divloop" in what:
    c = I.C1
    for flags in (0, sr.F_SCHED):
        for adv in (1, 8):
            for batch, iters in ((0, 16), (64, 16), (64, 70)):
                w = sr.divloop_workload(c.p_u32, 64, advance=adv, flags=flags, batch=batch)
                run(w, 1000, iters, sr.PDOM, 0)
                for T in (1, 16, 32):
                    run(w, 1000, iters, sr.SPEC_LOOP, T)
                if batch:
                    for split in (1, 2, 4):
                        wp = sr.divloop_workload(c.p_u32, 64, advance=adv, flags=flags | sr.F_POOL,
                                                 batch=batch, split=split)
                        run(wp, 1000, iters, sr.SPEC_LOOP, 16)
    # one block of 1024 threads with n = 1 (31 whole warps past n)
    run(sr.divloop_workload(c.p_u32, 64, flags=sr.F_SCHED, block=1024), 1, 16, sr.SPEC_LOOP, 16)
if "commoncall" in what:
    w = sr.commoncall_workload(64, I.C2.split_u32)
    for mode in (sr.PDOM, sr.SPEC_CALL):
        run(w, 1000, 1, mode, 0)
if "mcml" in what:
    m = I.C3
    for flags in (0, sr.F_SCHED, sr.F_STATIC, sr.F_STATIC | sr.F_SCHED):
        for unroll, defer in ((1, 0), (4, 0), (1, 8)):
            w = sr.mcml_workload(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz,
                                 m.step_cap, flags=flags, unroll=unroll, defer=defer)
            run(w, 333, 2, sr.PDOM, 0)
            for T in (8, 32):
                run(w, 333, 2, sr.SPEC_LOOP, T)
if "rsbench" in what:
    for prolog in (0, 256):
        for unroll in (1, 4, 12):
            for flags in (0, sr.F_SCHED, sr.F_STATIC, sr.F_STATIC | sr.F_SCHED):
                w = sr.rsbench_workload(64, prolog_fma=prolog, unroll=unroll, flags=flags)
                run(w, 1000, 4, sr.PDOM, 0)
                for T in (1, 24, 32):
                    run(w, 1000, 4, sr.SPEC_LOOP, T)
if "pathtrace" in what:
    import dataclasses
    c = dataclasses.replace(I.C4_SMALL, width=20, height=17)   # ragged: 340 lanes
    tris, mat, mats, cam = I.cornell_scene(c)
    buf, used = sr.upload_scene(tris, mat, mats, cam)
    n = c.width * c.height
    for flags in (0, sr.F_SCHED, sr.F_NOSPLIT, sr.F_COARSE, sr.F_MATGROUP, sr.F_MATGROUP | sr.F_SCHED,
                  sr.F_POOL, sr.F_POOL | sr.F_SCHED):
        w = sr.pathtrace_workload(buf.data_ptr(), used, c.width, c.height, c.max_depth,
                                  flags=flags, pool_spp=2 if flags & sr.F_POOL else 0)
        run(w, n, 2, sr.PDOM, 0)
        for T in (12, 32):
            run(w, n, 2, sr.SPEC_LOOP, T)
torch.cuda.synchronize()
sr.sr_finalize()
print(f"sanitize_run: {launches} launches ok")
