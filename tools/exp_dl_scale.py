"""Divergent loop (configs[0] shape) at other thread counts: how the launch time
scales with warps per SMSP (latency- vs throughput-bound).  CUDA-graph replays.
usage: python tools/exp_dl_scale.py"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cgo_damanijskymg20_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_damanijskymg20_b200 import sr  # noqa: E402

c = I.C1
stream = torch.cuda.Stream()
ctx = sr.Context.create(0, 1 << 24, stream)
out = []
import itertools
for fma, n in itertools.chain(((c.fma_count, n) for n in (592 * 32 // 4, 592 * 32, 32768, 2 * 592 * 32,
                                                          65536, 4 * 592 * 32, 131072, 262144)),
                              ((8, 32768), (0, 32768), (2000, 32768))):
    for name, mode, T, batch, V in (("pdom", sr.PDOM, 0, 0, 1), ("spec", sr.SPEC_LOOP, 16, 0, 8),
                                    ("spec_batch", sr.SPEC_LOOP, 16, 64, 8),
                                    ("pdom_batch", sr.PDOM, 0, 64, 1)):
        w = sr.divloop_workload(c.p_u32, fma, advance=V, batch=batch)
        ctx.ensure(sr.sr_workspace_bytes(w, n))
        sr.sr_run(w, n, c.iters, I.PRIMARY_SEED, mode, T)
        torch.cuda.synchronize()
        ms = []
        for _ in range(7):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record(stream)
            for _ in range(10):
                sr.sr_run(w, n, c.iters, I.PRIMARY_SEED, mode, T)
            e.record(stream)
            e.synchronize()
            ms.append(s.elapsed_time(e) / 10)
        r = dict(n=n, fma=fma, warps=n // 32, warps_per_smsp=n / 32 / 592, kernel=name,
                 us=statistics.median(ms) * 1e3)
        out.append(r)
        print(json.dumps(r), flush=True)
sr.sr_finalize()
