"""The oracle run on every host core (TEST INFRASTRUCTURE, imports oracle/ only).

The oracle is single-threaded C; these helpers split the task range into disjoint pieces and
call it from a thread pool (ctypes releases the GIL during each call), then put the pieces
back together: integer tallies are summed (addition of uint64 is associative, so the sum is
bit-identical to one call over the whole range), per-thread / per-pixel outputs are
concatenated in task order.  No arithmetic of the method happens here.
"""
from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

import oracle


def cores() -> int:
    return os.cpu_count() or 1


def _ranges(total: int, parts: int):
    b = [total * i // parts for i in range(parts + 1)]
    return [(b[i], b[i + 1] - b[i]) for i in range(parts) if b[i + 1] > b[i]]


def mcml(p, id0: int, count: int, seed: int, parts: int | None = None):
    parts = parts or 4 * cores()
    with ThreadPoolExecutor(max_workers=cores()) as ex:
        outs = list(ex.map(lambda r: oracle.mcml(p, id0 + r[0], r[1], seed), _ranges(count, parts)))
    res = {k: sum(o[k] for o in outs) for k in ("A", "Rd", "Tt", "counters_raw")}
    return res


def rsbench(t0: int, n: int, iters: int, seed: int, fma_count: int, prolog_fma: int = 0):
    with ThreadPoolExecutor(max_workers=cores()) as ex:
        outs = list(ex.map(lambda r: oracle.rsbench(t0 + r[0], r[1], iters, seed, fma_count,
                                                    prolog_fma=prolog_fma),
                           _ranges(n, 4 * cores())))
    return np.concatenate([o[0] for o in outs]), np.concatenate([o[1] for o in outs])


def pt_render(scene, width, height, spp, max_depth, seed, pixels):
    pixels = np.ascontiguousarray(pixels, np.uint32)
    chunks = [pixels[a:a + c] for a, c in _ranges(len(pixels), 4 * cores())]
    with ThreadPoolExecutor(max_workers=cores()) as ex:
        outs = list(ex.map(lambda px: oracle.pt_render(scene, width, height, spp, max_depth, seed,
                                                       pixels=px), chunks))
    rgb = np.concatenate([o[0] for o in outs])
    cnt = {k: sum(o[1][k] for o in outs) for k in outs[0][1]}
    return rgb, cnt
