"""CPU baseline of every config (BASELINE.md "CPU baseline plan"): the oracle as
it stands (oracle/, plain single-threaded C), on this host, two numbers per
config:

  1 core     one thread runs a bounded sample of the config's task range;
  all cores  the same oracle on os.cpu_count() threads over disjoint task-id
             ranges (ctypes releases the GIL during each oracle call), the
             integer outputs summed / concatenated -- checked bit-identical to
             a single-thread run of the same ids.

Samples are bounded (seconds each) and stated in the output; throughput is in
each config's own unit.  TEST/EVALUATION INFRASTRUCTURE: calls oracle/.

usage: python tools/cpu_baselines.py [--seconds S] [--out profiles/cpu_baselines_<tag>.json]
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import subprocess
import sys
import time
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from paper_conf_cgo_damanijskymg20_b200 import inputs as I  # noqa: E402


def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                return line.split(":", 1)[1].strip()
    except (OSError, subprocess.SubprocessError):
        pass
    return platform.processor() or "unknown"


def split(n, parts):
    """n tasks into `parts` contiguous ranges (start, count), count > 0."""
    parts = max(1, min(parts, n))
    b = [n * i // parts for i in range(parts + 1)]
    return [(b[i], b[i + 1] - b[i]) for i in range(parts) if b[i + 1] > b[i]]


def run_parallel(fn, n, threads):
    """fn(start, count) -> result, over `threads` disjoint ranges; wall seconds."""
    ranges = split(n, threads)
    t = time.perf_counter()
    with ThreadPoolExecutor(max_workers=len(ranges)) as ex:
        res = list(ex.map(lambda r: fn(*r), ranges))
    return res, time.perf_counter() - t


def calibrate(fn, unit_cost_guess, seconds):
    """Pick a sample size so that fn(0, n) takes about `seconds` on one thread."""
    n = max(1, int(unit_cost_guess))
    t = time.perf_counter()
    fn(0, n)
    dt = max(time.perf_counter() - t, 1e-6)
    return max(1, int(n * seconds / dt))


def measure(name, unit, fn, combine, n_one, n_all, threads, note):
    """One-thread rate on n_one tasks; all-threads rate on n_all tasks.  The
    partition itself is checked on the n_one sample: the threads' outputs,
    combined, equal the single-thread output bit for bit."""
    t = time.perf_counter()
    whole = fn(0, n_one)
    t1 = time.perf_counter() - t
    parts, _ = run_parallel(fn, n_one, threads)
    ok = bool(combine(parts, whole))
    parts = None
    _, tall = run_parallel(fn, n_all, threads)
    return {"config": name, "unit": unit,
            "one_core": {"value": n_one / t1, "sample": n_one, "seconds": t1, "cores": 1},
            "all_cores": {"value": n_all / tall, "sample": n_all, "seconds": tall,
                          "cores": threads, "partition_bit_identical": ok},
            "note": note}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seconds", type=float, default=4.0, help="single-thread seconds per config")
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    ap.add_argument("--only", default="", help="comma list: divloop,commoncall,mcml,rsbench,pathtrace")
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    thr = args.threads
    only = set(args.only.split(",")) if args.only else None
    rows = []
    seed = I.PRIMARY_SEED

    def want(k):
        return only is None or k in only

    if want("divloop"):   # configs[0]: unit = thread-iteration
        c = I.C1

        def f(t0, n):
            return oracle.divloop(t0, n, c.iters, seed, c.p_u32, c.fma_count)

        def comb(parts, whole):
            return all(np.array_equal(np.concatenate([p[i] for p in parts]), whole[i])
                       for i in range(2))
        n1 = min(c.n_threads, calibrate(f, 256, args.seconds))
        r = measure("configs[0] divergent loop", "thread-iterations/s",
                    f, comb, n1, c.n_threads, thr,
                    f"threads [0,n) x {c.iters} iterations; all cores = the full 32768 threads")
        for k in ("one_core", "all_cores"):
            r[k]["value"] *= c.iters
        rows.append(r)

    if want("commoncall"):   # configs[1]: unit = thread
        c = I.C2

        def f(t0, n):
            return oracle.commoncall(t0, n, c.iters, seed, c.split_u32, c.fma_count)

        def comb(parts, whole):
            return all(np.array_equal(np.concatenate([p[i] for p in parts]), whole[i])
                       for i in range(2))
        n1 = min(c.n_threads, calibrate(f, 4096, args.seconds))
        rows.append(measure("configs[1] common call", "threads/s", f, comb, n1,
                            min(c.n_threads, n1 * thr), thr,
                            "thread ids [0,n); all cores: n1 x threads ids (capped at 2^20)"))

    if want("mcml"):   # configs[2] (and configs[4]): unit = photon
        m = I.C3
        p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)

        def f(t0, n):
            return oracle.mcml(p, t0, n, seed)

        def comb(parts, whole):
            s = {k: sum(q[k].astype(np.uint64) for q in parts) for k in ("A", "Rd", "Tt")}
            cr = sum(q["counters_raw"] for q in parts)
            return all(np.array_equal(s[k], whole[k]) for k in s) and \
                np.array_equal(cr, whole["counters_raw"])
        n1 = calibrate(f, 2048, args.seconds)
        rows.append(measure("configs[2] Monte Carlo 3-layer slab", "photons/s", f, comb, n1,
                            n1 * thr, thr,
                            "photon ids [0,n); integer tallies summed over the threads"))

    if want("rsbench"):   # NEXT-1: unit = lookup
        c = I.NEXT1

        def f(t0, n):
            return oracle.rsbench(t0, n, c.iters, seed, c.fma_count)

        def comb(parts, whole):
            return all(np.array_equal(np.concatenate([p[i] for p in parts]), whole[i])
                       for i in range(2))
        n1 = min(c.n_threads, calibrate(f, 1024, args.seconds))
        r = measure("NEXT-1 RSBench shape", "lookups/s", f, comb, n1,
                    min(c.n_threads, n1 * thr), thr, f"threads [0,n) x {c.iters} lookups")
        for k in ("one_core", "all_cores"):
            r[k]["value"] *= c.iters
        rows.append(r)

    if want("pathtrace"):   # configs[3]: unit = path (brute-force closest hit, no BVH)
        c = I.C4
        tris, mat, mats, cam = I.cornell_scene(c)
        sc = oracle.pt_scene(tris, mat, mats, cam)
        rng = np.random.default_rng(seed)
        pix = rng.permutation(c.n_pixels).astype(np.uint32)   # a spread pixel subset

        def f(t0, n):
            return oracle.pt_render(sc, c.width, c.height, c.spp, c.max_depth, seed,
                                    pixels=pix[t0:t0 + n])

        def comb(parts, whole):
            return np.array_equal(np.concatenate([q[0] for q in parts]), whole[0])
        n1 = max(1, calibrate(f, 1, args.seconds))
        r = measure("configs[3] path tracer", "paths/s", f, comb, n1, n1 * thr, thr,
                    f"seeded random pixel subset x {c.spp} spp, brute-force closest hit over "
                    f"{len(mat)} triangles (the oracle has no BVH)")
        for k in ("one_core", "all_cores"):
            r[k]["value"] *= c.spp
        rows.append(r)

    out = {"host": {"cpu_model": cpu_model(), "os_cpu_count": os.cpu_count(),
                    "threads_used": thr},
           "oracle_build": "gcc -O2 -ffp-contract=off -fno-fast-math (oracle/build)",
           "configs": rows}
    s = json.dumps(out, indent=1)
    if args.out:
        with open(args.out, "w") as fh:
            fh.write(s + "\n")
    print(s)


if __name__ == "__main__":
    main()
