#!/usr/bin/env python
"""Benchmark of the Speculative Reconvergence hot path on B200.

Contract (driver): ``python bench.py --gpus N --steps K --warmup W`` prints ONE
JSON line on rank 0.  For N > 1 it is launched under torch.distributed.run, one
process per GPU, NCCL.

Headline workload: Monte Carlo photon transport in the
3-layer slab, Loop Merge (SR_SPEC_LOOP, T=32) -- one step = one sr_run over the
rank's photon shard plus, for N > 1, one NCCL all-reduce of the integer tallies.
N = 1: configs[2] (10^7 photons).  N > 1: configs[4], 10^9 photons in total split
over the N ranks (strong scaling); rank 0 also times the whole 10^9 alone (t_1 of
E_N = t_1/(N t_N)) and the line carries the weak-scaled 10^7-per-rank numbers
under "scaling_detail".  The PDOM kernel is timed the same way
("pdom" key).  At N = 1 the two microbenchmarks (configs[0], configs[1]) are
timed too ("configs" key), PDOM vs SPEC.

``--impl reference`` times the CPU oracle (oracle/, plain single-threaded C) on
a bounded sample of the same workload instead -- the reference arm of this
tier (there is no reference program to install).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "samples/sec and ncu SIMT efficiency, speculative vs PDOM, at 1/2/4/8 B200"
UNIT = "photons/s"
PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
PROFILE_CONST = os.path.join(ROOT, "profiles", "work_per_unit.json")
L2_FLUSH_BYTES = 256 << 20  # > 126 MB L2


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--threshold", type=int, default=32)
    ap.add_argument("--photons-per-gpu", type=int, default=0,
                    help="override the per-rank photon count of N = 1 / weak runs "
                         "(default: configs[2] = 10^7)")
    ap.add_argument("--total-photons", type=int, default=0,
                    help="N > 1 strong scaling: photons of the whole job (default: configs[4] "
                         "= 10^9)")
    ap.add_argument("--scaling", default="auto", choices=["auto", "strong", "weak"],
                    help="N > 1: strong (configs[4], default) or weak (10^7 per rank)")
    ap.add_argument("--t1-steps", type=int, default=2,
                    help="N > 1: timed single-GPU runs of the whole job (t_1 of E_N)")
    ap.add_argument("--block", type=int, default=0, help="MCML CTA size (0 = library default)")
    ap.add_argument("--unroll", type=int, default=0,
                    help="MCML steps per release (0 = inputs.C3.merge_unroll)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo: test the N>1 plumbing on one GPU (ranks share it)")
    ap.add_argument("--no-configs", action="store_true", help="skip the microbenchmark lines")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    return ap.parse_args()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi sampling DURING the timed region (B200_PROFILING.md)."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
            self.t.join(timeout=2)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if len(r) > 1 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) > 2 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, n in enumerate(names):
                if len(r) > 5 + i and r[5 + i].lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "samples": len(self.rows)}


# ---------------------------------------------------------------- timing
class Timer:
    """Per-step CUDA events on the launching stream; an L2 flush (a 256 MB
    write) between timed steps, outside the events."""

    def __init__(self, torch, stream):
        self.torch = torch
        self.stream = stream
        self.flush_buf = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=stream.device)

    def flush(self):
        with self.torch.cuda.stream(self.stream):
            self.flush_buf.fill_(1)

    def time_steps(self, fn, steps, warmup, barrier=None):
        torch = self.torch
        for _ in range(warmup):
            self.flush()
            fn()
        torch.cuda.synchronize()
        if barrier:
            barrier()
        torch.cuda.synchronize()
        ms = []
        for _ in range(steps):
            self.flush()
            s = torch.cuda.Event(enable_timing=True)
            e = torch.cuda.Event(enable_timing=True)
            s.record(self.stream)
            fn()
            e.record(self.stream)
            e.synchronize()
            ms.append(s.elapsed_time(e))
        torch.cuda.synchronize()
        if barrier:
            barrier()
        torch.cuda.synchronize()
        return ms


def load_json(path):
    try:
        with open(path) as f:
            return json.load(f)
    except (OSError, ValueError):
        return None


# ---------------------------------------------------------------- reference arm
def cpu_sample(photons: int, seed: int):
    """The oracle, as it stands, single-threaded on this host: photons/s."""
    import oracle
    from paper_conf_cgo_damanijskymg20_b200 import inputs as I
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    t = time.perf_counter()
    oracle.mcml(p, 0, photons, seed)
    return photons / (time.perf_counter() - t)


def cpu_sample_threads(photons: int, seed: int, threads: int):
    """The same oracle on `threads` host threads over disjoint photon-id ranges
    (ctypes releases the GIL inside each oracle call; integer tallies add up to
    the single-thread result bit for bit, tools/cpu_baselines.py checks it)."""
    from concurrent.futures import ThreadPoolExecutor

    import oracle
    from paper_conf_cgo_damanijskymg20_b200 import inputs as I
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    b = [photons * i // threads for i in range(threads + 1)]
    t = time.perf_counter()
    with ThreadPoolExecutor(max_workers=threads) as ex:
        list(ex.map(lambda i: oracle.mcml(p, b[i], b[i + 1] - b[i], seed), range(threads)))
    return photons / (time.perf_counter() - t)


def cpu_baseline(I, seconds=8.0):
    """cpu_baseline leg (rank 0, N = 1): ~`seconds` of single-thread oracle work,
    then ~`seconds` wall on every host core; value = the all-cores rate."""
    t = time.perf_counter()
    v1 = cpu_sample(1024, I.PRIMARY_SEED)
    n1 = max(1024, int(v1 * seconds))
    v1 = cpu_sample(n1, I.PRIMARY_SEED)
    cores = os.cpu_count() or 1
    n_all = max(cores, int(v1 * seconds) * cores)
    v_all = cpu_sample_threads(n_all, I.PRIMARY_SEED, cores)
    return {"value": v_all, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"photon ids [0,{n_all}) of configs[2], {cores} host threads over "
                      f"disjoint id ranges",
            "single_core": {"value": v1, "cores": 1,
                            "sample": f"photon ids [0,{n1}) of configs[2], one thread"},
            "seconds": time.perf_counter() - t}


def run_reference(args):
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    from paper_conf_cgo_damanijskymg20_b200 import inputs as I
    cores = os.cpu_count() or 1
    sample = 8192 * cores  # ~0.2-0.4 s of oracle work per thread per step
    for _ in range(args.warmup):
        cpu_sample_threads(sample // 8, I.PRIMARY_SEED, cores)
    vals = [cpu_sample_threads(sample, I.PRIMARY_SEED, cores) for _ in range(args.steps)]
    v = statistics.median(vals)
    desc = (f"photon ids [0,{sample}) of configs[2] per step, {cores} host threads over "
            f"disjoint id ranges")
    out = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": sample / v * 1e3,
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
           "data": "synthetic",
           "config": {"workload": f"mcml-3layer (configs[2]) {desc}",
                      "photons_per_gpu": I.C3.n_photons, "seed": I.PRIMARY_SEED},
           "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
                            "sample": desc},
           "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# ---------------------------------------------------------------- our arm
def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    from paper_conf_cgo_damanijskymg20_b200 import inputs as I
    from paper_conf_cgo_damanijskymg20_b200 import parallel as P
    from paper_conf_cgo_damanijskymg20_b200 import sr

    ws_n, rank, local = dist_env()
    if args.dist_backend == "gloo":
        # plumbing check of the multi-rank path with fewer GPUs than ranks
        local = local % max(1, torch.cuda.device_count())
    if ws_n > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
        else:
            dist.init_process_group("gloo")
    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    stream = torch.cuda.Stream(device=dev)
    sr.load()  # raises if libsr.so is missing: no fallback

    m = I.C3
    iters = m.iters
    T = args.threshold
    unroll = args.unroll if args.unroll else m.merge_unroll
    # N = 1: configs[2] (10^7 photons).  N > 1: configs[4] -- a fixed total of
    # 10^9 photons split over the ranks (strong scaling),
    # unless --scaling weak keeps 10^7 (or --photons-per-gpu) per rank.
    strong = ws_n > 1 and args.scaling != "weak"
    if strong:
        total = args.total_photons or I.C5_TOTAL_PHOTONS
        nt_total = (total + iters - 1) // iters
        lane0, nt = P.split_even(nt_total, ws_n, rank)
        total = nt_total * iters
        offset = lane0 * iters
    else:
        per_rank = args.photons_per_gpu or m.n_photons
        nt = (per_rank + iters - 1) // iters
        total = nt * iters * ws_n
        offset = P.task_offset_of(rank, nt * iters)
    per_rank = nt * iters

    def mc_workload(task_offset, flags=0):
        return sr.mcml_workload(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz,
                                m.step_cap, task_offset=task_offset, block=args.block,
                                unroll=unroll, flags=flags)

    w = mc_workload(offset)
    nbytes = sr.sr_workspace_bytes(w, nt)
    ctx = sr.Context.create(local, nbytes, stream)
    off, tb = sr.sr_workspace_region(w, nt, sr.T_GRID)
    _, cb = sr.sr_workspace_region(w, nt, sr.T_COUNTERS)
    barrier = (lambda: dist.barrier()) if ws_n > 1 else None
    timer = Timer(torch, stream)

    def tallies_view():   # GRID + COUNTERS, contiguous (re-taken: ctx.ensure may reallocate)
        return ctx.workspace[off:off + tb + cb].view(torch.int64)

    def step(mode, thr):
        sr.sr_run(w, nt, iters, I.PRIMARY_SEED, mode, thr)
        P.allreduce_tallies(tallies_view(), stream=stream)   # no-op at N = 1

    # device-timed region, SPEC (headline) with clocks sampled during it
    with ClockSampler(local) as clk:
        ms_spec = timer.time_steps(lambda: step(sr.SPEC_LOOP, T), args.steps, args.warmup, barrier)
    launch_spec = sr.sr_last_launch()
    ms_pdom = timer.time_steps(lambda: step(sr.PDOM, 0), args.steps, args.warmup, barrier)
    launch_pdom = sr.sr_last_launch()

    def max_over_ranks(x):
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        if ws_n > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    t_spec = max_over_ranks(statistics.mean(ms_spec))

    # the step's one collective timed alone (N > 1): the tally all-reduce over
    # GRID+COUNTERS, CUDA events on the launching stream, max over ranks -- the
    # measurement behind DESIGN.md's NEXT-4 decision (fusing it into the kernel
    # tail cannot move a step it is this small a share of)
    coll = None
    if ws_n > 1:
        def allreduce_only():
            P.allreduce_tallies(tallies_view(), stream=stream)
        ms_ar = timer.time_steps(allreduce_only, args.steps, args.warmup, barrier)
        t_ar = max_over_ranks(statistics.mean(ms_ar))
        coll = {"op": f"all_reduce(SUM) int64, {args.dist_backend}", "bytes": tb + cb,
                "ms": t_ar, "share_of_step": t_ar / t_spec}
    t_pdom = max_over_ranks(statistics.mean(ms_pdom))
    value = total / (t_spec * 1e-3)
    pdom_value = total / (t_pdom * 1e-3)

    # end to end through the public API: sr_run + (all-reduce) + sr_tally into
    # pinned host memory, host wall clock per step, max over ranks
    host = torch.empty(tb + cb, dtype=torch.uint8, pin_memory=True)
    import ctypes
    h2d = ctypes.sizeof(sr.Workload)   # the step's inputs: the workload descriptor
    e2e_ms = []
    for i in range(args.warmup + args.steps):
        torch.cuda.synchronize()
        if barrier:
            barrier()
        t0 = time.perf_counter()
        step(sr.SPEC_LOOP, T)
        sr.sr_tally(sr.T_GRID, host.data_ptr(), tb)
        sr.sr_tally(sr.T_COUNTERS, host.data_ptr() + tb, cb)
        t1 = time.perf_counter()
        if i >= args.warmup:
            e2e_ms.append((t1 - t0) * 1e3)
    t_e2e = max_over_ranks(statistics.mean(e2e_ms))
    counters = host[tb:tb + cb].view(torch.int64).numpy()
    steps_total = int(counters[1])  # after all-reduce: whole job
    assert int(counters[0]) == total, "photon count mismatch"

    # schedule-level efficiency of the common code (instrumented kernels, outside timing)
    def region_eff(mode, thr):
        wi = sr.mcml_workload(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz,
                              m.step_cap, task_offset=offset,
                              flags=sr.F_SCHED)   # U = 1: lanes per merged-loop iteration
        ni = min(nt, 32768)
        ctx.ensure(sr.sr_workspace_bytes(wi, ni))
        sr.sr_run(wi, ni, iters, I.PRIMARY_SEED, mode, thr)
        s = ctx.region(wi, ni, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS)
        s = s.cpu().numpy().astype("int64")
        rel, lanes = s[:, 1].sum(), s[:, 2].sum()
        return float(lanes / (32.0 * rel)) if rel else None

    eff_spec = region_eff(sr.SPEC_LOOP, T)
    eff_pdom = region_eff(sr.PDOM, 0)

    # N > 1: the whole job once more on rank 0 alone, in ONE launch per step over
    # every photon id [0, total): (i) the all-reduced tallies of the sharded run
    # must equal it bit for bit (SURVEY.md Sec. 8(e) invariant); (ii) strong
    # scaling: its device time is t_1 of E_N = t_1 / (N t_N)
    same_as_one_gpu = None
    scaling = None
    if ws_n > 1:
        t1 = None
        if rank == 0:
            w_all = mc_workload(0)
            nt_all = total // iters
            ctx.ensure(sr.sr_workspace_bytes(w_all, nt_all))
            ms_1 = timer.time_steps(
                lambda: sr.sr_run(w_all, nt_all, iters, I.PRIMARY_SEED, sr.SPEC_LOOP, T),
                args.t1_steps, 1)
            t1 = statistics.mean(ms_1)
            ref = torch.empty(tb + cb, dtype=torch.uint8, pin_memory=True)
            sr.sr_tally(sr.T_GRID, ref.data_ptr(), tb)
            sr.sr_tally(sr.T_COUNTERS, ref.data_ptr() + tb, cb)
            same_as_one_gpu = bool(torch.equal(ref, host))
        dist.barrier()
        # the other reading of configs[4]: a fixed 10^7 photons per rank (weak)
        nt_w = m.n_photons // iters
        w_weak = mc_workload(P.task_offset_of(rank, nt_w * iters))
        ctx.ensure(sr.sr_workspace_bytes(w_weak, nt_w))

        def weak_step():
            sr.sr_run(w_weak, nt_w, iters, I.PRIMARY_SEED, sr.SPEC_LOOP, T)
            P.allreduce_tallies(tallies_view(), stream=stream)
        t_weak = max_over_ranks(statistics.mean(
            timer.time_steps(weak_step, args.steps, args.warmup, barrier)))
        if rank == 0:
            v1 = total / (t1 * 1e-3)
            scaling = {
                "kind": "strong" if strong else "weak",
                "t1_ms": t1, "t1_value": v1,
                "t1_basis": f"rank 0 alone, all {total} photons in one launch per step, "
                            f"{args.t1_steps} timed steps",
                "efficiency": (t1 / (ws_n * t_spec)) if strong else value / (ws_n * v1),
                "efficiency_basis": ("E_N = t_1 / (N t_N), SURVEY.md Sec. 8(e)" if strong else
                                     "value_N / (N x t1_value)"),
                "weak": {"photons_per_gpu": nt_w * iters, "ms_per_step": t_weak,
                         "value": ws_n * nt_w * iters / (t_weak * 1e-3)}}

    peaks = load_json(PEAKS_FILE) or {}
    consts = load_json(PROFILE_CONST) or {}
    clocks = clk.summary()
    result = None
    if rank == 0:
        # roofline: issue-bound (plain ALU), algorithmic thread-instructions =
        # PDOM thread-instructions per photon-step (ncu, profiles/) x steps
        ipu = consts.get("mcml_thread_inst_per_step")
        f_mhz = peaks.get("sm_max_mhz", 1965.0)
        peak = 32 * 4 * 148 * f_mhz * 1e6 / 1e12   # T thread-inst/s
        rl = None
        if ipu:
            ach = ipu * steps_total / ws_n / (t_spec * 1e-3) / 1e12
            rl = {"bound": "alu", "achieved": ach, "peak": peak, "unit": "Tthread-inst/s",
                  "frac": ach / peak, "traffic": consts.get("mcml_spec_dram_bytes_per_launch"),
                  "kernel": "mcml_spec",
                  "peak_basis": f"592 SMSPs x 32 lanes x {f_mhz:.0f} MHz (sm_max_mhz of measured)",
                  "work_basis": "profiles/work_per_unit.json: PDOM thread-inst per photon step (ncu)"}
        if strong:
            workload_name = f"mcml-3layer configs[4]: {total} photons sharded over {ws_n} GPUs"
        elif ws_n > 1:
            workload_name = f"mcml-3layer configs[2] shape, {per_rank} photons per GPU (weak)"
        else:
            workload_name = f"mcml-3layer configs[2]: {total} photons"
        result = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws_n, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_spec, "higher_is_better": True,
            "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic",
            "config": {"workload": workload_name, "total_photons": total,
                       "photons_per_gpu": per_rank, "lanes": nt, "photons_per_lane": iters,
                       "threshold": T, "mode": "SPEC_LOOP", "seed": I.PRIMARY_SEED,
                       "merge_unroll": args.unroll if args.unroll else m.merge_unroll,
                       "l2": "flushed (256 MB write) between timed steps",
                       "launch": launch_spec, "launch_pdom": launch_pdom,
                       "parallelism": f"dp{ws_n} (photon-id shards + 1 "
                                      f"{args.dist_backend.upper()} int64 all-reduce)"},
            "pdom": {"value": pdom_value, "unit": UNIT, "ms_per_step": t_pdom},
            "speedup_vs_pdom": value / pdom_value,
            "common_region_efficiency": {"pdom": eff_pdom, "spec": eff_spec,
                                         "source": "per-warp schedule counters (SR_F_SCHED)"},
            "steps_per_photon": steps_total / total,
            "clocks": clocks,
            "e2e": {"value": total / (t_e2e * 1e-3), "unit": UNIT, "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": tb + cb},
            "gpu_launches": args.steps,
            "roofline": rl,
            "collective": coll,
            "tallies_equal_single_gpu_run": same_as_one_gpu,
            "scaling_detail": scaling,
        }
        simt = load_json(os.path.join(ROOT, "profiles", "simt_efficiency.json"))
        if simt:
            result["simt_efficiency_ncu"] = simt
    if ws_n > 1:
        dist.barrier()
    if rank == 0 and ws_n == 1 and not args.no_configs:
        result["configs"] = microbench_configs(torch, sr, I, ctx, stream, timer, args)
    if rank == 0 and ws_n == 1 and not args.no_cpu:
        result["cpu_baseline"] = cpu_baseline(I)
    if rank == 0:
        print(json.dumps(result), flush=True)
    sr.sr_finalize()
    if ws_n > 1:
        dist.destroy_process_group()


def microbench_configs(torch, sr, I, ctx, stream, timer, args):
    """configs[0] and configs[1]: PDOM vs SPEC, CUDA-graph replays of R launches."""
    out = {}
    peaks = load_json(PEAKS_FILE) or {}
    f_mhz = peaks.get("sm_max_mhz", 1965.0)
    fma_peak = 128 * 148 * f_mhz * 1e6  # FP32 FMA/s (FFMA2 = 2 per lane)

    def graph_time(w, n, iters, mode, thr, reps=20):
        ctx.ensure(sr.sr_workspace_bytes(w, n))
        g = torch.cuda.CUDAGraph()
        cap = torch.cuda.Stream(device=stream.device)
        sr.sr_init(ctx.device, cap.cuda_stream, ctx.workspace.data_ptr(), ctx.workspace.numel())
        sr.sr_run(w, n, iters, I.PRIMARY_SEED, mode, thr)  # warm (module load, attributes)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=cap):
            for _ in range(reps):
                sr.sr_run(w, n, iters, I.PRIMARY_SEED, mode, thr)
        sr.sr_init(ctx.device, stream.cuda_stream, ctx.workspace.data_ptr(), ctx.workspace.numel())

        def replay():
            with torch.cuda.stream(stream):   # the events are recorded on `stream`
                g.replay()
        ms = timer.time_steps(replay, max(args.steps, 5), args.warmup)
        return statistics.median(ms) / reps

    c = I.C1
    n_units = c.n_threads * c.iters
    exp_calls = None
    res = {}
    # as written (one Philox draw per iteration, in program order) and with the
    # conditions of 64 iterations evaluated together (prolog_batch, reading Q5') --
    # both kernels get the same prolog.  V = run-ahead iterations per advance round
    # (V = 1: the paper's one vote per iteration; V = 8 the default).  T = 16 is the
    # config's threshold; T = 32 = wait for every lane (Fig. 1(b)).
    # "pool": Loop Merge of the Expensive() calls over a warp task pool after the
    # batched prologs (SR_F_POOL; pool_split warps per 32 threads) -- beyond the paper's
    # Iteration Delay, which keeps each thread's calls on its own lane
    runs = (("pdom", sr.PDOM, 0, 1, 0, 0, 0), ("spec_t16", sr.SPEC_LOOP, 16, c.advance_unroll, 0, 0, 0),
            ("spec_t16_v1", sr.SPEC_LOOP, 16, 1, 0, 0, 0),
            ("spec_t8", sr.SPEC_LOOP, 8, c.advance_unroll, 0, 0, 0),
            ("spec_t32", sr.SPEC_LOOP, 32, c.advance_unroll, 0, 0, 0),
            ("pdom_batch", sr.PDOM, 0, 1, 64, 0, 0),
            ("spec_t16_batch", sr.SPEC_LOOP, 16, c.advance_unroll, 64, 0, 0),
            ("spec_t16_v1_batch", sr.SPEC_LOOP, 16, 1, 64, 0, 0),
            ("spec_t8_batch", sr.SPEC_LOOP, 8, c.advance_unroll, 64, 0, 0),
            ("spec_t32_batch", sr.SPEC_LOOP, 32, c.advance_unroll, 64, 0, 0),
            ("pool", sr.SPEC_LOOP, 16, c.advance_unroll, 64, sr.F_POOL, 1),
            (f"pool_split{c.pool_split}", sr.SPEC_LOOP, 16, c.advance_unroll, 64, sr.F_POOL,
             c.pool_split))
    for name, mode, thr, V, batch, fl, split in runs:
        w = sr.divloop_workload(c.p_u32, c.fma_count, advance=V, batch=batch, flags=fl, split=split)
        t = graph_time(w, c.n_threads, c.iters, mode, thr)
        sr.sr_run(w, c.n_threads, c.iters, I.PRIMARY_SEED, mode, thr)
        exp_calls = int(ctx.region(w, c.n_threads, sr.T_COUNTERS, torch.int64)[0].item())
        res[name] = {"value": n_units / (t * 1e-3), "unit": "thread-iterations/s", "ms": t,
                     "advance_unroll": V, "prolog_batch": batch, "pool_split": split if fl else None,
                     "fma_frac_of_peak": exp_calls * c.fma_count / (t * 1e-3) / fma_peak}
    res["speedup_pool_vs_pdom"] = res[f"pool_split{c.pool_split}"]["value"] / res["pdom"]["value"]
    for k in ("t16", "t16_v1", "t8", "t32"):
        res[f"speedup_{k}_vs_pdom"] = res[f"spec_{k}"]["value"] / res["pdom"]["value"]
        res[f"speedup_{k}_batch_vs_pdom_batch"] = (res[f"spec_{k}_batch"]["value"] /
                                                  res["pdom_batch"]["value"])
    res["expensive_calls"] = exp_calls
    # issue roofline: useful work = the as-written PDOM kernel's thread-instructions
    # (ncu, profiles/simt_efficiency.json), peak = 592 SMSPs x 32 lanes x f
    simt = load_json(os.path.join(ROOT, "profiles", "simt_efficiency.json")) or {}
    ti = (simt.get("divloop_pdom") or {}).get("thread_inst")
    if ti:
        peak = 592 * 32 * f_mhz * 1e6
        res["issue_roofline"] = {
            "thread_inst": ti,
            "frac": {k: ti / (v["ms"] * 1e-3) / peak for k, v in res.items()
                     if isinstance(v, dict) and "ms" in v},
            "basis": "as-written PDOM thread-inst (ncu) / time / (592 x 32 x sm_max_mhz)"}
    out["divloop"] = res

    c = I.C2
    w = sr.commoncall_workload(c.fma_count, c.split_u32)
    res = {}
    for name, mode in (("pdom", sr.PDOM), ("spec_call", sr.SPEC_CALL)):
        t = graph_time(w, c.n_threads, c.iters, mode, 0, reps=5)
        res[name] = {"value": c.n_threads / (t * 1e-3), "unit": "threads/s", "ms": t,
                     "fma_frac_of_peak": c.n_threads * c.fma_count / (t * 1e-3) / fma_peak}
    res["speedup_vs_pdom"] = res["spec_call"]["value"] / res["pdom"]["value"]
    out["commoncall"] = res

    # NEXT-1: RSBench-shaped nested trip-count loop (Fig. 3), PDOM vs Loop Merge
    c = I.NEXT1
    res = {}
    # default: the warp task pool; "_static": lane l runs thread l's lookups itself
    for name, mode, thr, flags in (("pdom", sr.PDOM, 0, 0),
                                   (f"spec_t{c.threshold}", sr.SPEC_LOOP, c.threshold, 0),
                                   (f"spec_t{c.threshold}_static", sr.SPEC_LOOP, c.threshold,
                                    sr.F_STATIC)):
        w = sr.rsbench_workload(c.fma_count, unroll=c.merge_unroll, flags=flags)
        t = graph_time(w, c.n_threads, c.iters, mode, thr, reps=5)
        sr.sr_run(w, c.n_threads, c.iters, I.PRIMARY_SEED, mode, thr)
        nucs = int(ctx.region(w, c.n_threads, sr.T_COUNTERS, torch.int64)[0].item())
        # FMA roofline: every nuclide body is fma_count FMAs (FFMA2, reading R8)
        res[name] = {"value": c.n_threads * c.iters / (t * 1e-3), "unit": "lookups/s", "ms": t,
                     "fma_frac_of_peak": nucs * c.fma_count / (t * 1e-3) / fma_peak}
    res["speedup_vs_pdom"] = res[f"spec_t{c.threshold}"]["value"] / res["pdom"]["value"]
    res["nuclides"] = nucs
    out["rsbench"] = res

    # ... with an expensive task fetch (2048-FMA prolog, Fig. 9's XSBench case):
    # refilling idle lanes costs more, the best threshold drops (T = 32 shown too)
    c = I.NEXT1_FETCH
    res = {"prolog_fma": c.prolog_fma}
    for name, mode, thr, flags in (("pdom", sr.PDOM, 0, 0),
                                   (f"spec_t{c.threshold}", sr.SPEC_LOOP, c.threshold, 0),
                                   ("spec_t32", sr.SPEC_LOOP, 32, 0),
                                   (f"spec_t{c.threshold}_static", sr.SPEC_LOOP, c.threshold,
                                    sr.F_STATIC)):
        w = sr.rsbench_workload(c.fma_count, prolog_fma=c.prolog_fma, unroll=c.merge_unroll,
                                flags=flags)
        t = graph_time(w, c.n_threads, c.iters, mode, thr, reps=5)
        res[name] = {"value": c.n_threads * c.iters / (t * 1e-3), "unit": "lookups/s", "ms": t}
    res["speedup_vs_pdom"] = res[f"spec_t{c.threshold}"]["value"] / res["pdom"]["value"]
    out["rsbench_fetch"] = res

    # configs[3]: path tracer, 1024^2 x 16 spp over the 1,044,494-triangle BVH scene
    c = I.C4
    tris, mat, mats, cam = I.cornell_scene(c)
    buf, used = sr.upload_scene(tris, mat, mats, cam, ctx.device)
    w_fixed = sr.pathtrace_workload(buf.data_ptr(), used, c.width, c.height, c.max_depth)
    # the warp's paths pooled (SR_F_POOL): per-path radiance kept for the ordered sums
    w_pool = sr.pathtrace_workload(buf.data_ptr(), used, c.width, c.height, c.max_depth,
                                   flags=sr.F_POOL, pool_spp=c.spp)
    ctx.ensure(sr.sr_workspace_bytes(w_pool, c.n_pixels))
    res = {"scene_triangles": int(len(tris)), "scene_bytes": int(used)}
    # split node-granularity Loop Merge, 8 node visits per release, soft barrier
    # T = inputs.C4.threshold (best of the threshold sweep, profiles/); each lane on
    # its own pixel, and with the warp's paths pooled
    sname = f"spec_t{c.threshold}"
    for name, mode, thr, w in (("pdom", sr.PDOM, 0, w_fixed),
                               (sname, sr.SPEC_LOOP, c.threshold, w_fixed),
                               (sname + "_pool", sr.SPEC_LOOP, c.threshold, w_pool)):
        ms = timer.time_steps(lambda: sr.sr_run(w, c.n_pixels, c.spp, I.PRIMARY_SEED, mode, thr),
                              max(3, min(args.steps, 5)), 1)
        t = statistics.median(ms)
        cnt = ctx.region(w, c.n_pixels, sr.T_COUNTERS, torch.int64).cpu().numpy()
        res[name] = {"value": c.n_pixels * c.spp / (t * 1e-3), "unit": "paths/s", "ms": t,
                     "rays": int(cnt[1]), "node_visits": int(cnt[2]), "tri_tests": int(cnt[3]),
                     "launch": sr.sr_last_launch()}
    # the merged kernel's best schedule (the pooled paths) and the fixed-pixel one
    res["speedup_vs_pdom"] = res[sname + "_pool"]["value"] / res["pdom"]["value"]
    res["speedup_fixed_pixel_vs_pdom"] = res[sname]["value"] / res["pdom"]["value"]
    # issue roofline (as MC): useful work = thread-instructions per path of a PDOM
    # kernel whose lanes each execute only their own path (profiles/work_per_unit.json,
    # pt_basis), peak = 592 SMSPs x 32 lanes x f
    per_path = (load_json(PROFILE_CONST) or {}).get("pt_thread_inst_per_path")
    if per_path:
        peak = 592 * 32 * f_mhz * 1e6
        res["issue_roofline"] = {
            "thread_inst_per_path": per_path,
            "frac": {k: per_path * res[k]["value"] / peak for k in ("pdom", sname, sname + "_pool")},
            "basis": "profiles/work_per_unit.json pt_thread_inst_per_path (ncu, as-compiled "
                     "PDOM) x paths/s / (592 x 32 x sm_max_mhz)"}
    out["pathtrace"] = res
    return out


if __name__ == "__main__":
    main()
