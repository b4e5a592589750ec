"""GPU parity of NEXT-1 (RSBench-shaped nested trip-count loop) vs the oracle:
per-thread sums bit-exact in every mode and threshold, schedule counters equal
to the loop-merge warp simulator, and sampled threads at the full config."""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import sr

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    c = sr.Context.create(0, 1 << 24)
    yield c
    torch.cuda.synchronize()
    sr.sr_finalize()


def run(ctx, w, n, iters, seed, mode, T):
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, iters, seed, mode, T)
    out = ctx.region(w, n, sr.T_PERTHREAD, torch.int32).view(-1, 2).cpu().numpy()
    cnt = ctx.region(w, n, sr.T_COUNTERS, torch.int64).cpu().numpy()
    return out[:, 0].view(np.float32).copy(), out[:, 1].view(np.uint32).copy(), cnt


@pytest.mark.parametrize("seed", I.SEEDS)
@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 1), (sr.SPEC_LOOP, 4),
                                    (sr.SPEC_LOOP, 16), (sr.SPEC_LOOP, 32)])
@pytest.mark.parametrize("flags", [0, sr.F_STATIC])   # warp task pool (default) / static
def test_rsbench_bit_exact_small(ctx, seed, mode, T, flags):
    n, iters = 700, 6
    acc_o, nuc_o = oracle.rsbench(0, n, iters, seed)
    acc, nuc, cnt = run(ctx, sr.rsbench_workload(block=64, flags=flags), n, iters, seed, mode, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(nuc, nuc_o)
    assert cnt[0] == nuc_o.sum()


@pytest.mark.parametrize("T,U", [(24, 2), (32, 3), (4, 4)])
def test_rsbench_unrolled_merge_bit_exact(ctx, T, U):
    """up to U inner iterations per release: same bits"""
    n, iters = 700, 6
    acc_o, nuc_o = oracle.rsbench(3, n, iters, 9)
    acc, nuc, cnt = run(ctx, sr.rsbench_workload(block=64, task_offset=3, unroll=U), n, iters,
                        9, sr.SPEC_LOOP, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(nuc, nuc_o)


@pytest.mark.parametrize("T,U", [(24, 2), (32, 4)])
def test_rsbench_unrolled_schedule_matches_simulator(ctx, T, U):
    n, iters = 256, 8
    w = sr.rsbench_workload(flags=sr.F_SCHED | sr.F_STATIC, block=64, unroll=U)
    run(ctx, w, n, iters, 5, sr.SPEC_LOOP, T)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    _, _, trips = oracle.rsbench(0, n, iters, 5, fma_count=0, trips=True)
    for wi in range(n // 32):
        s = oracle.ws_loopmerge(trips[32 * wi:32 * wi + 32], oracle.SPEC_LOOP, T, U=U)
        g = sched[wi]
        assert g[0] == s["rounds"] and (g[1], g[2]) == s["RELEASE"], wi
        assert (g[3], g[4]) == s["LAUNCH"], wi


@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 4), (sr.SPEC_LOOP, 32)])
def test_rsbench_schedule_matches_simulator(ctx, mode, T):
    n, iters = 256, 8
    w = sr.rsbench_workload(flags=sr.F_SCHED | sr.F_STATIC, block=64)
    run(ctx, w, n, iters, 5, mode, T)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    _, _, trips = oracle.rsbench(0, n, iters, 5, fma_count=0, trips=True)
    for wi in range(n // 32):
        s = oracle.ws_loopmerge(trips[32 * wi:32 * wi + 32],
                                oracle.PDOM if mode == sr.PDOM else oracle.SPEC_LOOP, T)
        g = sched[wi]
        assert (g[1], g[2]) == s["STEP"], wi
        if mode == sr.SPEC_LOOP:
            assert g[0] == s["rounds"] and (g[3], g[4]) == s["LAUNCH"], wi


@pytest.mark.parametrize("n,iters,T,U,block", [(700, 6, 24, 12, 64), (333, 5, 4, 1, 96),
                                               (31, 40, 32, 3, 256), (1, 7, 16, 2, 32),
                                               (100, 0, 24, 12, 64), (65, 129, 24, 12, 128)])
def test_rsbench_pool_bit_exact(ctx, n, iters, T, U, block):
    """the warp task pool: ragged warps (a partial warp's idle lanes work on its
    threads' lookups), one thread, zero lookups, many lookups per thread"""
    acc_o, nuc_o = oracle.rsbench(11, n, iters, 3)
    w = sr.rsbench_workload(block=block, task_offset=11, unroll=U)
    acc, nuc, cnt = run(ctx, w, n, iters, 3, sr.SPEC_LOOP, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(nuc, nuc_o)
    assert cnt[0] == nuc_o.sum()


@pytest.mark.parametrize("T,U,n", [(24, 1, 256), (24, 12, 256), (4, 3, 200), (32, 2, 77)])
def test_rsbench_pool_schedule_matches_simulator(ctx, T, U, n):
    iters = 8
    w = sr.rsbench_workload(flags=sr.F_SCHED, block=64, unroll=U)
    run(ctx, w, n, iters, 5, sr.SPEC_LOOP, T)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    _, _, trips = oracle.rsbench(0, n, iters, 5, fma_count=0, trips=True)
    for wi in range((n + 31) // 32):
        s = oracle.ws_loopmerge_pool(trips[32 * wi:32 * wi + 32], T, U=U)
        g = sched[wi]
        assert g[0] == s["rounds"] and (g[1], g[2]) == s["RELEASE"], wi
        assert (g[3], g[4]) == s["ADVANCE"], wi


def test_rsbench_full_config_sampled(ctx):
    c = I.NEXT1
    w = sr.rsbench_workload(c.fma_count)
    a_spec, n_spec, _ = run(ctx, w, c.n_threads, c.iters, I.PRIMARY_SEED, sr.SPEC_LOOP,
                            c.threshold)
    a_pdom, n_pdom, _ = run(ctx, w, c.n_threads, c.iters, I.PRIMARY_SEED, sr.PDOM, 0)
    assert np.array_equal(a_spec.view(np.uint32), a_pdom.view(np.uint32))
    assert np.array_equal(n_spec, n_pdom)
    rng = np.random.default_rng(1)
    for t in rng.choice(c.n_threads, 64, replace=False):
        acc_o, nuc_o = oracle.rsbench(int(t), 1, c.iters, I.PRIMARY_SEED, c.fma_count)
        assert a_spec[t].view(np.uint32) == acc_o[0].view(np.uint32) and n_spec[t] == nuc_o[0]


@pytest.mark.parametrize("prolog", [256, 2048, 8])   # generic, compile-time, smallest
@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 4), (sr.SPEC_LOOP, 16),
                                    (sr.SPEC_LOOP, 32)])
def test_rsbench_expensive_prolog_bit_exact(ctx, prolog, mode, T):
    """The expensive-task-fetch variant (Fig. 9's XSBench case): every mode and
    threshold equals the oracle bit for bit, also in the schedule counters'
    kernels (the prolog does not change the trip counts)."""
    n, iters = 333, 5
    acc_o, nuc_o = oracle.rsbench(7, n, iters, I.PRIMARY_SEED, prolog_fma=prolog)
    w = sr.rsbench_workload(block=96, task_offset=7, prolog_fma=prolog)
    acc, nuc, cnt = run(ctx, w, n, iters, I.PRIMARY_SEED, mode, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(nuc, nuc_o)


def test_rsbench_expensive_prolog_full_config_sampled(ctx):
    c = I.NEXT1_FETCH
    w = sr.rsbench_workload(c.fma_count, prolog_fma=c.prolog_fma)
    a, nn, _ = run(ctx, w, c.n_threads, c.iters, I.PRIMARY_SEED, sr.SPEC_LOOP, c.threshold)
    rng = np.random.default_rng(2)
    for t in rng.choice(c.n_threads, 16, replace=False):
        acc_o, nuc_o = oracle.rsbench(int(t), 1, c.iters, I.PRIMARY_SEED, c.fma_count,
                                      prolog_fma=c.prolog_fma)
        assert a[t].view(np.uint32) == acc_o[0].view(np.uint32) and nn[t] == nuc_o[0]
