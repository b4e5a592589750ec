"""GPU parity: the CUDA path through the C ABI vs the CPU oracle (B200 only).

Bar (BASELINE.json north_star): per-thread FP outputs bit-exact (the library
is built with --fmad=false, explicit FMAs are IEEE on both sides), integer
tallies bit-exact, schedule counters equal to the warp simulator's.
"""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import sr

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

SEEDS = I.SEEDS


@pytest.fixture(scope="module")
def ctx():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    c = sr.Context.create(0, 1 << 26)
    yield c
    torch.cuda.synchronize()
    sr.sr_finalize()


def u64(t):
    return t.cpu().numpy().view(np.uint64)


def run_divloop(ctx, w, n, iters, seed, mode, T):
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, iters, seed, mode, T)
    out = ctx.region(w, n, sr.T_PERTHREAD, torch.int32).view(-1, 2).cpu().numpy()
    cnt = u64(ctx.region(w, n, sr.T_COUNTERS, torch.int64))
    return out[:, 0].view(np.float32).copy(), out[:, 1].view(np.uint32).copy(), cnt


# ------------------------------------------------------------------ building blocks
@pytest.mark.parametrize("fn", [sr.FN_LOGF, sr.FN_SIN2PI, sr.FN_COS2PI])
def test_device_math_bit_exact_all_rng_inputs(ctx, fn):
    """sr_logf / sr_sincos2pif on every one of the 2^24 inputs the RNG can give."""
    k = np.arange(1 if fn == sr.FN_LOGF else 0, (1 << 24) + (1 if fn == sr.FN_LOGF else 0),
                  dtype=np.float64)
    x = (k * 2.0**-24).astype(np.float32)
    xd = torch.from_numpy(x).cuda()
    od = torch.empty_like(xd)
    sr.sr_math_eval(fn, xd.data_ptr(), od.data_ptr(), x.size)
    ctx.stream.synchronize()
    got = od.cpu().numpy()
    ref = oracle.eval_batch(fn, x)
    bad = np.nonzero(got.view(np.uint32) != ref.view(np.uint32))[0]
    assert bad.size == 0, (bad[:5], x[bad[:5]], got[bad[:5]], ref[bad[:5]])


@pytest.mark.parametrize("fn", [sr.FN_EXPENSIVE_1000, sr.FN_EXPENSIVE_2000])
def test_device_expensive_bit_exact(ctx, fn):
    x = (np.arange(1 << 16, dtype=np.float64) * 2.0**-16).astype(np.float32)
    xd = torch.from_numpy(x).cuda()
    od = torch.empty_like(xd)
    sr.sr_math_eval(fn, xd.data_ptr(), od.data_ptr(), x.size)
    ctx.stream.synchronize()
    assert np.array_equal(od.cpu().numpy().view(np.uint32), oracle.eval_batch(fn, x).view(np.uint32))


# ---------------------------- the MC step's division / sqrt on their domains
def eval_p(ctx, fn, p, x):
    xd = torch.from_numpy(np.ascontiguousarray(x, np.float32)).cuda()
    od = torch.empty_like(xd)
    sr.sr_math_eval_p(fn, float(np.float32(p)), xd.data_ptr(), od.data_ptr(), x.size)
    ctx.stream.synchronize()
    return od.cpu().numpy()


def assert_bits(got, ref, x):
    bad = np.nonzero(got.view(np.uint32) != ref.view(np.uint32))[0]
    assert bad.size == 0, (bad.size, x[bad[:5]], got[bad[:5]], ref[bad[:5]])


F32 = np.float32
ALL_XI = (np.arange(1 << 24, dtype=np.float64) * 2.0**-24).astype(F32)   # every U01 value


@pytest.mark.parametrize("mut", [100.0, 200.0, 2.0**-20, 2.0**20, 7.31, 1000.0])
def test_div_dom_path_length_every_rng_input(ctx, mut):
    """s = -log(U01c)/mu_t: the kernel's div_dom(log, mu_t) negated == IEEE (-log)/mu_t on
    all 2^24 inputs (IEEE division is sign-symmetric, the numerator is never -0)."""
    x = ((np.arange(1 << 24, dtype=np.float64) + 1) * 2.0**-24).astype(F32)
    lg = oracle.eval_batch(sr.FN_LOGF, x)
    got = -eval_p(ctx, sr.FNP_DIV_XP, mut, lg)
    assert_bits(got, (-lg) / F32(mut), lg)


@pytest.mark.parametrize("n", [1.4, 1.33, 1.5, 1.0 + 2.0**-10, 2.0**10, 2.0**-10, 1.0 - 2.0**-10])
def test_fresnel_fast_path_every_cosine(ctx, n):
    """MCML's Fresnel sub-step on the FAST kernels' div_dom / sqrt_dom == the IEEE
    operations, reflectance and transmitted cosine, for EVERY binary32 cos(incidence)
    in [0, 1], both directions (into and out of the denser medium), at the indices
    of configs[2] (1.4 | 1) and at the edges of mc_fast_domain (ratio 1 + 2^-10,
    n = 2^10 and 2^-10)."""
    total = 0x3F800000 + 1                       # bit patterns of +0 .. 1.0
    chunk = 1 << 26
    for rev in (0, 4):
        for what in (0, 2):                      # reflectance, ca2
            for b in range(0, total, chunk):
                bits = torch.arange(b, min(b + chunk, total), dtype=torch.int64, device="cuda")
                x = bits.to(torch.int32).view(torch.float32)
                fast, ieee = torch.empty_like(x), torch.empty_like(x)
                p = float(np.float32(n))
                sr.sr_math_eval_p(sr.FNP_FRESNEL + 1 + what + rev, p, x.data_ptr(), fast.data_ptr(),
                                  x.numel())
                sr.sr_math_eval_p(sr.FNP_FRESNEL + what + rev, p, x.data_ptr(), ieee.data_ptr(),
                                  x.numel())
                ctx.stream.synchronize()
                bad = (fast.view(torch.int32) != ieee.view(torch.int32)).nonzero()
                assert bad.numel() == 0, (n, rev, what, int(bad.numel()),
                                          x[bad[:5, 0]].tolist(), fast[bad[:5, 0]].tolist(),
                                          ieee[bad[:5, 0]].tolist())


@pytest.mark.parametrize("p", [3.0, -0.37, 2.0**-40, 2.0**40, 1.0 + 2.0**-23])
def test_div_dom_log_uniform_operands(ctx, p):
    """x / p and p / x for 2^22 operands of both signs, log-uniform over [2^-60, 2^60]."""
    rng = np.random.default_rng(7)
    n = 1 << 22
    x = (np.exp2(rng.uniform(-60, 60, n)) * rng.choice([-1.0, 1.0], n)).astype(F32)
    x[:3] = [F32(1.0), F32(-1.0), F32(0.0)]   # +0 / p is in the domain for p > 0 only
    pf = F32(p)
    with np.errstate(divide="ignore"):
        got = eval_p(ctx, sr.FNP_DIV_XP, pf, x)
        ref = x / pf
        keep = (x != 0) | (pf > 0)
        assert_bits(got[keep], ref[keep], x[keep])
        got = eval_p(ctx, sr.FNP_DIV_PX, pf, x[3:])
        assert_bits(got, pf / x[3:], x[3:])


@pytest.mark.parametrize("p", [1.41e-3, 0.37, 1.0, 0.999999])
def test_div2_dom_rotation_quotients(ctx, p):
    """the rotation's paired quotients t / sqrt(1 - uz^2): |t| in [2^-100, 2], divisor in
    [1.41e-3, 1] -- 2^22 log-uniform numerators of both signs, lane by lane == IEEE"""
    rng = np.random.default_rng(11)
    n = 1 << 22
    x = (np.exp2(rng.uniform(-100, 1, n)) * rng.choice([-1.0, 1.0], n)).astype(F32)
    assert_bits(eval_p(ctx, sr.FNP_DIV2_XP, p, x), x / F32(p), x)


def test_sqrt_dom_matches_ieee(ctx):
    """every binary32 in [2^-25, 1) (the 1 - c^2 arguments), +0, and 2^22 log-uniform
    values over [2^-101, 2^127]"""
    rng = np.random.default_rng(3)
    dense = np.arange(np.float32(2.0**-25).view(np.uint32), np.float32(1.0).view(np.uint32),
                      dtype=np.uint32).view(F32)
    wide = np.exp2(rng.uniform(-101, 127, 1 << 22)).astype(F32)
    x = np.concatenate([dense, wide, np.array([0.0, 1.0, 2.0**-101], F32)])
    assert_bits(eval_p(ctx, sr.FNP_SQRT, 0.0, x), np.sqrt(x), x)


def hg_ieee(g, xi):
    """oracle/mcml.c's Henyey-Greenstein cos(theta) (reading R6), binary32 step by step"""
    g = F32(g)
    g2 = g * g
    one_m_g2, one_p_g2, one_m_g, two_g = F32(1) - g2, F32(1) + g2, F32(1) - g, F32(2) * g
    tmp = one_m_g2 / (one_m_g + two_g * xi)
    cost = (one_p_g2 - tmp * tmp) / two_g
    return np.clip(cost, F32(-1), F32(1)).astype(F32)


@pytest.mark.parametrize("g", [0.80, 0.90, 0.75, -0.8, 0.5, -0.3, 2.0**-18, -(2.0**-18),
                               0.99999994])
def test_hg_cost_and_sint_every_rng_input(ctx, g):
    """the MC step's HG cos(theta) and sin(theta) on all 2^24 xi == IEEE binary32"""
    cost = hg_ieee(g, ALL_XI)
    assert_bits(eval_p(ctx, sr.FNP_HG_COST, g, ALL_XI), cost, ALL_XI)
    assert_bits(eval_p(ctx, sr.FNP_HG_SINT, g, ALL_XI), np.sqrt(F32(1) - cost * cost), ALL_XI)


@pytest.mark.parametrize("layers,dr", [
    (((1.4, 4.0, 96.0, 1e-30, 0.01), (1.4, 1.0, 199.0, 0.9, 0.1)), 0.01),   # |g| < 2^-18
    (((1.3, 2e-7, 1e-7, 0.5, 0.05),), 0.01),                                 # mu_t < 2^-20
    (((1.3, 2e6, 1e6, 0.5, 0.05),), 0.01),                                   # mu_t > 2^20
    (I.THREE_LAYER, 1e-13),                                                  # dr < 2^-40
])
@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 32)])
def test_mcml_outside_fast_domain_bit_exact(ctx, layers, dr, mode, T):
    """layers outside the fast division domain run the guarded-IEEE kernels: still exact"""
    m = I.MCML(layers=layers, dr=dr)
    ref = mc_oracle(m, 0, 2048, 5)
    got = run_mc(ctx, mc_workload(m), 256, 8, 5, mode, T, m)
    assert_mc_equal(got, ref)


# ------------------------------------------------------------------ config 1
@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 1), (sr.SPEC_LOOP, 4),
                                    (sr.SPEC_LOOP, 16), (sr.SPEC_LOOP, 32)])
@pytest.mark.parametrize("block", [32, 64, 256])
def test_divloop_bit_exact_small(ctx, seed, mode, T, block):
    n, iters = 1000, 64   # 31.25 warps: several CTAs and a ragged tail
    acc_o, cnt_o = oracle.divloop(0, n, iters, seed)
    acc, cnt, tot = run_divloop(ctx, sr.divloop_workload(block=block), n, iters, seed, mode, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(cnt, cnt_o)
    assert tot[0] == cnt_o.sum()


@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 16)])
def test_divloop_bit_exact_full_config(ctx, mode, T):
    c = I.C1
    acc_o, cnt_o = oracle.divloop(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.p_u32, c.fma_count)
    acc, cnt, tot = run_divloop(ctx, sr.divloop_workload(c.p_u32, c.fma_count), c.n_threads,
                                c.iters, I.PRIMARY_SEED, mode, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(cnt, cnt_o)


@pytest.mark.parametrize("kw,n,iters,off", [
    (dict(fma_count=0), 100, 8, 0),                # no FMA: add tree only (runtime path)
    (dict(fma_count=8), 65, 8, 0),                 # one round, runtime loop
    (dict(fma_count=2000), 33, 16, 0),             # other compile-time instantiation
    (dict(p_u32=0), 64, 16, 0),                    # never wants
    (dict(p_u32=0xFFFFFFFF), 64, 16, 0),           # always wants
    (dict(), 1, 64, 0),                            # a single thread
    (dict(), 100, 0, 0),                           # zero iterations
    (dict(), 100, 16, (1 << 40) + 12345),          # 64-bit task ids
])
@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 16), (sr.SPEC_LOOP, 32)])
def test_divloop_edge_cases(ctx, kw, n, iters, off, mode, T):
    w = sr.divloop_workload(task_offset=off, **kw)
    p = dict(p_u32=1 << 29, fma_count=1000); p.update(kw)
    acc_o, cnt_o = oracle.divloop(off, n, iters, 7, p["p_u32"], p["fma_count"])
    acc, cnt, _ = run_divloop(ctx, w, n, iters, 7, mode, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(cnt, cnt_o)



@pytest.mark.parametrize("T,V", [(16, 2), (16, 8), (32, 4), (4, 64)])
def test_divloop_advance_unroll_bit_exact(ctx, T, V):
    """run-ahead lanes taking up to V iterations per advance round: same bits"""
    n, iters = 1000, 64
    acc_o, cnt_o = oracle.divloop(0, n, iters, 7)
    acc, cnt, _ = run_divloop(ctx, sr.divloop_workload(block=64, advance=V), n, iters, 7,
                              sr.SPEC_LOOP, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(cnt, cnt_o)


@pytest.mark.parametrize("T,V", [(16, 2), (16, 4), (32, 8)])
def test_divloop_advance_unroll_schedule_matches_simulator(ctx, T, V):
    n, iters = 2000, 64
    w = sr.divloop_workload(flags=sr.F_SCHED, block=64, advance=V)
    run_divloop(ctx, w, n, iters, I.PRIMARY_SEED, sr.SPEC_LOOP, T)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    want = oracle.divloop_wants(0, n, iters, I.PRIMARY_SEED)
    for wi in range((n + 31) // 32):
        s = oracle.ws_divloop(want[32 * wi:32 * wi + 32], oracle.SPEC_LOOP, T, V=V)
        g = sched[wi]
        assert (g[1], g[2]) == s["EXPENSIVE"], wi
        assert g[0] == s["rounds"] and (g[3], g[4]) == s["ADVANCE"], wi

@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 1), (sr.SPEC_LOOP, 16),
                                    (sr.SPEC_LOOP, 32)])
def test_divloop_schedule_matches_simulator(ctx, mode, T):
    """Per-warp rounds / releases / lane counts equal oracle part 2 exactly."""
    n, iters = 2000, 64
    w = sr.divloop_workload(flags=sr.F_SCHED, block=64)
    run_divloop(ctx, w, n, iters, I.PRIMARY_SEED, mode, T)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    want = oracle.divloop_wants(0, n, iters, I.PRIMARY_SEED)
    for wi in range((n + 31) // 32):
        ww = want[32 * wi:32 * wi + 32]
        s = oracle.ws_divloop(ww, oracle.PDOM if mode == sr.PDOM else oracle.SPEC_LOOP, T)
        g = sched[wi]
        assert (g[1], g[2]) == s["EXPENSIVE"], wi
        if mode == sr.SPEC_LOOP:
            assert g[0] == s["rounds"], wi
            assert (g[3], g[4]) == s["ADVANCE"] and s["PROLOG"] == s["ADVANCE"], wi


# batched prolog (prolog_batch = 64, reading Q5'): same bits, same schedule
@pytest.mark.parametrize("mode,T,V", [(sr.PDOM, 0, 1), (sr.SPEC_LOOP, 1, 1), (sr.SPEC_LOOP, 16, 1),
                                      (sr.SPEC_LOOP, 16, 8), (sr.SPEC_LOOP, 32, 8),
                                      (sr.SPEC_LOOP, 8, 100)])
@pytest.mark.parametrize("n,iters,off", [(1000, 64, 0), (333, 200, 0), (65, 63, 0),
                                         (100, 0, 0), (1, 129, 0), (97, 65, (1 << 40) + 7)])
def test_divloop_batch_bit_exact(ctx, mode, T, V, n, iters, off):
    """iters > 64 crosses mask windows (200 = 3 x 64 + 8; 129; 65), V = 100 spans them"""
    acc_o, cnt_o = oracle.divloop(off, n, iters, 7)
    w = sr.divloop_workload(task_offset=off, block=64, advance=V, batch=64)
    acc, cnt, tot = run_divloop(ctx, w, n, iters, 7, mode, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(cnt, cnt_o)
    assert tot[0] == cnt_o.sum()


@pytest.mark.parametrize("kw", [dict(p_u32=0), dict(p_u32=0xFFFFFFFF), dict(fma_count=8)])
@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 16)])
def test_divloop_batch_edge_cases(ctx, kw, mode, T):
    p = dict(p_u32=1 << 29, fma_count=1000); p.update(kw)
    acc_o, cnt_o = oracle.divloop(0, 100, 70, 7, p["p_u32"], p["fma_count"])
    acc, cnt, _ = run_divloop(ctx, sr.divloop_workload(batch=64, advance=8, **kw), 100, 70, 7,
                              mode, T)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(cnt, cnt_o)


def test_divloop_batch_full_config(ctx):
    c = I.C1
    acc_o, cnt_o = oracle.divloop(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.p_u32, c.fma_count)
    for mode, T in ((sr.PDOM, 0), (sr.SPEC_LOOP, 16), (sr.SPEC_LOOP, 1)):
        w = sr.divloop_workload(c.p_u32, c.fma_count, advance=c.advance_unroll, batch=64)
        acc, cnt, _ = run_divloop(ctx, w, c.n_threads, c.iters, I.PRIMARY_SEED, mode, T)
        assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32)), (mode, T)
        assert np.array_equal(cnt, cnt_o), (mode, T)


@pytest.mark.parametrize("mode,T,V", [(sr.PDOM, 0, 1), (sr.SPEC_LOOP, 16, 1), (sr.SPEC_LOOP, 16, 8),
                                      (sr.SPEC_LOOP, 4, 3)])
def test_divloop_batch_schedule_matches_simulator(ctx, mode, T, V):
    n, iters = 2000, 64
    w = sr.divloop_workload(flags=sr.F_SCHED, block=64, advance=V, batch=64)
    run_divloop(ctx, w, n, iters, I.PRIMARY_SEED, mode, T)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    want = oracle.divloop_wants(0, n, iters, I.PRIMARY_SEED)
    for wi in range((n + 31) // 32):
        s = oracle.ws_divloop(want[32 * wi:32 * wi + 32],
                              oracle.PDOM if mode == sr.PDOM else oracle.SPEC_LOOP, T,
                              V=V if mode == sr.SPEC_LOOP else 1)
        g = sched[wi]
        assert (g[1], g[2]) == s["EXPENSIVE"], wi
        if mode == sr.SPEC_LOOP:
            assert g[0] == s["rounds"] and (g[3], g[4]) == s["ADVANCE"], wi


# warp task pool of the Expensive() calls (SR_F_POOL, prolog_batch = 64)
@pytest.mark.parametrize("n,iters,off,block", [(1000, 64, 0, 64), (333, 200, 0, 96), (65, 63, 0, 32),
                                               (100, 0, 0, 64), (1, 129, 0, 64),
                                               (97, 65, (1 << 40) + 7, 512), (32768, 64, 0, 64)])
@pytest.mark.parametrize("split", [1, 2, 4])
def test_divloop_pool_bit_exact(ctx, n, iters, off, block, split):
    acc_o, cnt_o = oracle.divloop(off, n, iters, 7)
    w = sr.divloop_workload(task_offset=off, block=block, batch=64, flags=sr.F_POOL, split=split)
    acc, cnt, tot = run_divloop(ctx, w, n, iters, 7, sr.SPEC_LOOP, 16)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(cnt, cnt_o)
    assert tot[0] == cnt_o.sum()


@pytest.mark.parametrize("kw", [dict(p_u32=0), dict(p_u32=0xFFFFFFFF), dict(fma_count=8),
                                dict(fma_count=2000)])
@pytest.mark.parametrize("split", [1, 4])
def test_divloop_pool_edge_cases(ctx, kw, split):
    p = dict(p_u32=1 << 29, fma_count=1000); p.update(kw)
    acc_o, cnt_o = oracle.divloop(0, 100, 70, 7, p["p_u32"], p["fma_count"])
    w = sr.divloop_workload(batch=64, flags=sr.F_POOL, split=split, **kw)
    acc, cnt, _ = run_divloop(ctx, w, 100, 70, 7, sr.SPEC_LOOP, 32)
    assert np.array_equal(acc.view(np.uint32), acc_o.view(np.uint32))
    assert np.array_equal(cnt, cnt_o)


@pytest.mark.parametrize("n,iters", [(2000, 64), (77, 130)])
@pytest.mark.parametrize("split", [1, 2, 4])
def test_divloop_pool_schedule_closed_form(ctx, n, iters, split):
    """per window: one batched advance per slice (64 / split iterations) of every
    valid lane, then ceil(N/32) releases running the window's N wanted calls
    (split = 1: the warp's queue; split > 1: the CTA's, dealt to its warps)"""
    w = sr.divloop_workload(flags=sr.F_SCHED | sr.F_POOL, block=64, batch=64, split=split)
    run_divloop(ctx, w, n, iters, I.PRIMARY_SEED, sr.SPEC_LOOP, 16)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    want = oracle.divloop_wants(0, n, iters, I.PRIMARY_SEED)
    for wi in range((n + 31) // 32):
        ww = want[32 * wi:32 * wi + 32]
        nv = len(ww)
        Ns = [int(ww[:, b:min(b + 64, iters)].sum()) for b in range(0, iters, 64)]
        rel = sum((N + 31) // 32 for N in Ns)
        g = sched[wi]
        assert g[1] == rel and g[2] == sum(Ns), wi
        assert g[3] == len(Ns) * split and g[4] == len(Ns) * split * nv, wi
        assert g[0] == rel + len(Ns) * split, wi


# ------------------------------------------------------------------ config 2
def run_cc(ctx, w, n, iters, seed, mode):
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, iters, seed, mode, 0)
    y = ctx.region(w, n, sr.T_PERTHREAD, torch.float32).cpu().numpy().copy()
    return y, u64(ctx.region(w, n, sr.T_COUNTERS, torch.int64))


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("mode", [sr.PDOM, sr.SPEC_CALL])
@pytest.mark.parametrize("n,iters,block", [(1000, 1, 256), (77, 3, 32), (4096, 1, 1024)])
def test_commoncall_bit_exact(ctx, seed, mode, n, iters, block):
    y_o, arm = oracle.commoncall(0, n, iters, seed)
    y, cnt = run_cc(ctx, sr.commoncall_workload(block=block), n, iters, seed, mode)
    assert np.array_equal(y.view(np.uint32), y_o.view(np.uint32))
    if iters == 1:
        assert cnt[0] == arm.sum()


@pytest.mark.parametrize("mode", [sr.PDOM, sr.SPEC_CALL])
def test_commoncall_bit_exact_full_config(ctx, mode):
    c = I.C2
    y_o, _ = oracle.commoncall(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.split_u32, c.fma_count)
    y, _ = run_cc(ctx, sr.commoncall_workload(c.fma_count, c.split_u32), c.n_threads, c.iters,
                  I.PRIMARY_SEED, mode)
    assert np.array_equal(y.view(np.uint32), y_o.view(np.uint32))


@pytest.mark.parametrize("mode", [sr.PDOM, sr.SPEC_CALL])
def test_commoncall_schedule_matches_simulator(ctx, mode):
    n = 1000
    w = sr.commoncall_workload(flags=sr.F_SCHED)
    run_cc(ctx, w, n, 1, I.PRIMARY_SEED, mode)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    _, arm = oracle.commoncall(0, n, 1, I.PRIMARY_SEED)
    for wi in range((n + 31) // 32):
        s = oracle.ws_commoncall(arm[32 * wi:32 * wi + 32],
                                 oracle.PDOM if mode == sr.PDOM else oracle.SPEC_CALL)
        assert (sched[wi][1], sched[wi][2]) == s["CALL"], wi


# ------------------------------------------------------------------ configs 3/5
def mc_oracle(m, id0, count, seed):
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    return oracle.mcml(p, id0, count, seed, steps=True)


def mc_workload(m, **kw):
    return sr.mcml_workload(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap, **kw)


def run_mc(ctx, w, n, iters, seed, mode, T, m):
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, iters, seed, mode, T)
    g = u64(ctx.region(w, n, sr.T_GRID, torch.int64))
    nA = m.nz * m.nr
    cnt = u64(ctx.region(w, n, sr.T_COUNTERS, torch.int64))
    return dict(A=g[:nA], Rd=g[nA:nA + m.nr], Tt=g[nA + m.nr:], counters=cnt[:8])


def assert_mc_equal(got, ref):
    assert np.array_equal(got["A"], ref["A"].ravel())
    assert np.array_equal(got["Rd"], ref["Rd"])
    assert np.array_equal(got["Tt"], ref["Tt"])
    assert np.array_equal(got["counters"], ref["counters_raw"])


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("flags", [0, sr.F_STATIC])
@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 1), (sr.SPEC_LOOP, 8),
                                    (sr.SPEC_LOOP, 32)])
def test_mcml_bit_exact_small(ctx, seed, flags, mode, T):
    m = I.C3
    nt, it = 300, 5   # ragged: 9.4 warps, 1500 photons
    ref = mc_oracle(m, 0, nt * it, seed)
    got = run_mc(ctx, mc_workload(m, flags=flags, block=128), nt, it, seed, mode, T, m)
    assert_mc_equal(got, ref)


@pytest.mark.parametrize("name", ["BEER_LAMBERT", "NO_ABSORPTION", "VAN_DE_HULST",
                                  "MISMATCHED_ABSORBER"])
@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 32)])
def test_mcml_bit_exact_pin_workloads(ctx, name, mode, T):
    m = getattr(I, name)
    ref = mc_oracle(m, 5000, 4096, 11)
    got = run_mc(ctx, mc_workload(m, task_offset=5000), 512, 8, 11, mode, T, m)
    assert_mc_equal(got, ref)


@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 4), (sr.SPEC_LOOP, 32)])
def test_mcml_schedule_matches_simulator(ctx, mode, T):
    m = I.C3
    nt, it = 96, 6
    w = mc_workload(m, flags=sr.F_STATIC | sr.F_SCHED, block=32)
    run_mc(ctx, w, nt, it, 3, mode, T, m)
    sched = ctx.region(w, nt, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    ref = mc_oracle(m, 0, nt * it, 3)
    steps = ref["steps"].reshape(it, nt).T     # photon l + k*nt -> [lane, k]
    for wi in range(nt // 32):
        ns = steps[32 * wi:32 * wi + 32]
        s = oracle.ws_loopmerge(ns, oracle.PDOM if mode == sr.PDOM else oracle.SPEC_LOOP, T)
        g = sched[wi]
        assert (g[1], g[2]) == s["STEP"], wi
        if mode == sr.SPEC_LOOP:
            assert g[0] == s["rounds"] and (g[3], g[4]) == s["LAUNCH"], wi


@pytest.mark.parametrize("flags", [0, sr.F_STATIC])
@pytest.mark.parametrize("T,U", [(32, 2), (32, 4), (16, 3)])
def test_mcml_unrolled_merge_bit_exact(ctx, flags, T, U):
    m = I.C3
    nt, it = 300, 5
    ref = mc_oracle(m, 0, nt * it, 19)
    got = run_mc(ctx, mc_workload(m, flags=flags, block=128, unroll=U), nt, it, 19,
                 sr.SPEC_LOOP, T, m)
    assert_mc_equal(got, ref)


@pytest.mark.parametrize("T,U", [(32, 2), (8, 4)])
def test_mcml_unrolled_schedule_matches_simulator(ctx, T, U):
    m = I.C3
    nt, it = 96, 6
    w = mc_workload(m, flags=sr.F_STATIC | sr.F_SCHED, block=32, unroll=U)
    run_mc(ctx, w, nt, it, 3, sr.SPEC_LOOP, T, m)
    sched = ctx.region(w, nt, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    ev, off, ns = oracle.mcml_events_batch(p, 0, nt * it, 3)
    for wi in range(nt // 32):
        lanes = np.arange(32 * wi, 32 * wi + 32)
        ids = lanes[:, None] + np.arange(it)[None, :] * nt
        s = oracle.ws_loopmerge_raw(ns[ids], ev, off[ids].ravel(), oracle.SPEC_LOOP, T, U=U)
        g = sched[wi]
        assert g[0] == s["rounds"] and (g[1], g[2]) == s["RELEASE"], wi
        assert (g[3], g[4]) == s["LAUNCH"], wi


@pytest.mark.parametrize("flags", [0, sr.F_STATIC])
@pytest.mark.parametrize("T,Tb", [(32, 1), (32, 8), (16, 4), (32, 32)])
def test_mcml_deferred_boundary_bit_exact(ctx, flags, T, Tb):
    m = I.C3
    nt, it = 300, 5
    ref = mc_oracle(m, 0, nt * it, 17)
    got = run_mc(ctx, mc_workload(m, flags=flags, block=128, defer=Tb), nt, it, 17,
                 sr.SPEC_LOOP, T, m)
    assert_mc_equal(got, ref)


@pytest.mark.parametrize("T,Tb", [(32, 8), (16, 4), (32, 32)])
def test_mcml_deferred_schedule_matches_simulator(ctx, T, Tb):
    m = I.C3
    nt, it = 96, 6
    w = mc_workload(m, flags=sr.F_STATIC | sr.F_SCHED, block=32, defer=Tb)
    run_mc(ctx, w, nt, it, 3, sr.SPEC_LOOP, T, m)
    sched = ctx.region(w, nt, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    ev, off, ns = oracle.mcml_events_batch(p, 0, nt * it, 3)
    for wi in range(nt // 32):
        lanes = np.arange(32 * wi, 32 * wi + 32)
        ids = lanes[:, None] + np.arange(it)[None, :] * nt
        s = oracle.ws_loopmerge_defer_raw(ns[ids], ev, off[ids].ravel(), T, Tb)
        g = sched[wi]
        assert g[0] == s["rounds"], wi
        assert (g[1], g[2]) == s["STEP"], wi
        assert (g[3], g[4]) == s["LAUNCH"], wi
        assert (g[5], g[6]) == s["B_REL"], wi


def test_mcml_full_size_invariants(ctx):
    """Config 3 at full size in the bench launch configuration: PDOM == SPEC
    (T=32, 16) bit for bit, == the sum of two shards, and a slice far into the
    id range equals the oracle."""
    m = I.C3
    nt, it = m.n_threads, m.iters
    w = mc_workload(m, unroll=m.merge_unroll)      # the bench's launch configuration
    full = run_mc(ctx, w, nt, it, I.PRIMARY_SEED, sr.SPEC_LOOP, m.threshold, m)
    assert full["counters"][0] == nt * it
    for mode, T in ((sr.PDOM, 0), (sr.SPEC_LOOP, 16)):
        o = run_mc(ctx, w, nt, it, I.PRIMARY_SEED, mode, T, m)
        for k in full:
            assert np.array_equal(o[k], full[k]), (mode, T, k)
    half = nt // 2
    a = run_mc(ctx, mc_workload(m), half, it, I.PRIMARY_SEED, sr.SPEC_LOOP, 32, m)
    b = run_mc(ctx, mc_workload(m, task_offset=half * it), nt - half, it, I.PRIMARY_SEED,
               sr.SPEC_LOOP, 32, m)
    for k in full:
        assert np.array_equal(a[k] + b[k], full[k]), k
    c = full["counters"]
    assert c[2] + c[3] + c[4] + c[6] + c[7] == nt * it   # every photon ends exactly once
    off = 9_000_000
    ref = mc_oracle(m, off, 20000, I.PRIMARY_SEED)
    got = run_mc(ctx, mc_workload(m, task_offset=off), 20000, 1, I.PRIMARY_SEED, sr.SPEC_LOOP,
                 32, m)
    assert_mc_equal(got, ref)


@pytest.mark.parametrize("n,iters,off,cap", [
    (1, 1, 0, 100000),                  # one lane, one photon
    (33, 2, 0, 100000),                 # one full warp + a 1-lane warp
    (64, 3, 0, 3),                      # step cap hit by nearly every photon
    (100, 2, (1 << 40) + 12345, 100000),  # ids above 2^32: the counter's task_hi word
    (96, 1, 2**64 - 97, 100000),        # top of the 64-bit id space (end = 2^64 - 1)
])
@pytest.mark.parametrize("mode,T,U", [(sr.PDOM, 0, 1), (sr.SPEC_LOOP, 32, 4), (sr.SPEC_LOOP, 8, 1)])
@pytest.mark.parametrize("flags", [0, sr.F_STATIC])
def test_mcml_edge_cases(ctx, n, iters, off, cap, mode, T, U, flags):
    import dataclasses
    m = dataclasses.replace(I.C3, step_cap=cap)
    ref = mc_oracle(m, off, n * iters, I.PRIMARY_SEED)
    got = run_mc(ctx, mc_workload(m, task_offset=off, flags=flags, unroll=U), n, iters,
                 I.PRIMARY_SEED, mode, T, m)
    assert_mc_equal(got, ref)
