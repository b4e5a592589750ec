"""Pins of the oracle's config-1 (divloop) and config-2 (commoncall) programs.

Closed forms (a linear recurrence solved exactly), distributional identities
(E[cnt] = iters*p from BASELINE.json north_star) and range invariants.
"""
import math

import numpy as np
import pytest

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I

M = 1.0 - 2.0**-10
CK = [(k + 1) / 16.0 for k in range(8)]


def expensive_closed_form(u, fma_count):
    """a_k(n) = M^n (a_k(0) - C_k/(1-M)) + C_k/(1-M): exact solution of
    a <- a*M + C_k, n = fma_count/8 times; r = sum_k a_k(n)."""
    n = fma_count // 8
    fix = [c / (1.0 - M) for c in CK]
    return sum(M**n * (u + k - fix[k]) + fix[k] for k in range(8))


def expensive_tol(fma_count):
    # each fmaf rounds once (<= 1/2 ulp of |a| <= 512 -> 2^-15); errors are
    # damped by M < 1 but bound them by n * 1/2ulp per chain, 8 chains, +tree
    n = fma_count // 8
    return 8 * n * 2.0**-15 + 8 * 2.0**-12


@pytest.mark.parametrize("fma_count", [8, 1000, 2000, 16000])
@pytest.mark.parametrize("u", [0.0, 0.25, 0.5, 0.999])
def test_expensive_matches_closed_form(u, fma_count):
    got = oracle.lib().or_expensive(u, fma_count)
    assert abs(got - expensive_closed_form(u, fma_count)) <= expensive_tol(fma_count)


def test_expensive_zero_fmas_is_add_tree():
    # no FMA: r = sum_k (u + k) = 8u + 28, exact for these u
    for u in (0.0, 0.5, 0.75):
        assert oracle.lib().or_expensive(u, 0) == 8 * u + 28


def test_divloop_expected_calls_closed_form():
    c = I.C1
    acc, cnt = oracle.divloop(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.p_u32, c.fma_count)
    p = c.p_u32 / 2**32
    # E[cnt] = iters * p (north_star), cnt ~ Binomial(iters, p) per thread
    sigma = math.sqrt(c.iters * p * (1 - p) / c.n_threads)
    assert abs(cnt.mean() - c.iters * p) < 5 * sigma
    assert abs(cnt.var() - c.iters * p * (1 - p)) < 0.3
    # acc / cnt lies in [r(0), r(1)] (r is increasing in u) ...
    lo = expensive_closed_form(0.0, c.fma_count) - expensive_tol(c.fma_count)
    hi = expensive_closed_form(1.0, c.fma_count) + expensive_tol(c.fma_count)
    nz = cnt > 0
    per = acc[nz] / cnt[nz]
    assert per.min() >= lo - 1e-3 and per.max() <= hi + 1e-3
    assert np.all(acc[~nz] == 0.0)
    # ... and its mean is r(E[u]) (r is affine in u)
    mean_r = acc.sum(dtype=np.float64) / cnt.sum()
    assert abs(mean_r - expensive_closed_form(0.5, c.fma_count)) < 0.05


def test_divloop_degenerate_cases():
    acc, cnt = oracle.divloop(0, 64, 0, 7)
    assert np.all(cnt == 0) and np.all(acc == 0)
    acc, cnt = oracle.divloop(0, 64, 16, 7, p_u32=0)
    assert np.all(cnt == 0)
    acc, cnt = oracle.divloop(0, 64, 16, 7, p_u32=0xFFFFFFFF)
    assert cnt.min() >= 15  # P(u0 == 2^32-1) is 2^-32


def test_divloop_thread_offset_is_a_shift():
    a1, c1 = oracle.divloop(0, 100, 8, 3)
    a2, c2 = oracle.divloop(40, 60, 8, 3)
    assert np.array_equal(a1[40:], a2) and np.array_equal(c1[40:], c2)


def test_divloop_wants_match_counts():
    w = oracle.divloop_wants(5, 300, 64, 11)
    _, cnt = oracle.divloop(5, 300, 64, 11)
    assert np.array_equal(w.sum(1), cnt)


def test_commoncall_arms_and_ranges():
    c = I.C2
    n = 1 << 16
    y, arm = oracle.commoncall(0, n, 1, I.PRIMARY_SEED, c.split_u32, c.fma_count)
    assert abs(arm.mean() - 0.5) < 5 * math.sqrt(0.25 / n)
    tol = expensive_tol(c.fma_count)
    f = lambda u: expensive_closed_form(u, c.fma_count)
    t = y[arm == 1]
    assert t.min() >= f(0.0) - tol and t.max() <= f(1.0) + tol
    e = y[arm == 0]  # else arm: foo(x*0.5+0.25)^2, x1 in [0.25, 0.75)
    assert e.min() >= (f(0.25) - tol) ** 2 * (1 - 1e-6)
    assert e.max() <= (f(0.75) + tol) ** 2 * (1 + 1e-6)
    assert abs(t.mean() - f(0.5)) < 0.05


def test_commoncall_iters_accumulate():
    y1, _ = oracle.commoncall(0, 50, 1, 9)
    y2, _ = oracle.commoncall(0, 50, 2, 9)
    assert np.all(y2 > y1)


def test_divloop_per_thread_sums_match_float64_closed_form():
    """Every thread's (acc, cnt) re-derived in float64 from the definition
    (reading R3: condition u0 < p_u32 of the thread's Philox draw at event i,
    Expensive() of U01(u1) by the recurrence's closed form, acc the in-order sum):
    cnt exactly, acc within the accumulated binary32 rounding bound."""
    c = I.C1
    t0, n, seed = 12345, 256, I.PRIMARY_SEED
    acc, cnt = oracle.divloop(t0, n, c.iters, seed, c.p_u32, c.fma_count)
    key = [seed & 0xFFFFFFFF, seed >> 32]
    for j in range(n):
        t = t0 + j
        a64, k, mag = 0.0, 0, 0.0
        for i in range(c.iters):
            u = oracle.philox([i, 1 << 16, t & 0xFFFFFFFF, t >> 32], key)
            if int(u[0]) < c.p_u32:
                r = expensive_closed_form((int(u[1]) >> 8) * 2.0**-24, c.fma_count)
                a64 += r
                mag += abs(a64)
                k += 1
        assert cnt[j] == k, j
        # each call within expensive_tol, each of the k additions within 2^-24 |acc|
        bound = k * expensive_tol(c.fma_count) + mag * 2.0**-24
        assert abs(float(acc[j]) - a64) <= bound, (j, float(acc[j]), a64, bound)


def test_commoncall_per_thread_matches_float64_definition():
    """Every thread's y re-derived in float64 from reading R4: then-arm iff
    u0 < split_u32, y = foo(x) with x = U01(u1); else y = foo(fl(fl(x/2) + 1/4))^2
    (the argument's two binary32 roundings are exact here), foo by the closed form."""
    c = I.C2
    t0, n, seed = 99, 300, I.PRIMARY_SEED
    y, arm = oracle.commoncall(t0, n, 1, seed, c.split_u32, c.fma_count)
    key = [seed & 0xFFFFFFFF, seed >> 32]
    tol = expensive_tol(c.fma_count)
    for j in range(n):
        t = t0 + j
        u = oracle.philox([0, 2 << 16, t & 0xFFFFFFFF, t >> 32], key)
        x = (int(u[1]) >> 8) * 2.0**-24
        then = int(u[0]) < c.split_u32
        assert bool(arm[j]) == then, j
        if then:
            want, bound = expensive_closed_form(x, c.fma_count), tol
        else:
            r = expensive_closed_form(x * 0.5 + 0.25, c.fma_count)
            want, bound = r * r, 2 * abs(r) * tol + r * r * 2.0**-23
        assert abs(float(y[j]) - want) <= bound, (j, float(y[j]), want, bound)
