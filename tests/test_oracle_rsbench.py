"""Pins of the oracle's RSBench-shaped workload (NEXT-1, Fig. 3):
material selection frequencies, trip-count statistics, the body's closed
form, and per-thread sums within the closed-form range."""
import math

import numpy as np

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from tests.test_oracle_microbench import expensive_closed_form, expensive_tol

PROB = [0.140, 0.052, 0.275, 0.134, 0.154, 0.064, 0.066, 0.055, 0.008, 0.015, 0.025, 0.013]
NUCS = [321, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9]


def test_material_table_and_pick_boundaries():
    nucs, thr, pick = oracle.rs_table()
    assert nucs == NUCS and min(nucs) == 4 and max(nucs) == 321   # "4 to 321"
    assert all(a < b for a, b in zip(thr, thr[1:])) and thr[-1] == 2**32 - 1
    assert abs(thr[0] - 0.140 * 2**32) <= 1
    for m in range(11):
        assert pick(thr[m] - 1) == m and pick(thr[m]) == m + 1
    assert pick(0) == 0 and pick(2**32 - 1) == 11


def test_trip_count_distribution():
    c = I.NEXT1
    n, iters = 20000, 8
    _, nuc, trips = oracle.rsbench(0, n, iters, I.PRIMARY_SEED, fma_count=0, trips=True)
    assert np.array_equal(trips.sum(1), nuc)
    vals, counts = np.unique(trips, return_counts=True)
    assert set(vals) <= set(NUCS)
    # chi^2 of the material frequencies (materials with equal trip counts merged)
    exp = {}
    for p, k in zip(PROB, NUCS):
        exp[k] = exp.get(k, 0.0) + p
    N = trips.size
    chi2 = sum((counts[list(vals).index(k)] - N * p) ** 2 / (N * p) for k, p in exp.items())
    assert chi2 < len(exp) + 5 * math.sqrt(2 * len(exp))
    mean = sum(p * k for p, k in zip(PROB, NUCS))
    assert abs(trips.mean() - mean) < 5 * trips.std() / math.sqrt(N)


def test_body_closed_form():
    L = oracle.lib()
    import ctypes as C
    L.or_rs_body.argtypes = [C.c_float, C.c_uint32, C.c_uint32]
    L.or_rs_body.restype = C.c_float
    for E in (0.0, 0.3, 0.9):
        for nuc in (0, 17, 354):
            start = np.float32(np.float32(E) + np.float32(nuc * 2.0**-9))
            got = L.or_rs_body(E, nuc, 64)
            assert abs(got - expensive_closed_form(float(start), 64)) <= expensive_tol(64)


def test_thread_sums_within_closed_form_range():
    acc, nuc = oracle.rsbench(0, 500, 4, 3, fma_count=64)
    lo = expensive_closed_form(0.0, 64) - expensive_tol(64)
    hi = expensive_closed_form(1.0 + 354 * 2.0**-9, 64) + expensive_tol(64)
    per = acc / nuc
    assert per.min() >= lo * (1 - 1e-5) and per.max() <= hi * (1 + 1e-5)


def test_expensive_prolog_changes_energies_not_trips():
    """prolog_fma (reading R8'): the lookup prolog computes E = Expensive(U01,
    prolog_fma); trip counts are untouched and every per-nuclide value lies in
    the closed-form range of a body started from the prolog's range."""
    n, it = 300, 4
    _, nuc0, tr0 = oracle.rsbench(0, n, it, 3, fma_count=64, trips=True)
    acc, nuc, tr = oracle.rsbench(0, n, it, 3, fma_count=64, trips=True, prolog_fma=2048)
    assert np.array_equal(nuc, nuc0) and np.array_equal(tr, tr0)
    e_lo = expensive_closed_form(0.0, 2048) - expensive_tol(2048)
    e_hi = expensive_closed_form(1.0, 2048) + expensive_tol(2048)
    lo = expensive_closed_form(e_lo, 64) - expensive_tol(64)
    hi = expensive_closed_form(e_hi + 354 * 2.0**-9, 64) + expensive_tol(64)
    per = acc / nuc
    assert per.min() >= lo * (1 - 1e-5) and per.max() <= hi * (1 + 1e-5)
    acc_plain, _ = oracle.rsbench(0, n, it, 3, fma_count=64)
    assert not np.array_equal(acc, acc_plain)


def test_per_thread_sums_match_float64_definition():
    """Each thread's (acc, nuclides) re-derived from the definition (reading R8):
    lookup k draws Philox(k, RS<<16, thread); material = the first whose cumulative
    probability threshold floor(2^32 sum p) exceeds u0 (thresholds recomputed here
    from the published probabilities); E = U01(u1); nuclide j of material m is
    (37m + 13j) mod 355 and its body is Expensive() of fl(E + nuc/512) by the
    recurrence's closed form; acc is the in-order sum.  Nuclides exactly, acc
    within the accumulated binary32 rounding bound."""
    thr, cum = [], 0.0
    for i, p in enumerate(PROB):
        cum += p
        thr.append(2**32 - 1 if i == len(PROB) - 1 else math.floor(cum * 2**32))
    t0, n, iters, seed = 777, 64, 6, I.PRIMARY_SEED
    acc, nuc = oracle.rsbench(t0, n, iters, seed)
    key = [seed & 0xFFFFFFFF, seed >> 32]
    fma = 64
    for j in range(n):
        t = t0 + j
        a64, nn, mag = 0.0, 0, 0.0
        for k in range(iters):
            u = oracle.philox([k, 5 << 16, t & 0xFFFFFFFF, t >> 32], key)
            m = next(i for i, th in enumerate(thr) if int(u[0]) < th) if int(u[0]) < thr[-1] \
                else len(thr) - 1
            E = np.float32((int(u[1]) >> 8) * 2.0**-24)
            xs = 0.0
            for i in range(NUCS[m]):
                nid = (37 * m + 13 * i) % 355
                start = float(np.float32(E + np.float32(nid * 2.0**-9)))
                xs += expensive_closed_form(start, fma)
            a64 += xs
            mag += abs(xs) * NUCS[m] + abs(a64)
            nn += NUCS[m]
        assert nuc[j] == nn, j
        bound = nn * expensive_tol(fma) + mag * 2.0**-24
        assert abs(float(acc[j]) - a64) <= bound, (j, float(acc[j]), a64, bound)
