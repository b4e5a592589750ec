"""Pins of the lane-mask warp simulator (oracle part 2).

Fig. 1 worked example, closed forms, conservation laws and brute-force
enumeration of every want pattern / trip-count combination of 4-lane warps,
plus an exhaustive search over all legal interleavings for the optimum.
"""
import itertools
import math

import numpy as np
import pytest

import oracle
from oracle import PDOM, SPEC_LOOP, SPEC_CALL
from paper_conf_cgo_damanijskymg20_b200 import inputs as I


def test_fig1_worked_example():
    # Fig. 1: 4 lanes each want Expensive() in a different iteration.
    want = np.eye(4, dtype=np.uint8)
    pd = oracle.ws_divloop(want, PDOM, 0, W=4)
    assert pd["EXPENSIVE"] == (4, 4)      # run 4x serially, 1 lane each: 25%
    sr = oracle.ws_divloop(want, SPEC_LOOP, 4, W=4)
    assert sr["EXPENSIVE"] == (1, 4)      # run once, converged: 100%


def _all_patterns(W, L):
    for bits in range(1 << (W * L)):
        yield np.array([(bits >> b) & 1 for b in range(W * L)], np.uint8).reshape(W, L)


@pytest.mark.parametrize("L", [1, 2, 3, 4])
def test_divloop_bruteforce_4_lanes(L):
    W = 4
    for want in _all_patterns(W, L):
        K = want.sum(1)
        pd = oracle.ws_divloop(want, PDOM, 0, W=W)
        assert pd["EXPENSIVE"][1] == K.sum()
        assert pd["EXPENSIVE"][0] == int(want.any(0).sum())
        execs = []
        for T in range(1, W + 1):
            sr = oracle.ws_divloop(want, SPEC_LOOP, T, W=W)
            assert sr["EXPENSIVE"][1] == K.sum()                       # conservation
            assert sr["EXPENSIVE"][0] >= K.max()                        # lower bound
            assert sr["PROLOG"][1] == W * L                              # every iteration once
            execs.append(sr["EXPENSIVE"][0])
        assert execs[0] == pd["EXPENSIVE"][0]                           # T=1 == PDOM
        assert execs[-1] == K.max()                                     # T=W: max_l K_l


def test_divloop_optimum_exhaustive_search():
    rng = np.random.default_rng(0)
    pats = list(_all_patterns(3, 3)) + [rng.integers(0, 2, (4, 4)).astype(np.uint8)
                                        for _ in range(40)]
    for want in pats:
        opt = oracle.ws_divloop_optimum(want)
        assert opt == want.sum(1).max()
        assert oracle.ws_divloop(want, SPEC_LOOP, want.shape[0], W=want.shape[0])["EXPENSIVE"][0] == opt


def test_divloop_closed_forms_config1():
    c = I.C1
    want = oracle.divloop_wants(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.p_u32)
    p = c.p_u32 / 2**32
    n_warps = c.n_threads // 32
    pd, t32, t1 = [], [], []
    for w in range(n_warps):
        ww = want[32 * w:32 * w + 32]
        pd.append(oracle.ws_divloop(ww, PDOM, 0)["EXPENSIVE"][0])
        s32 = oracle.ws_divloop(ww, SPEC_LOOP, 32)
        t32.append(s32["EXPENSIVE"][0])
        assert t32[-1] == ww.sum(1).max()
        if w < 64:
            t1.append(oracle.ws_divloop(ww, SPEC_LOOP, 1)["EXPENSIVE"][0])
            assert t1[-1] == pd[-1]
    q = 1 - (1 - p) ** 32
    # PDOM: E[execs per warp] = iters * (1 - (1-p)^32) = 63.108
    assert abs(np.mean(pd) - c.iters * q) < 5 * math.sqrt(c.iters * q * (1 - q) / n_warps)
    # SR, T=32: E[max of 32 Binomial(64, p)] = sum_k (1 - F(k)^32) = 13.855
    from scipy.stats import binom
    ks = np.arange(0, c.iters + 1)
    e_max = float(np.sum(1 - binom.cdf(ks, c.iters, p) ** 32))
    assert abs(e_max - 13.855) < 5e-3
    assert abs(np.mean(t32) - e_max) < 0.15


def test_divloop_partial_warp_and_threshold_above_valid():
    want = np.array([[1, 0, 1], [0, 1, 1], [1, 1, 0]], np.uint8)
    sr = oracle.ws_divloop(want, SPEC_LOOP, 32, W=32)   # T > valid lanes: R = {} releases
    assert sr["EXPENSIVE"] == (2, 6)
    assert sr["ROUND"][1] == sr["ROUND"][0] * 3          # invalid lanes never in a mask


def test_commoncall_counts():
    for arm in ([1] * 32, [0] * 32, [1, 0] * 16):
        arm = np.array(arm, np.uint8)
        pd = oracle.ws_commoncall(arm, PDOM)
        sc = oracle.ws_commoncall(arm, SPEC_CALL)
        assert pd["CALL"][0] == int(arm.any()) + int((1 - arm).any())
        assert pd["CALL"][1] == 32 and sc["CALL"] == (1, 32)
    # foo-region efficiency 50% -> 100% for the 50/50 split
    arm = np.array([1, 0] * 16, np.uint8)
    pd = oracle.ws_commoncall(arm, PDOM)
    assert pd["CALL"][1] / (32 * pd["CALL"][0]) == 0.5


@pytest.mark.parametrize("K", [1, 2])
def test_loopmerge_bruteforce_4_lanes(K):
    W = 4
    for ns in itertools.product(range(1, 5), repeat=W * K):
        n = np.array(ns, np.uint32).reshape(W, K)
        pd = oracle.ws_loopmerge(n, PDOM, 0, W=W)
        assert pd["STEP"][1] == n.sum()
        assert pd["STEP"][0] == n.max(0).sum()                  # sum_k max_l n(l,k)
        t1 = oracle.ws_loopmerge(n, SPEC_LOOP, 1, W=W)
        assert t1["STEP"] == pd["STEP"]                         # T=1 == PDOM
        tw = oracle.ws_loopmerge(n, SPEC_LOOP, W, W=W)
        assert tw["STEP"][0] == n.sum(1).max()                  # max_l sum_k n(l,k)
        assert tw["STEP"][1] == n.sum()
        assert tw["LAUNCH"][1] == W * K
        for T in (2, 3):
            t = oracle.ws_loopmerge(n, SPEC_LOOP, T, W=W)
            assert t["STEP"][1] == n.sum() and t["STEP"][0] >= n.sum(1).max()


def test_loopmerge_event_split_sums_to_step():
    p = oracle.mc_params(I.C3.layers)
    K, W = 3, 32
    ev = [[oracle.mcml_events(p, l + k * W, 1) for k in range(K)] for l in range(W)]
    n = np.array([[len(e) for e in row] for row in ev], np.uint32)
    for mode, T in ((PDOM, 0), (SPEC_LOOP, 32), (SPEC_LOOP, 8)):
        r = oracle.ws_loopmerge(n, mode, T, events=ev)
        assert r["STEP_BOUNDARY"][1] + r["STEP_INTERACT"][1] == r["STEP"][1] == n.sum()


def _mc_events(K, W, seed):
    p = oracle.mc_params(I.C3.layers)
    ev, off, ns = oracle.mcml_events_batch(p, 0, W * K, seed)
    ids = np.arange(W)[:, None] + np.arange(K)[None, :] * W
    return ev, off, ns, ids


@pytest.mark.parametrize("T,Tb", [(32, 32), (32, 4), (16, 8), (1, 1)])
def test_loopmerge_defer_conservation(T, Tb):
    K, W = 4, 32
    ev, off, ns, ids = _mc_events(K, W, 9)
    r = oracle.ws_loopmerge_defer_raw(ns[ids], ev, off[ids].ravel(), T, Tb)
    nb = int(((ev & oracle.EV_BOUNDARY) != 0).sum())
    nm = int(((ev & oracle.EV_MATCHED) != 0).sum())    # equal-index boundaries: no part B
    assert 0 < nm < nb and not ((ev & oracle.EV_MATCHED) & ~((ev & 1) * 0xffff)).any()
    assert r["STEP"][1] == ns.sum()                   # every step runs part A once
    assert r["B_REL"][1] == nb - nm                   # every other boundary sub-step runs once
    assert r["EV0"][1] == nb                          # ... after parking in part A
    assert r["BI"][1] == nm                           # matched ones finish in part A
    assert r["A_TAIL"][1] == ns.sum() - (nb - nm)
    assert r["NEV0"][1] == ns.sum() - nb
    assert r["LAUNCH"][1] == W * K
    # the parked set is released in fewer executions than boundary steps
    assert r["B_REL"][0] <= max(nb, 1)


def test_loopmerge_defer_groups_boundaries():
    """Deferral raises the boundary code's active lanes per execution."""
    K, W = 8, 32
    ev, off, ns, ids = _mc_events(K, W, 4)
    plain = oracle.ws_loopmerge_raw(ns[ids], ev, off[ids].ravel(), oracle.SPEC_LOOP, 32)
    defer = oracle.ws_loopmerge_defer_raw(ns[ids], ev, off[ids].ravel(), 32, 8)
    eff = lambda x: x[1] / max(1, 32 * x[0])
    assert eff(defer["B_REL"]) > 4 * eff(plain["STEP_BOUNDARY"])


def test_divloop_advance_unroll_invariants():
    """V iterations per advance round: every lane-iteration's prolog still
    runs exactly once, every wanting iteration's Expensive exactly once; at T = 32 the
    releases (all lanes parked at their next wanting iteration) do not depend on V."""
    rng = np.random.default_rng(5)
    want = (rng.random((32, 64)) < 0.125).astype(np.uint8)
    base = oracle.ws_divloop(want, oracle.SPEC_LOOP, 32)
    for V in (2, 3, 8, 64):
        for T in (1, 8, 16, 32):
            s = oracle.ws_divloop(want, oracle.SPEC_LOOP, T, V=V)
            assert s["PROLOG"][1] == 32 * 64 - int(want.sum()) + int(want.sum())
            assert s["EXPENSIVE"][1] == int(want.sum())
            if T == 32:
                assert s["EXPENSIVE"] == base["EXPENSIVE"]
            assert s["rounds"] <= oracle.ws_divloop(want, oracle.SPEC_LOOP, T)["rounds"]


# ------------------------------------------------------------------ task pool
def _pool_makespan(ns, W):
    """Greedy list schedule of the pool (task q = k*n_valid + l, in order) on W
    unit-speed lanes, ties to the lower lane: written independently of the
    simulator, as an event simulation over time."""
    n_valid, K = ns.shape
    tasks = [int(ns[q % n_valid, q // n_valid]) for q in range(n_valid * K)]
    free_at = [0] * W
    end = 0
    for d in tasks:
        t = min(free_at)
        lane = free_at.index(t)   # lowest lane among the earliest free
        free_at[lane] = t + d
        end = max(end, t + d)
    return end


@pytest.mark.parametrize("K,vals", [(1, [1, 2, 3, 4]), (2, [1, 2, 3]), (3, [1, 3])])
def test_pool_bruteforce_4_lanes(K, vals):
    """every trip-count combination in {1,2,3}^(4K) of a 4-lane warp:
    conservation, T = 1 runs the pool batch by batch (STEP executions = sum of
    each batch's longest task), T = W is greedy list scheduling (STEP executions
    = its makespan), U > 1 never adds rounds or releases"""
    W = 4
    for combo in itertools.product(vals, repeat=W * K):
        ns = np.array(combo, np.uint32).reshape(W, K)
        tot = int(ns.sum())
        s1 = oracle.ws_loopmerge_pool(ns, 1, W=W)
        sW = oracle.ws_loopmerge_pool(ns, W, W=W)
        for s in (s1, sW):
            assert s["STEP"][1] == tot and s["RELEASE"] == s["STEP"]
            assert s["LAUNCH"][1] == W * K
            assert s["rounds"] == s["RELEASE"][0] + s["ADVANCE"][0]
        tasks = [int(ns[q % W, q // W]) for q in range(W * K)]
        assert s1["STEP"][0] == sum(max(tasks[b:b + W]) for b in range(0, W * K, W))
        assert s1["ADVANCE"][0] == K
        assert sW["STEP"][0] == _pool_makespan(ns, W)
        for U in (2, 3):
            su = oracle.ws_loopmerge_pool(ns, W, U=U, W=W)
            assert su["STEP"][1] == tot and su["LAUNCH"][1] == W * K
            assert su["RELEASE"][0] <= sW["RELEASE"][0] and su["rounds"] <= sW["rounds"]


def test_pool_partial_warp_and_hand_schedule():
    # 3 valid threads x 2 tasks on a 4-lane warp: the 4th lane works too
    ns = np.array([[3, 1], [2, 2], [1, 5]], np.uint32)
    s = oracle.ws_loopmerge_pool(ns, 4, W=4)
    # tasks q0..q5 = 3,2,1,1,2,5; lanes 0..3 take q0..q3 at t=0 (3,2,1,1);
    # t=1: lanes 2,3 free -> q4 (2) on lane 2, q5 (5) on lane 3 -> ends at 6
    assert s["STEP"] == (6, 14) and s["LAUNCH"] == (2, 6) and s["ENTRY"] == (1, 3)
    assert s["ADVANCE"] == (2, 4 + 2)   # round 1: all 4 lanes idle; t=1: lanes 2, 3


# ------------------------------------------------------------------ task stream (MC dynamic claiming)
def _stream_ref(ns, W, T, U=1):
    """the dynamic-claim schedule as an independent set-based event loop"""
    Q = len(ns)
    alive, exh, left, q = set(), set(), {}, 0
    rounds, rel, adv, launch = 0, [0, 0], [0, 0], [0, 0]
    while True:
        P = set(alive)
        R = {l for l in range(W) if l not in alive and l not in exh}
        if not P and not R:
            break
        rounds += 1
        if len(P) >= T or not R:
            S = set(P)
            for _ in range(U):
                if not S:
                    break
                rel[0] += 1
                rel[1] += len(S)
                for l in sorted(S):
                    left[l] -= 1
                    if left[l] == 0:
                        alive.discard(l)
                        S.discard(l)
        else:
            adv[0] += 1
            adv[1] += len(R)
            got = 0
            for l in sorted(R):
                if q >= Q:
                    exh.add(l)
                    continue
                left[l] = int(ns[q])
                q += 1
                got += 1
                alive.add(l)
            if got:
                launch[0] += 1
                launch[1] += got
    return rounds, tuple(rel), tuple(adv), tuple(launch)


def test_stream_matches_reference_and_closed_forms():
    rng = np.random.default_rng(5)
    for trial in range(400):
        W = int(rng.integers(1, 9))
        Q = int(rng.integers(0, 40))
        ns = rng.integers(1, 7, Q).astype(np.uint32)
        T = int(rng.integers(1, W + 1))
        U = int(rng.integers(1, 4))
        s = oracle.ws_loopmerge_stream(ns, SPEC_LOOP, T, U=U, W=W)
        r = _stream_ref(ns, W, T, U)
        assert (s["rounds"], s["STEP"], s["ADVANCE"], s["LAUNCH"]) == r, (trial, ns, W, T, U)
        assert s["STEP"][1] == int(ns.sum()) and s["LAUNCH"][1] == Q
        pd = oracle.ws_loopmerge_stream(ns, PDOM, 0, W=W)
        assert pd["STEP"][1] == int(ns.sum()) and pd["LAUNCH"][1] == Q
        assert pd["STEP"][0] == sum(int(ns[b:b + W].max()) for b in range(0, Q, W))


def test_stream_events_split_every_step():
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    ev, off, ns = oracle.mcml_events_batch(p, 0, 200, I.PRIMARY_SEED)
    s = oracle.ws_loopmerge_stream(ns, SPEC_LOOP, 32, U=4, ev=np.ascontiguousarray(ev),
                                   ev_off=off)
    assert s["STEP"][1] == int(ns.sum()) == len(ev)
    assert s["STEP_BOUNDARY"][1] + s["STEP_INTERACT"][1] == s["STEP"][1]
    assert s["STEP_BOUNDARY"][1] == int((np.asarray(ev) & 1).sum())
