"""Pins of the oracle's Monte Carlo photon transport (configs 3/5).

Closed forms (Beer-Lambert, Rsp, Fresnel equations), an exact integer
conservation law, a published benchmark slab, and sharding invariance.
"""
import math
import os

import numpy as np
import pytest

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
FX = 2.0**32


def P(m):
    return oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)


def test_beer_lambert_absorbed_fraction_and_depth_profile():
    m = I.BEER_LAMBERT
    N = 400000
    o = oracle.mcml(P(m), 0, N, I.PRIMARY_SEED)
    mua, d = m.layers[0][1], m.layers[0][4]
    A_exact = 1 - math.exp(-mua * d)
    sig = math.sqrt(A_exact * (1 - A_exact) / N)
    assert abs(o["A"].sum() / FX / N - A_exact) < 5 * sig
    assert abs(o["Tt"].sum() / FX / N - (1 - A_exact)) < 5 * sig
    assert o["Rd"].sum() == 0
    # all absorption on the axis (pencil beam, no scattering)
    assert o["A"][:, 1:].sum() == 0
    # depth histogram vs mua*exp(-mua z): chi^2 over the 100 bins
    counts = o["A"][:, 0] / FX
    assert np.all(counts == np.round(counts))  # each absorption deposits w = 1 exactly
    z = np.arange(m.nz + 1) * m.dz
    expect = N * (np.exp(-mua * z[:-1]) - np.exp(-mua * z[1:]))
    chi2 = ((counts - expect) ** 2 / expect).sum()
    assert chi2 < m.nz + 5 * math.sqrt(2 * m.nz)


def test_mismatched_absorber_multiple_reflection_closed_form():
    """n = 1.4 slab in air, mua = 5, mus = 0, d = 0.1 cm, pencil beam at normal
    incidence: every boundary hit is the ca1 > COSZERO case, r = ((n-1)/(n+1))^2
    at both faces, and (mus = 0) an interaction deposits the whole weight.  With
    T = exp(-mua d) the photon that entered (weight w0 = 1 - r) leaves through
    the bottom with probability T(1-r)/(1-r^2 T^2) and through the top with
    r T^2 (1-r)/(1-r^2 T^2) (the multiple-reflection series).  Pins the
    mismatched-boundary branch in transport: reflect vs transmit, the uz
    reversal, s_left continuation, Rd at the top and Tt at the bottom."""
    m = I.MISMATCHED_ABSORBER
    p = P(m)
    N = 400000
    o = oracle.mcml(p, 0, N, I.PRIMARY_SEED)
    c = o["counters"]
    n_, mua, _, _, d = m.layers[0]
    r = ((n_ - 1.0) / (n_ + 1.0)) ** 2
    T = math.exp(-mua * d)
    den = 1.0 - r * r * T * T
    p_tt, p_rd = T * (1 - r) / den, r * T * T * (1 - r) / den
    for k, pk in (("tt_exits", p_tt), ("rd_exits", p_rd)):
        assert abs(c[k] / N - pk) < 5 * math.sqrt(pk * (1 - pk) / N), (k, c[k] / N, pk)
    # every exit and every absorption carries the whole entering weight, on axis
    w0 = np.float32(1.0) - np.float32(oracle.mcml_rsp(p))
    fxw = int(np.float32(w0) * np.float32(FX))
    assert int(o["Tt"].sum()) == c["tt_exits"] * fxw and int(o["Tt"][1:].sum()) == 0
    assert int(o["Rd"].sum()) == c["rd_exits"] * fxw and int(o["Rd"][1:].sum()) == 0
    n_abs = N - c["tt_exits"] - c["rd_exits"]
    assert int(o["A"].sum()) == n_abs * fxw and o["A"][:, 1:].sum() == 0
    assert c["rr_kills"] == 0 and c["capped"] == 0 and c["zero_w"] == n_abs
    # absorption depth profile: the downward pass k contributes mua e^{-mua z}
    # weighted by (r^2 T^2)^k, the upward pass the mirror image weighted by r T (...)
    z = np.arange(m.nz + 1) * m.dz
    down = np.exp(-mua * z[:-1]) - np.exp(-mua * z[1:])
    up = np.exp(-mua * (d - z[1:])) - np.exp(-mua * (d - z[:-1]))
    expect = N * (down + r * T * up) / den
    counts = o["A"][:, 0] / float(fxw)
    chi2 = ((counts - expect) ** 2 / expect).sum()
    assert chi2 < m.nz + 5 * math.sqrt(2 * m.nz)


def test_specular_reflectance_closed_form():
    p = P(I.C3)
    assert oracle.mcml_rsp(p) == pytest.approx(((1.0 - 1.4) / (1.0 + 1.4)) ** 2, rel=1e-6)


@pytest.mark.parametrize("ni,nt", [(1.4, 1.0), (1.0, 1.4), (1.33, 1.5)])
def test_fresnel_matches_textbook(ni, nt):
    L = oracle.lib()
    import ctypes as C
    L.or_mcml_fresnel.argtypes = [C.c_float, C.c_float, C.c_float, C.POINTER(C.c_float)]
    L.or_mcml_fresnel.restype = C.c_float
    for th in np.linspace(0.0, 89.0, 60):
        c1 = math.cos(math.radians(th))
        s2 = ni / nt * math.sin(math.radians(th))
        ca2 = C.c_float()
        r = L.or_mcml_fresnel(ni, nt, np.float32(c1), C.byref(ca2))
        if s2 >= 1.0:
            assert r == 1.0
            continue
        c2 = math.sqrt(1 - s2 * s2)
        rs = ((ni * c1 - nt * c2) / (ni * c1 + nt * c2)) ** 2
        rp = ((ni * c2 - nt * c1) / (ni * c2 + nt * c1)) ** 2
        assert r == pytest.approx(0.5 * (rs + rp), rel=2e-4, abs=2e-6)
        assert ca2.value == pytest.approx(c2, rel=1e-5, abs=1e-6)


def test_no_absorption_conserves_weight_exactly():
    m = I.NO_ABSORPTION
    p = P(m)
    N = 20000
    o = oracle.mcml(p, 0, N, I.PRIMARY_SEED)
    c = o["counters"]
    assert o["A"].sum() == 0 and c["rr_kills"] == 0 and c["capped"] == 0
    assert c["rd_exits"] + c["tt_exits"] == N
    w0 = np.float32(1.0) - np.float32(oracle.mcml_rsp(p))
    fxw = int(np.float32(w0) * np.float32(FX))
    assert int(o["Rd"].sum()) + int(o["Tt"].sum()) == N * fxw


def test_van_de_hulst_slab():
    row = [l.split() for l in open(os.path.join(GOLDEN, "mcml_validation.txt"))
           if l.strip() and not l.startswith("#")][0]
    n_, mua, mus, g, d, Rd_ref, Tt_ref = map(float, row[1:])
    m = I.MCML(layers=((n_, mua, mus, g, d),))
    N = 1_000_000
    o = oracle.mcml(P(m), 0, N, I.PRIMARY_SEED)
    Rd = o["Rd"].sum() / FX / N
    Tt = o["Tt"].sum() / FX / N
    assert abs(Rd - Rd_ref) < 5 * math.sqrt(Rd_ref * (1 - Rd_ref) / N)
    assert abs(Tt - Tt_ref) < 5 * math.sqrt(Tt_ref * (1 - Tt_ref) / N)


def test_energy_balance_three_layer():
    # absorbed + reflected + transmitted + Rsp + roulette balance ~ 1
    p = P(I.C3)
    N = 20000
    o = oracle.mcml(p, 0, N, I.PRIMARY_SEED)
    tot = (o["A"].sum() + o["Rd"].sum() + o["Tt"].sum()) / FX / N + oracle.mcml_rsp(p)
    assert abs(tot - 1.0) < 0.01  # roulette is unbiased, not exact
    c = o["counters"]
    assert c["photons"] == N
    assert c["rd_exits"] + c["tt_exits"] + c["rr_kills"] + c["capped"] + c["zero_w"] == N


def test_sharding_invariance_exact():
    p = P(I.C3)
    full = oracle.mcml(p, 1000, 600, 5)
    parts = [oracle.mcml(p, 1000 + a, b - a, 5) for a, b in ((0, 250), (250, 251), (251, 600))]
    for key in ("A", "Rd", "Tt", "counters_raw"):
        s = sum(q[key].astype(np.uint64) for q in parts)
        assert np.array_equal(s, full[key])


def test_event_stream_matches_step_counts():
    p = P(I.C3)
    o = oracle.mcml(p, 77, 20, 3, steps=True)
    for k in range(20):
        ev = oracle.mcml_events(p, 77 + k, 3).astype(np.int64)
        assert len(ev) == o["steps"][k]
        bnd = (ev & oracle.EV_BOUNDARY) != 0
        outcome = ev & (oracle.EV_REFLECT | oracle.EV_EXIT | oracle.EV_TRANSMIT)
        spin = ev & (oracle.EV_SPIN_AXIS | oracle.EV_SPIN_GENERAL)
        # a boundary step has exactly one outcome and no spin; an interaction the reverse
        assert np.all(np.where(bnd, np.isin(outcome, [4, 8, 16]), outcome == 0))
        assert np.all(np.where(bnd, spin == 0, np.isin(spin, [64, 128])))
        # the step after a boundary step resumes the leftover path length
        assert np.all(((ev[1:] & oracle.EV_SLEFT) != 0) == bnd[:-1])
        assert (ev[0] & oracle.EV_SLEFT) == 0
        # only the last step can exit
        assert np.all((ev[:-1] & oracle.EV_EXIT) == 0)


def test_equal_layers_equal_one_slab():
    """A slab cut into three layers with identical optics scatters light exactly
    like the uncut slab (an internal boundary between equal indices is not
    physical: Fresnel r = 0, the step continues with its leftover length, MCML
    ref. [2] of the paper).  Pins the layer-crossing code -- leftover path
    length, layer index, the matched-boundary branch -- statistically: Rd, Tt
    and the absorbed weight per depth band agree within 5 sigma (sigma the
    [0,1]-bounded-mean bound sqrt(p(1-p)/N), doubled for the difference)."""
    n_, mua, mus, g = 1.4, 2.0, 98.0, 0.8
    one = I.MCML(layers=((n_, mua, mus, g, 0.06),), nz=60, dz=0.001)
    three = I.MCML(layers=((n_, mua, mus, g, 0.02),) * 3, nz=60, dz=0.001)
    N = 200000
    a = oracle.mcml(P(one), 0, N, I.PRIMARY_SEED)
    b = oracle.mcml(P(three), 0, N, I.PRIMARY_SEED)
    ev = np.concatenate([oracle.mcml_events(P(three), k, I.PRIMARY_SEED) for k in range(200)])
    assert ((ev & oracle.EV_MATCHED) != 0).sum() > 0     # the crossings happen
    bands = lambda o: o["A"].sum(axis=1).reshape(6, 10).sum(axis=1)
    for qa, qb in [(a["Rd"].sum(), b["Rd"].sum()), (a["Tt"].sum(), b["Tt"].sum()),
                   *zip(bands(a), bands(b))]:
        pa, pb = qa / FX / N, qb / FX / N
        sig = math.sqrt(max(pa, 1e-6) * (1 - pa) / N)
        assert abs(pa - pb) < 2 * 5 * sig, (pa, pb)


def test_matched_boundary_events():
    """MATCHED marks exactly the boundary steps between layers of equal index:
    never an exit, always a reflect or a transmit, and only inside the slab."""
    p = P(I.C3)
    for k in range(50):
        ev = oracle.mcml_events(p, k, I.PRIMARY_SEED).astype(np.int64)
        m = (ev & oracle.EV_MATCHED) != 0
        assert np.all((ev[m] & oracle.EV_BOUNDARY) != 0)
        assert np.all((ev[m] & (oracle.EV_EXIT | oracle.EV_EXTERNAL)) == 0)
        assert np.all(np.isin(ev[m] & (oracle.EV_REFLECT | oracle.EV_TRANSMIT), [4, 16]))
    # configs[2] has equal indices throughout: every internal crossing is matched
    ev = np.concatenate([oracle.mcml_events(p, k, I.PRIMARY_SEED) for k in range(300)]).astype(np.int64)
    internal = ((ev & oracle.EV_BOUNDARY) != 0) & ((ev & oracle.EV_EXTERNAL) == 0)
    assert np.array_equal(internal, (ev & oracle.EV_MATCHED) != 0)
