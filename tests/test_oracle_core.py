"""Pins of the oracle's RNG and math (no GPU).

Each pin ties the oracle to something other than itself: published
known-answer vectors, double-precision libm over every reachable input,
exact integer identities.
"""
import math
import os

import numpy as np
import pytest

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_philox_known_answers():
    rows = [l.split() for l in open(os.path.join(GOLDEN, "philox_kat.txt"))
            if l.strip() and not l.startswith("#")]
    assert len(rows) == 3
    for r in rows:
        v = [int(x, 16) for x in r]
        out = oracle.philox(v[0:4], v[4:6])
        assert [int(x) for x in out] == v[6:10]


def test_philox_distinct_counters_decorrelate():
    # 4096 counters differing in one word -> ~uniform outputs (mean of u01 ~ 1/2)
    vals = [oracle.philox([i, 1 << 16, 7, 0], [20200222, 0])[0] for i in range(4096)]
    u = np.array(vals, np.float64) / 2**32
    assert abs(u.mean() - 0.5) < 5 * math.sqrt(1 / 12 / 4096)
    assert len(set(vals)) == 4096


def test_u01_exact_and_bounded():
    L = oracle.lib()
    assert L.or_u01(0) == 0.0
    assert L.or_u01(0xFFFFFFFF) == 1.0 - 2.0**-24
    assert L.or_u01c(0) == 2.0**-24
    assert L.or_u01c(0xFFFFFFFF) == 1.0
    for u in (1 << 8, 12345 << 8, 0xDEADBEEF):
        assert L.or_u01(u) == (u >> 8) * 2.0**-24


def test_sr_logf_exhaustive_2ulp():
    # every x = k*2^-24, k in [1, 2^24], against double log (R5)
    assert oracle.lib().or_sweep_logf_ulp() <= 2.0


def test_sr_sincos2pif_exhaustive_2ulp():
    # every xi = k*2^-24, k < 2^24, against double sin/cos; exact zeros exact
    assert oracle.lib().or_sweep_sincos2pif_ulp() <= 2.0


def test_sr_math_special_values():
    assert oracle.sr_logf(1.0) == 0.0
    assert oracle.sr_logf(0.5) == pytest.approx(-math.log(2), rel=2**-23)
    assert oracle.sr_sincos2pif(0.0) == (0.0, 1.0)
    assert oracle.sr_sincos2pif(0.25) == (1.0, 0.0)
    assert oracle.sr_sincos2pif(0.5) == (0.0, -1.0)
    assert oracle.sr_sincos2pif(0.75) == (-1.0, 0.0)
    s, c = oracle.sr_sincos2pif(0.125)
    assert s == pytest.approx(math.sqrt(0.5), rel=2**-22) and s == c
