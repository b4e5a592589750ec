"""The all-cores oracle helper (tests/oracle_threads.py) reproduces the single-threaded oracle
bit for bit: summed integer tallies, concatenated per-thread / per-pixel outputs."""
import numpy as np

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from tests import oracle_threads as OT


def test_mcml_threads_equal_one_call():
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    one = oracle.mcml(p, 1000, 3000, 5)
    par = OT.mcml(p, 1000, 3000, 5, parts=7)
    for k in ("A", "Rd", "Tt", "counters_raw"):
        assert np.array_equal(one[k], par[k]), k


def test_rsbench_threads_equal_one_call():
    a1, n1 = oracle.rsbench(17, 301, 3, 9, 16, prolog_fma=8)
    a2, n2 = OT.rsbench(17, 301, 3, 9, 16, prolog_fma=8)
    assert np.array_equal(a1.view(np.uint32), a2.view(np.uint32)) and np.array_equal(n1, n2)


def test_pt_render_threads_equal_one_call():
    c = I.C4_SMALL
    tris, mat, mats, cam = I.cornell_scene(c)
    sc = oracle.pt_scene(tris, mat, mats, cam)
    pix = np.arange(5, c.width * c.height, 37, dtype=np.uint32)
    r1, c1 = oracle.pt_render(sc, c.width, c.height, 2, c.max_depth, 3, pixels=pix)
    r2, c2 = OT.pt_render(sc, c.width, c.height, 2, c.max_depth, 3, pix)
    assert np.array_equal(r1.view(np.uint32), r2.view(np.uint32)) and c1 == c2
