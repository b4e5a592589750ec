"""Full-size parity: every configuration at BASELINE.json's size, in the launch configuration
bench.py times, compared element by element with the oracle run on every host core
(tests/oracle_threads.py; the oracle itself is unchanged, only split over disjoint task ranges).

* configs[2] MC: all 10^7 photons, SPEC_LOOP (dynamic claiming, merge unroll, T = 32) and PDOM,
  every tally bin and counter bit-exact (integer);
* NEXT-1 RSBench: all 131072 x 32 lookups of both the plain and the expensive-fetch variant
  at their bench unroll and threshold, every per-thread sum bit-exact;
* configs[3] path tracer: one full image row and one full column of the 1024^2 x 16 spp frame
  (2047 pixels, every sample), SPEC and PDOM, bit-exact.

Barriers "are not required for correctness of the program": every schedule must
reproduce the unannotated program's result, which is what the oracle computes.
"""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import sr
from tests import oracle_threads as OT

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


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


@pytest.fixture(scope="module")
def mc_ref():
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    return OT.mcml(p, 0, m.n_photons, I.PRIMARY_SEED)


@pytest.mark.parametrize("mode,T", [(sr.SPEC_LOOP, I.C3.threshold), (sr.PDOM, 0)])
def test_mcml_full_config_equals_oracle(ctx, mc_ref, mode, T):
    m = I.C3
    w = sr.mcml_workload(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap,
                         unroll=m.merge_unroll)          # bench.py's launch configuration
    ctx.ensure(sr.sr_workspace_bytes(w, m.n_threads))
    sr.sr_run(w, m.n_threads, m.iters, I.PRIMARY_SEED, mode, T)
    g = u64(ctx.region(w, m.n_threads, sr.T_GRID, torch.int64))
    cnt = u64(ctx.region(w, m.n_threads, sr.T_COUNTERS, torch.int64))
    nA = m.nz * m.nr
    assert np.array_equal(g[:nA], mc_ref["A"].ravel())
    assert np.array_equal(g[nA:nA + m.nr], mc_ref["Rd"])
    assert np.array_equal(g[nA + m.nr:], mc_ref["Tt"])
    assert np.array_equal(cnt[:8], mc_ref["counters_raw"])
    assert int(cnt[0]) == m.n_photons


@pytest.mark.parametrize("cfg_name", ["NEXT1", "NEXT1_FETCH"])
def test_rsbench_full_config_equals_oracle(ctx, cfg_name):
    c = getattr(I, cfg_name)
    acc_o, nuc_o = OT.rsbench(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.fma_count,
                              prolog_fma=c.prolog_fma)
    w = sr.rsbench_workload(c.fma_count, prolog_fma=c.prolog_fma, unroll=c.merge_unroll)
    ctx.ensure(sr.sr_workspace_bytes(w, c.n_threads))
    for mode, T in ((sr.SPEC_LOOP, c.threshold), (sr.PDOM, 0)):
        sr.sr_run(w, c.n_threads, c.iters, I.PRIMARY_SEED, mode, T)
        out = ctx.region(w, c.n_threads, sr.T_PERTHREAD, torch.int32).view(-1, 2).cpu().numpy()
        assert np.array_equal(out[:, 0].view(np.uint32), acc_o.view(np.uint32)), (mode, T)
        assert np.array_equal(out[:, 1].view(np.uint32), nuc_o), (mode, T)
        cnt = u64(ctx.region(w, c.n_threads, sr.T_COUNTERS, torch.int64))
        assert int(cnt[0]) == int(nuc_o.sum())


def test_pathtrace_full_row_and_column_equal_oracle(ctx):
    c = I.C4
    tris, mat, mats, cam = I.cornell_scene(c)
    buf, used = sr.upload_scene(tris, mat, mats, cam)
    row, col = 511, 300
    pix = np.unique(np.concatenate([row * c.width + np.arange(c.width),
                                    np.arange(c.height) * c.width + col])).astype(np.uint32)
    assert len(pix) == c.width + c.height - 1
    ref, rc = OT.pt_render(oracle.pt_scene(tris, mat, mats, cam), c.width, c.height, c.spp,
                           c.max_depth, I.PRIMARY_SEED, pix)
    w = sr.pathtrace_workload(buf.data_ptr(), used, c.width, c.height, c.max_depth)
    ctx.ensure(sr.sr_workspace_bytes(w, c.n_pixels))
    for mode, T in ((sr.SPEC_LOOP, c.threshold), (sr.PDOM, 0)):
        sr.sr_run(w, c.n_pixels, c.spp, I.PRIMARY_SEED, mode, T)
        rgb = ctx.region(w, c.n_pixels, sr.T_PERTHREAD, torch.float32).view(-1, 3).cpu().numpy()
        bad = np.nonzero((rgb[pix].view(np.uint32) != ref.view(np.uint32)).any(1))[0]
        assert bad.size == 0, (mode, pix[bad[:5]], rgb[pix[bad[:5]]], ref[bad[:5]])
    assert rc["paths"] == len(pix) * c.spp
