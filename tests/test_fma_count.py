"""GPU pin (iv) of SURVEY.md Sec. 8(c6): the FP32 FMAs the kernels EXECUTE
(ncu `sm__sass_thread_inst_executed_op_ffma{,2}_pred_on`, predicated-on lanes
only) equal the algorithmic FMAs of the workload exactly -- `fma_count` per
Expensive() call times the number of calls the oracle's event streams imply.
So neither schedule runs the common code for a lane that does not want it
(the masks are exact), and SR runs precisely the work PDOM runs (P:262-265:
speculation only moves convergence).

Runs on CPU over the committed ncu capture (profiles/simt_efficiency.json) of
the SAME SASS (per-kernel hash); a stale capture skips."""
import json
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

from paper_conf_cgo_damanijskymg20_b200 import inputs as I  # noqa: E402


def expensive_calls(family):
    """(calls, fma_count) at the configs[] size the profile launches."""
    import numpy as np
    import oracle
    if family == "divloop":
        c = I.C1
        want = oracle.divloop_wants(0, c.n_threads, c.iters, I.PRIMARY_SEED, c.p_u32)
        return int(np.asarray(want).sum()), c.fma_count
    if family == "commoncall":
        c = I.C2
        return c.n_threads * c.iters, c.fma_count
    c = I.NEXT1
    _, _, trips = oracle.rsbench(0, c.n_threads, c.iters, I.PRIMARY_SEED, fma_count=0, trips=True)
    return int(np.asarray(trips, dtype=np.int64).sum()), c.fma_count


CASES = [("divloop_pdom", "divloop"), ("divloop_spec(T=16)", "divloop"),
         ("commoncall_pdom", "commoncall"), ("commoncall_spec", "commoncall"),
         ("rs_pdom", "rsbench"), ("rs_spec(T=24)", "rsbench")]


@pytest.fixture(scope="module")
def measured():
    import __graft_entry__
    __graft_entry__.build()
    import sass_regions
    return (json.load(open(os.path.join(ROOT, "profiles", "simt_efficiency.json"))),
            set(sass_regions.kernel_hashes("divloop_|commoncall_|rs_").values()))


@pytest.mark.parametrize("label,family", CASES)
def test_executed_fmas_equal_algorithmic_fmas(measured, label, family):
    m, hashes = measured
    r = m.get(label)
    if not r or r.get("ffma2_thread_inst") is None:
        pytest.skip(f"no ffma2 count for {label} in profiles/simt_efficiency.json")
    if r.get("sass_sha") not in hashes:
        pytest.skip(f"{label}: stored ncu measurement is for different SASS (re-profile)")
    calls, fma = expensive_calls(family)
    # Expensive() = fma_count/2 FFMA2 (two chains per instruction), no scalar FFMA
    assert r["ffma2_thread_inst"] * 2 + r["ffma_thread_inst"] == calls * fma, (label, r, calls)
