"""The C ABI boundary without a GPU: the library loads, exports every symbol
include/sr.h declares, validates arguments before touching a device, and
reports missing devices as SR_E_CUDA (there is no CPU fallback)."""
import ctypes as C
import os
import re

import pytest

import __graft_entry__  # noqa: F401  (sys.path)
from paper_conf_cgo_damanijskymg20_b200 import build as B
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import sr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def lib():
    B.build()
    return sr.load()


def declared_symbols():
    txt = open(os.path.join(ROOT, "include", "sr.h")).read()
    return sorted(set(re.findall(r"SR_API\s+[\w\s\*]*?\b(sr_\w+)\s*\(", txt)))


def test_exports_every_declared_symbol(lib):
    syms = declared_symbols()
    assert set(syms) == set(sr.EXPORTS)
    for s in syms:
        assert hasattr(lib, s), s


def test_struct_layout_matches_header():
    # compile a tiny C probe against include/sr.h and compare sizeof/offsetof
    import subprocess
    import tempfile
    src = r'''
#include <stdio.h>
#include <stddef.h>
#include "sr.h"
int main(void){
 printf("%zu %zu %zu %zu %zu %zu %zu\n", sizeof(sr_workload), offsetof(sr_workload, divloop),
  offsetof(sr_workload, commoncall), offsetof(sr_workload, mcml), offsetof(sr_workload, pathtrace),
  sizeof(sr_mcml_params), offsetof(sr_workload, grid_ctas));
 return 0;}
'''
    with tempfile.TemporaryDirectory() as d:
        open(os.path.join(d, "p.c"), "w").write(src)
        subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), "-o",
                               os.path.join(d, "p"), os.path.join(d, "p.c")])
        got = list(map(int, subprocess.check_output([os.path.join(d, "p")]).split()))
    W = sr.Workload
    assert got == [C.sizeof(W), W.divloop.offset, W.commoncall.offset, W.mcml.offset,
                   W.pathtrace.offset, C.sizeof(sr.MCMLParams), W.grid_ctas.offset]


def test_no_gpu_is_reported_as_cuda_error():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(sr.SRError) as e:
        sr.sr_init(0, None, None, 0)
    assert e.value.code == sr.SR_E_CUDA


def test_run_validation_before_state():
    w = sr.divloop_workload()
    cases = [
        (dict(n=0), sr.SR_E_INVALID),
        (dict(threshold=33), sr.SR_E_INVALID),
        (dict(mode=sr.SPEC_CALL), sr.SR_E_INVALID),       # call merge is for COMMONCALL only
        (dict(mode=7), sr.SR_E_INVALID),
        (dict(iters=1 << 31, n=1 << 33), sr.SR_E_INVALID),  # n*iters overflow
        (dict(), sr.SR_E_STATE),                           # valid, but no sr_init
    ]
    for kw, code in cases:
        a = dict(n=64, iters=4, mode=sr.SPEC_LOOP, threshold=16); a.update(kw)
        with pytest.raises(sr.SRError) as e:
            sr.sr_run(w, a["n"], a["iters"], 1, a["mode"], a["threshold"])
        assert e.value.code == code, (kw, str(e.value))
    cc = sr.commoncall_workload()
    for mode, T in ((sr.SPEC_LOOP, 0), (sr.SPEC_CALL, 16)):
        with pytest.raises(sr.SRError) as e:
            sr.sr_run(cc, 64, 1, 1, mode, T)
        assert e.value.code == sr.SR_E_INVALID
    bad = sr.divloop_workload(fma_count=1001)
    with pytest.raises(sr.SRError) as e:
        sr.sr_run(bad, 64, 1, 1, sr.PDOM, 0)
    assert e.value.code == sr.SR_E_INVALID and "multiple of 8" in str(e.value)
    bad = sr.divloop_workload(block=48)
    with pytest.raises(sr.SRError):
        sr.sr_run(bad, 64, 1, 1, sr.PDOM, 0)
    for batch in (2, 8, 63, 65):
        bad = sr.divloop_workload(batch=batch)
        with pytest.raises(sr.SRError) as e:
            sr.sr_run(bad, 64, 1, 1, sr.PDOM, 0)
        assert e.value.code == sr.SR_E_INVALID and "prolog_batch" in str(e.value)
    with pytest.raises(sr.SRError) as e:
        sr.sr_run(sr.divloop_workload(flags=sr.F_POOL), 64, 1, 1, sr.SPEC_LOOP, 16)
    assert e.value.code == sr.SR_E_INVALID and "SR_F_POOL" in str(e.value)
    with pytest.raises(sr.SRError) as e:
        sr.sr_run(sr.divloop_workload(batch=64, block=1024), 64, 1, 1, sr.PDOM, 0)
    assert e.value.code == sr.SR_E_INVALID and "block_threads <= 512" in str(e.value)
    for fl, spp in ((sr.F_POOL, 0), (sr.F_POOL | sr.F_COARSE, 4), (sr.F_POOL | sr.F_MATGROUP, 4),
                    (sr.F_POOL, 5000)):
        bad = sr.pathtrace_workload(1 << 20, 1 << 20, 8, 8, flags=fl, pool_spp=spp)
        with pytest.raises(sr.SRError) as e:
            sr.sr_run(bad, 64, 4, 1, sr.SPEC_LOOP, 12)
        assert e.value.code == sr.SR_E_INVALID and "SR_F_POOL" in str(e.value)
    for split in (3, 5, 8):
        bad = sr.divloop_workload(batch=64, flags=sr.F_POOL, split=split)
        with pytest.raises(sr.SRError) as e:
            sr.sr_run(bad, 64, 64, 1, sr.SPEC_LOOP, 16)
        assert e.value.code == sr.SR_E_INVALID and "pool_split" in str(e.value)


def test_mcml_param_validation():
    m = I.C3
    for layers in ([], [(1.4, -1.0, 10.0, 0.9, 0.1)], [(1.4, 1.0, 10.0, 1.0, 0.1)],
                   [(1.4, 0.0, 0.0, 0.5, 0.1)], [(1.4, 1, 1, 0.5, 0.1)] * 9):
        w = sr.mcml_workload(layers) if len(layers) <= 8 else None
        if w is None:
            continue
        with pytest.raises(sr.SRError) as e:
            sr.sr_workspace_region(w, 100, sr.T_GRID)
        assert e.value.code == sr.SR_E_INVALID
    w = sr.mcml_workload(m.layers, nr=0)
    assert sr.sr_workspace_bytes(w, 100) == 0


def test_workspace_layout():
    m = I.C3
    w = sr.mcml_workload(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    og, ng = sr.sr_workspace_region(w, 1000, sr.T_GRID)
    oc, nc = sr.sr_workspace_region(w, 1000, sr.T_COUNTERS)
    assert ng == 8 * (m.nz * m.nr + 2 * m.nr) and nc == 8 * sr.N_COUNTERS
    assert oc == og + ng                  # one contiguous int64 all-reduce
    assert og % 256 == 0
    assert sr.sr_workspace_region(w, 1000, sr.T_PERTHREAD)[1] == 0
    d = sr.divloop_workload()
    assert sr.sr_workspace_region(d, 1000, sr.T_PERTHREAD)[1] == 8000
    assert sr.sr_workspace_region(d, 1000, sr.T_SCHED)[1] == 0
    ds = sr.divloop_workload(flags=sr.F_SCHED)
    assert sr.sr_workspace_region(ds, 1000, sr.T_SCHED)[1] == 32 * 32
    total = sr.sr_workspace_bytes(ds, 1000)
    for r in range(5):
        o, n = sr.sr_workspace_region(ds, 1000, r)
        assert o + n <= total


def test_tally_and_finalize_state():
    sr.sr_finalize()
    sr.sr_finalize()  # idempotent
    with pytest.raises(sr.SRError) as e:
        sr.sr_tally(sr.T_COUNTERS, None, 0)
    assert e.value.code == sr.SR_E_STATE
    assert "sm_100a" in sr.sr_build_info()


def test_sass_is_sm100a_and_uses_the_intended_instructions():
    import subprocess
    out = subprocess.run(["cuobjdump", "-sass", sr.LIB_PATH], capture_output=True, text=True).stdout
    assert "arch = sm_100a" in out
    funcs = {}
    cur = None
    for line in out.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            cur = m.group(1); funcs[cur] = []
        elif cur and "/*" in line:
            funcs[cur].append(line)
    def ops(pat, name):
        return sum(1 for l in funcs[name] if re.search(pat, l))
    for f in funcs:
        if "commoncall_pdom" in f:
            assert ops(r"\bCALL\.", f) == 2, f          # foo from both arms
        if "commoncall_spec" in f:
            assert ops(r"\bCALL\.", f) == 1, f          # the one hoisted call
        if "divloop_spec" in f or "mcml_spec" in f:
            assert ops(r"\bVOTE\.", f) >= 2, f          # __ballot_sync scheduler
        if "ILi125ELb0" in f:
            assert ops(r"\bFFMA2\b", f) == 500, f       # 1000 FMAs as FFMA2, unrolled
        if re.search(r"\dmcml_(pdom|spec)", f):
            # paired IEEE products only: every FFMA2 adds the -0 pair from the kernel
            # parameters (a uniform register), never a contracted product + sum
            # -- except the three FFMA2 of div2_dom (the rotation's paired quotients,
            # explicit fma.rn.f32x2) in the FAST kernels
            ff = [l for l in funcs[f] if re.search(r"\bFFMA2\b", l)]
            assert ff, f
            other = [l for l in ff
                     if not re.search(r"FFMA2\s+[^;]*,\s*([^,;]+);", l).group(1).strip()
                     .startswith("UR")]
            assert len(other) == (3 if re.search(r"ILb[01]ELb[01]ELb1E", f) else 0), (f, other)
    # the FAST MC kernels drop the FCHK range checks and slow-path
    # branches of the path length, the log's s and both Henyey-Greenstein divisions
    for f in funcs:
        m = re.search(r"(mcml_(?:pdom|spec)ILb[01]ELb[01]E)Lb1E", f)
        if m:
            guarded = next(g for g in funcs if m.group(1) + "Lb0E" in g)
            assert ops(r"\bFCHK\b", guarded) - ops(r"\bFCHK\b", f) >= 3, f
