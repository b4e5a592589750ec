"""CPU oracle for the Speculative Reconvergence hot path -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_cgo_damanijskymg20_b200``) never imports it, and this package
never imports the product path.  See ``oracle/oracle.h`` for what each
function computes and which paper passage it follows.

This module is argument marshalling only (ctypes + numpy); every number is
computed by the plain C in ``oracle/*.c``.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "liboracle.so")
SOURCES = ["philox.c", "srmath.c", "divloop.c", "commoncall.c", "mcml.c", "warpsim.c",
           "pathtrace.c", "rsbench.c", "pttrace.c"]
CFLAGS = ["-O2", "-std=gnu11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
          "-Wall", "-Wno-unused-function"]

TAG_DIV, TAG_CALL, TAG_MC, TAG_PT = 1, 2, 3, 4
PDOM, SPEC_LOOP, SPEC_CALL, SPEC_LOOP_POOL = 0, 1, 2, 3
# region ids (oracle.h)
DL = dict(ENTRY=0, PROLOG=1, EXPENSIVE=2, EPILOG=3, ROUND=4, RELEASE=5, ADVANCE=6)
CC = dict(ENTRY=0, THEN=1, ELSE_PRE=2, CALL=3, ELSE_POST=4, MERGE=5)
PT = {k: i for i, k in enumerate(
    "ENTRY OUTER LAUNCH BOUNCE TBEGIN STEP NODE PUSH NOPUSH NEXTNONE POP LEAFIF LEAF TT TT_U "
    "TT_V TT_T TT_ID TT_UPD SH SH_HIT SH_SURF SH_DIFF SH_MIRR SH_GLASS SH_RR SH_END ROUND REL "
    "LREL NREL ADV PSUM".split())}
LM = dict(ENTRY=0, LAUNCH=1, STEP=2, STEP_BOUNDARY=3, STEP_INTERACT=4, ROUND=5, RELEASE=6,
          ADVANCE=7, **{f"EV{b}": 8 + b for b in range(16)}, **{f"NEV{b}": 24 + b for b in range(16)},
          A_RR=40, B_RR=41, B_REL=42, BI=43, A_TAIL=44, CLAIM=45, CLAIMIT=46, CHUNK=47)
# MC step event bits (oracle.h OR_EV_*)
EV_BOUNDARY, EV_SLEFT, EV_REFLECT, EV_EXIT, EV_TRANSMIT, EV_ROULETTE, EV_SPIN_AXIS, \
    EV_SPIN_GENERAL, EV_EXTERNAL, EV_MATCHED = 1, 2, 4, 8, 16, 32, 64, 128, 256, 512
MC_COUNTERS = ["photons", "steps", "rd_exits", "tt_exits", "rr_kills", "rr_survive", "capped",
               "zero_w"]
MAX_LAYERS = 8


def build(force: bool = False) -> str:
    srcs = [os.path.join(HERE, s) for s in SOURCES if os.path.exists(os.path.join(HERE, s))]
    newest = max(os.path.getmtime(s) for s in srcs + [os.path.join(HERE, "oracle.h")])
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < newest:
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, *srcs, "-lm"])
        os.replace(tmp, LIB)
    return LIB


class _Layer(C.Structure):
    _fields_ = [("n", C.c_float), ("mua", C.c_float), ("mus", C.c_float), ("g", C.c_float),
                ("d", C.c_float)]


class MCParams(C.Structure):
    _fields_ = [("n_layers", C.c_uint32), ("layer", _Layer * MAX_LAYERS), ("n_above", C.c_float),
                ("n_below", C.c_float), ("dr", C.c_float), ("dz", C.c_float), ("nr", C.c_uint32),
                ("nz", C.c_uint32), ("step_cap", C.c_uint32)]


class WsCounts(C.Structure):
    _fields_ = [("rounds", C.c_uint64), ("execs", C.c_uint64 * 48), ("lanes", C.c_uint64 * 48)]

    def as_dict(self, names):
        return {"rounds": int(self.rounds),
                **{k: (int(self.execs[v]), int(self.lanes[v])) for k, v in names.items()}}


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        L = _lib
        u32p, u64p, f32p, u8p = (C.POINTER(C.c_uint32), C.POINTER(C.c_uint64),
                                 C.POINTER(C.c_float), C.POINTER(C.c_uint8))
        L.or_philox4x32_10.argtypes = [u32p, u32p, u32p]
        L.or_u01.argtypes = [C.c_uint32]; L.or_u01.restype = C.c_float
        L.or_u01c.argtypes = [C.c_uint32]; L.or_u01c.restype = C.c_float
        L.or_sr_logf.argtypes = [C.c_float]; L.or_sr_logf.restype = C.c_float
        L.or_sr_sincos2pif.argtypes = [C.c_float, f32p, f32p]
        L.or_sweep_logf_ulp.restype = C.c_double
        L.or_sweep_sincos2pif_ulp.restype = C.c_double
        L.or_expensive.argtypes = [C.c_float, C.c_uint32]; L.or_expensive.restype = C.c_float
        L.or_divloop.argtypes = [u32p, C.c_uint64, C.c_uint64, C.c_uint32, C.c_uint64, f32p, u32p]
        L.or_divloop_wants.argtypes = [u32p, C.c_uint64, C.c_uint64, C.c_uint32, C.c_uint64, u8p]
        L.or_commoncall.argtypes = [u32p, C.c_uint64, C.c_uint64, C.c_uint32, C.c_uint64, f32p,
                                    u8p]
        L.or_mcml.argtypes = [C.POINTER(MCParams), C.c_uint64, C.c_uint64, C.c_uint64, u64p, u64p,
                              u64p, u64p, u32p]
        L.or_mcml_events.argtypes = [C.POINTER(MCParams), C.c_uint64, C.c_uint64, C.POINTER(C.c_uint16), C.c_uint32]
        L.or_mcml_events.restype = C.c_uint32
        L.or_mcml_rsp.argtypes = [C.POINTER(MCParams)]; L.or_mcml_rsp.restype = C.c_float
        L.ws_divloop.argtypes = [u8p, C.c_uint32, C.c_uint32, C.c_uint32, C.c_int, C.c_uint32,
                                 C.POINTER(WsCounts)]
        L.ws_divloop_adv.argtypes = [u8p, C.c_uint32, C.c_uint32, C.c_uint32, C.c_int,
                                     C.c_uint32, C.c_uint32, C.POINTER(WsCounts)]
        L.ws_commoncall.argtypes = [u8p, C.c_uint32, C.c_uint32, C.c_int, C.POINTER(WsCounts)]
        L.ws_loopmerge.argtypes = [u32p, C.POINTER(C.c_uint16), u64p, C.c_uint32, C.c_uint32, C.c_uint32, C.c_int,
                                   C.c_uint32, C.POINTER(WsCounts)]
        L.ws_divloop_optimum.argtypes = [u8p, C.c_uint32, C.c_uint32]
        L.ws_divloop_optimum.restype = C.c_uint32
        if hasattr(L, "or_pt_render"):
            _bind_pt(L)
    return _lib


def _p(a, ct):
    return a.ctypes.data_as(C.POINTER(ct))


# ---------------------------------------------------------------- RNG / math
def philox(ctr, key):
    c = np.asarray(ctr, dtype=np.uint32); k = np.asarray(key, dtype=np.uint32)
    out = np.zeros(4, np.uint32)
    lib().or_philox4x32_10(_p(c, C.c_uint32), _p(k, C.c_uint32), _p(out, C.c_uint32))
    return out


def eval_batch(fn: int, x):
    x = np.ascontiguousarray(x, np.float32)
    out = np.empty_like(x)
    L = lib()
    L.or_eval_batch.argtypes = [C.c_int, C.POINTER(C.c_float), C.POINTER(C.c_float), C.c_uint64]
    L.or_eval_batch(fn, _p(x, C.c_float), _p(out, C.c_float), x.size)
    return out


def sr_logf(x: float) -> float:
    return lib().or_sr_logf(x)


def sr_sincos2pif(x: float):
    s, c = C.c_float(), C.c_float()
    lib().or_sr_sincos2pif(x, C.byref(s), C.byref(c))
    return s.value, c.value


# ---------------------------------------------------------------- config 1
def divloop(t0, n, iters, seed, p_u32=1 << 29, fma_count=1000):
    prm = np.array([p_u32, fma_count], np.uint32)
    acc = np.zeros(n, np.float32); cnt = np.zeros(n, np.uint32)
    lib().or_divloop(_p(prm, C.c_uint32), t0, n, iters, seed, _p(acc, C.c_float),
                     _p(cnt, C.c_uint32))
    return acc, cnt


def divloop_wants(t0, n, iters, seed, p_u32=1 << 29, fma_count=1000):
    prm = np.array([p_u32, fma_count], np.uint32)
    w = np.zeros(n * iters, np.uint8)
    lib().or_divloop_wants(_p(prm, C.c_uint32), t0, n, iters, seed, _p(w, C.c_uint8))
    return w.reshape(n, iters)


# ---------------------------------------------------------------- config 2
def commoncall(t0, n, iters, seed, split_u32=1 << 31, fma_count=2000):
    prm = np.array([fma_count, split_u32], np.uint32)
    y = np.zeros(n, np.float32); arm = np.zeros(n, np.uint8)
    lib().or_commoncall(_p(prm, C.c_uint32), t0, n, iters, seed, _p(y, C.c_float),
                        _p(arm, C.c_uint8))
    return y, arm


# ---------------------------------------------------------------- NEXT-1 (RSBench shape)
RS_MATS, RS_NUCLIDES = 12, 355


def rsbench(t0, n, iters, seed, fma_count=64, trips=False, prolog_fma=0):
    L = lib()
    u32p, f32p = C.POINTER(C.c_uint32), C.POINTER(C.c_float)
    L.or_rsbench.argtypes = [C.c_uint32, C.c_uint32, C.c_uint64, C.c_uint64, C.c_uint32,
                             C.c_uint64, f32p, u32p, u32p]
    acc = np.zeros(n, np.float32); nuc = np.zeros(n, np.uint32)
    tr = np.zeros(n * iters, np.uint32) if trips else None
    L.or_rsbench(fma_count, prolog_fma, t0, n, iters, seed, _p(acc, C.c_float),
                 _p(nuc, C.c_uint32), _p(tr, C.c_uint32) if trips else None)
    return (acc, nuc, tr.reshape(n, iters)) if trips else (acc, nuc)


def rs_table():
    L = lib()
    L.or_rs_nuclides.restype = C.c_uint32; L.or_rs_nuclides.argtypes = [C.c_uint32]
    L.or_rs_threshold.restype = C.c_uint32; L.or_rs_threshold.argtypes = [C.c_uint32]
    L.or_rs_pick.restype = C.c_uint32; L.or_rs_pick.argtypes = [C.c_uint32]
    return ([L.or_rs_nuclides(m) for m in range(RS_MATS)],
            [L.or_rs_threshold(m) for m in range(RS_MATS)], L.or_rs_pick)


# ---------------------------------------------------------------- configs 3/5
def mc_params(layers, n_above=1.0, n_below=1.0, dr=0.01, dz=0.002, nr=256, nz=255,
              step_cap=100000) -> MCParams:
    p = MCParams()
    p.n_layers = len(layers)
    for i, (n_, mua, mus, g, d) in enumerate(layers):
        p.layer[i] = _Layer(n_, mua, mus, g, d)
    p.n_above, p.n_below, p.dr, p.dz = n_above, n_below, dr, dz
    p.nr, p.nz, p.step_cap = nr, nz, step_cap
    return p


def mcml(p: MCParams, id0, count, seed, steps=False):
    A = np.zeros(p.nz * p.nr, np.uint64); Rd = np.zeros(p.nr, np.uint64)
    Tt = np.zeros(p.nr, np.uint64); cnt = np.zeros(8, np.uint64)
    st = np.zeros(count, np.uint32) if steps else None
    lib().or_mcml(C.byref(p), id0, count, seed, _p(A, C.c_uint64), _p(Rd, C.c_uint64),
                  _p(Tt, C.c_uint64), _p(cnt, C.c_uint64),
                  _p(st, C.c_uint32) if steps else None)
    out = dict(A=A.reshape(p.nz, p.nr), Rd=Rd, Tt=Tt, counters=dict(zip(MC_COUNTERS, map(int, cnt))),
               counters_raw=cnt)
    if steps:
        out["steps"] = st
    return out


def mcml_events(p: MCParams, pid, seed, cap=1 << 20):
    ev = np.zeros(cap, np.uint16)
    n = lib().or_mcml_events(C.byref(p), pid, seed, _p(ev, C.c_uint16), cap)
    return ev[:n].copy()


def mcml_events_batch(p: MCParams, id0, count, seed, cap=None):
    """(ev uint16[total], off uint64[count], nsteps uint32[count])"""
    L = lib()
    L.or_mcml_events_batch.argtypes = [C.POINTER(MCParams), C.c_uint64, C.c_uint64, C.c_uint64,
                                       C.POINTER(C.c_uint16), C.c_uint64,
                                       C.POINTER(C.c_uint64), C.POINTER(C.c_uint32)]
    L.or_mcml_events_batch.restype = C.c_uint64
    cap = cap or count * 2000
    ev = np.zeros(cap, np.uint16)
    off = np.zeros(count, np.uint64)
    ns = np.zeros(count, np.uint32)
    used = L.or_mcml_events_batch(C.byref(p), id0, count, seed, _p(ev, C.c_uint16), cap,
                                  _p(off, C.c_uint64), _p(ns, C.c_uint32))
    if used == 2**64 - 1:
        return mcml_events_batch(p, id0, count, seed, cap * 4)
    return ev[:used], off, ns


def mcml_rsp(p: MCParams) -> float:
    return lib().or_mcml_rsp(C.byref(p))


# ---------------------------------------------------------------- simulator
def ws_divloop(want, mode, T, W=32, n_valid=None, V=1):
    """V = iterations a run-ahead lane may take per advance round (1: reading Q5)."""
    want = np.ascontiguousarray(want, np.uint8)
    n_valid = want.shape[0] if n_valid is None else n_valid
    o = WsCounts()
    lib().ws_divloop_adv(_p(want, C.c_uint8), W, n_valid, want.shape[1], mode, T, V,
                         C.byref(o))
    return o.as_dict(DL)


def ws_commoncall(arm, mode, W=32):
    arm = np.ascontiguousarray(arm, np.uint8)
    o = WsCounts()
    lib().ws_commoncall(_p(arm, C.c_uint8), W, arm.shape[0], mode, C.byref(o))
    return o.as_dict(CC)


def ws_loopmerge(nsteps, mode, T, W=32, events=None, U=1):
    """nsteps: [n_valid, K] uint32; events: optional list-of-lists of uint16 arrays;
    U = inner iterations per release (events=None only)."""
    nsteps = np.ascontiguousarray(nsteps, np.uint32)
    n_valid, K = nsteps.shape
    o = WsCounts()
    if U != 1:
        assert events is None
        return ws_loopmerge_raw(nsteps, None, None, mode, T, W, U)
    if events is not None:
        flat = [events[l][k] for l in range(n_valid) for k in range(K)]
        off = np.zeros(len(flat), np.uint64)
        np.cumsum([len(e) for e in flat[:-1]], out=off[1:]) if len(flat) > 1 else None
        ev = np.ascontiguousarray(np.concatenate(flat) if flat else np.zeros(1), np.uint16)
        lib().ws_loopmerge(_p(nsteps, C.c_uint32), _p(ev, C.c_uint16), _p(off, C.c_uint64), W,
                           n_valid, K, mode, T, C.byref(o))
    else:
        lib().ws_loopmerge(_p(nsteps, C.c_uint32), None, None, W, n_valid, K, mode, T, C.byref(o))
    return o.as_dict(LM)


def ws_loopmerge_raw(nsteps, ev_flat, ev_off, mode, T, W=32, U=1):
    """nsteps [n_valid, K]; ev_off [n_valid*K] offsets into the flat event buffer;
    U = steps per release (partial unroll of the merged loop)."""
    nsteps = np.ascontiguousarray(nsteps, np.uint32)
    if ev_off is not None:
        ev_off = np.ascontiguousarray(ev_off, np.uint64)
    n_valid, K = nsteps.shape
    o = WsCounts()
    L = lib()
    L.ws_loopmerge_unrolled.argtypes = [C.POINTER(C.c_uint32), C.POINTER(C.c_uint16),
                                        C.POINTER(C.c_uint64), C.c_uint32, C.c_uint32,
                                        C.c_uint32, C.c_int, C.c_uint32, C.c_uint32,
                                        C.POINTER(WsCounts)]
    L.ws_loopmerge_unrolled(_p(nsteps, C.c_uint32),
                            None if ev_flat is None else _p(ev_flat, C.c_uint16),
                            None if ev_off is None else _p(ev_off, C.c_uint64),
                            W, n_valid, K, mode, T, U, C.byref(o))
    return o.as_dict(LM)


def pt_trace(img, width, height, spp, max_depth, seed, pixels=None, cap=None):
    """(ops uint16, off uint64[n+1], rgb float32[n, 3]) -- see oracle.h or_pt_trace.
    img: the scene image (uint8 numpy array, sr_scene_build_host)."""
    img = np.ascontiguousarray(img, np.uint8)
    n = width * height if pixels is None else len(pixels)
    pix = None if pixels is None else np.ascontiguousarray(pixels, np.uint32)
    cap = cap or n * spp * 400
    L = lib()
    L.or_pt_trace.argtypes = [C.POINTER(C.c_uint8), C.c_uint64, C.c_uint32, C.c_uint32,
                              C.c_uint32, C.c_uint32, C.c_uint64, C.POINTER(C.c_uint32),
                              C.c_uint32, C.POINTER(C.c_uint16), C.c_uint64,
                              C.POINTER(C.c_uint64), C.POINTER(C.c_float)]
    L.or_pt_trace.restype = C.c_uint64
    ops = np.zeros(cap, np.uint16)
    off = np.zeros(n + 1, np.uint64)
    rgb = np.zeros((n, 3), np.float32)
    used = L.or_pt_trace(_p(img, C.c_uint8), img.size, width, height, spp, max_depth, seed,
                         None if pix is None else _p(pix, C.c_uint32), n, _p(ops, C.c_uint16),
                         cap, _p(off, C.c_uint64), _p(rgb, C.c_float))
    if used == 2**64 - 2:
        raise ValueError("not a scene image")
    if used == 2**64 - 1:
        return pt_trace(img, width, height, spp, max_depth, seed, pixels, cap * 4)
    return ops[:used], off, rgb


def ws_pt(ops, off, mode, T=0, U=1):
    """one warp's PDOM / split Loop Merge schedule (off: n_valid + 1 offsets);
    mode SPEC_LOOP_POOL: the split merge with the warp's paths pooled"""
    ops = np.ascontiguousarray(ops, np.uint16)
    off = np.ascontiguousarray(off, np.uint64)
    o = WsCounts()
    L = lib()
    L.ws_pt.argtypes = [C.POINTER(C.c_uint16), C.POINTER(C.c_uint64), C.c_uint32, C.c_int,
                        C.c_uint32, C.c_uint32, C.POINTER(WsCounts)]
    L.ws_pt(_p(ops, C.c_uint16), _p(off, C.c_uint64), len(off) - 1, mode, T, U, C.byref(o))
    return o.as_dict(PT)


def ws_loopmerge_stream(nsteps, mode, T, U=1, W=32, ev=None, ev_off=None):
    """Loop Merge / PDOM with dynamic claiming from one task stream (the MC
    kernels' default task source): nsteps [Q] uint32, optional events."""
    nsteps = np.ascontiguousarray(nsteps, np.uint32)
    o = WsCounts()
    L = lib()
    L.ws_loopmerge_stream.argtypes = [C.POINTER(C.c_uint32), C.POINTER(C.c_uint16),
                                      C.POINTER(C.c_uint64), C.c_uint32, C.c_uint64, C.c_int,
                                      C.c_uint32, C.c_uint32, C.POINTER(WsCounts)]
    if ev_off is not None:
        ev_off = np.ascontiguousarray(ev_off, np.uint64)
    L.ws_loopmerge_stream(_p(nsteps, C.c_uint32), None if ev is None else _p(ev, C.c_uint16),
                          None if ev_off is None else _p(ev_off, C.c_uint64), W,
                          nsteps.shape[0], mode, T, U, C.byref(o))
    return o.as_dict(LM)


def ws_loopmerge_pool(nsteps, T, U=1, W=32):
    """Loop Merge over the warp's task pool: nsteps [n_valid, K] uint32 (task k of
    thread l); task q = k * n_valid + l is claimed by idle lanes in lane order."""
    nsteps = np.ascontiguousarray(nsteps, np.uint32)
    n_valid, K = nsteps.shape
    o = WsCounts()
    L = lib()
    L.ws_loopmerge_pool.argtypes = [C.POINTER(C.c_uint32), C.c_uint32, C.c_uint32, C.c_uint32,
                                    C.c_uint32, C.c_uint32, C.POINTER(WsCounts)]
    L.ws_loopmerge_pool(_p(nsteps, C.c_uint32), W, n_valid, K, T, U, C.byref(o))
    return o.as_dict(LM)


def ws_loopmerge_defer_raw(nsteps, ev_flat, ev_off, T, Tb, W=32):
    """Loop Merge + nested Iteration Delay of the boundary sub-step."""
    nsteps = np.ascontiguousarray(nsteps, np.uint32)
    if ev_off is not None:
        ev_off = np.ascontiguousarray(ev_off, np.uint64)
    n_valid, K = nsteps.shape
    o = WsCounts()
    L = lib()
    L.ws_loopmerge_defer.argtypes = [C.POINTER(C.c_uint32), C.POINTER(C.c_uint16),
                                     C.POINTER(C.c_uint64), C.c_uint32, C.c_uint32, C.c_uint32,
                                     C.c_uint32, C.c_uint32, C.POINTER(WsCounts)]
    L.ws_loopmerge_defer(_p(nsteps, C.c_uint32), _p(ev_flat, C.c_uint16), _p(ev_off, C.c_uint64),
                         W, n_valid, K, T, Tb, C.byref(o))
    return o.as_dict(LM)


def ws_divloop_optimum(want):
    want = np.ascontiguousarray(want, np.uint8)
    return lib().ws_divloop_optimum(_p(want, C.c_uint8), want.shape[0], want.shape[1])


class PTScene(C.Structure):
    _fields_ = [("tris", C.POINTER(C.c_float)), ("mat", C.POINTER(C.c_uint32)),
                ("n_tris", C.c_uint32), ("mats", C.POINTER(C.c_float)), ("n_mats", C.c_uint32),
                ("cam", C.c_float * 16)]


def _bind_pt(L):
    fp = C.POINTER(C.c_float)
    L.or_pt_closest.argtypes = [fp, C.c_uint32, fp, fp, fp]
    L.or_pt_closest.restype = C.c_int64
    L.or_pt_render.argtypes = [C.POINTER(PTScene), C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32,
                               C.c_uint64, C.POINTER(C.c_uint32), C.c_uint32, fp,
                               C.POINTER(C.c_uint64)]


def pt_scene(tris, mat, mats, cam):
    """Keeps the numpy arrays alive alongside the ctypes view."""
    tris = np.ascontiguousarray(tris, np.float32); mat = np.ascontiguousarray(mat, np.uint32)
    mats = np.ascontiguousarray(mats, np.float32)
    s = PTScene(_p(tris, C.c_float), _p(mat, C.c_uint32), len(mat), _p(mats, C.c_float), len(mats))
    for i, v in enumerate(np.asarray(cam, np.float32)[:16]):
        s.cam[i] = v
    s._keep = (tris, mat, mats)
    return s


def pt_render(scene, width, height, spp, max_depth, seed, pixels=None):
    lib()
    n = width * height if pixels is None else len(pixels)
    rgb = np.zeros(3 * n, np.float32)
    cnt = np.zeros(2, np.uint64)
    pix = None if pixels is None else np.ascontiguousarray(pixels, np.uint32)
    lib().or_pt_render(C.byref(scene), width, height, spp, max_depth, seed,
                       None if pix is None else _p(pix, C.c_uint32), n, _p(rgb, C.c_float),
                       _p(cnt, C.c_uint64))
    return rgb.reshape(n, 3), dict(paths=int(cnt[0]), rays=int(cnt[1]))


def pt_closest(scene, o, d):
    o = np.ascontiguousarray(o, np.float32); d = np.ascontiguousarray(d, np.float32)
    t = C.c_float()
    i = lib().or_pt_closest(scene.tris, scene.n_tris, _p(o, C.c_float), _p(d, C.c_float),
                            C.byref(t))
    return int(i), t.value


# ---------------------------------------------------------------- step building blocks (pins)
def mcml_step_length(mut, u0):
    """or_mcml_step_length over an array of Philox words u0."""
    u = np.ascontiguousarray(u0, np.uint32)
    out = np.empty(u.size, np.float32)
    L = lib()
    L.or_mcml_eval_batch.argtypes = [C.c_int, C.c_float, C.POINTER(C.c_uint32),
                                     C.POINTER(C.c_float), C.c_uint64]
    L.or_mcml_eval_batch(0, mut, _p(u, C.c_uint32), _p(out, C.c_float), u.size)
    return out


def mcml_hg_cost(g, u1):
    """or_mcml_hg_cost(g, U01(u1)) over an array of Philox words u1."""
    u = np.ascontiguousarray(u1, np.uint32)
    out = np.empty(u.size, np.float32)
    L = lib()
    L.or_mcml_eval_batch.argtypes = [C.c_int, C.c_float, C.POINTER(C.c_uint32),
                                     C.POINTER(C.c_float), C.c_uint64]
    L.or_mcml_eval_batch(1, g, _p(u, C.c_uint32), _p(out, C.c_float), u.size)
    return out


def mcml_spin(cost, xi_psi, u):
    L = lib()
    fp = C.POINTER(C.c_float)
    L.or_mcml_spin.argtypes = [C.c_float, C.c_float, fp, fp]
    ui = np.ascontiguousarray(u, np.float32)
    uo = np.zeros(3, np.float32)
    L.or_mcml_spin(cost, xi_psi, _p(ui, C.c_float), _p(uo, C.c_float))
    return uo


def pt_scatter(kind, ior, d, ng, u):
    """or_pt_scatter: the direction half of one path-tracer bounce."""
    L = lib()
    fp = C.POINTER(C.c_float)
    L.or_pt_scatter.argtypes = [C.c_uint32, C.c_float, fp, fp, C.POINTER(C.c_uint32), fp]
    di = np.ascontiguousarray(d, np.float32); ni = np.ascontiguousarray(ng, np.float32)
    uu = np.ascontiguousarray(u, np.uint32)
    do = np.zeros(3, np.float32)
    L.or_pt_scatter(kind, ior, _p(di, C.c_float), _p(ni, C.c_float), _p(uu, C.c_uint32),
                    _p(do, C.c_float))
    return do
