"""Thin ctypes binding of libsr (include/sr.h) -- argument marshalling only.

Every function named ``sr_*`` here calls the C entry point of the same name
and raises :class:`SRError` on a negative status.  Device memory, streams and
process groups come from PyTorch (plumbing); every step of the hot path runs
in libsr's CUDA kernels.  There is no CPU fallback: :func:`load` raises if
``libsr.so`` is missing, and ``sr_init`` fails with ``SR_E_CUDA`` without a GPU.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libsr.so")

SR_OK, SR_E_INVALID, SR_E_STATE, SR_E_NOMEM, SR_E_CUDA = 0, -1, -2, -3, -4
PDOM, SPEC_LOOP, SPEC_CALL = 0, 1, 2
WL_DIVLOOP, WL_COMMONCALL, WL_MCML, WL_PATHTRACE, WL_RSBENCH = 0, 1, 2, 3, 4
F_SCHED, F_STATIC, F_COARSE, F_NOSPLIT, F_MATGROUP, F_POOL = 1, 2, 4, 8, 16, 32
T_PERTHREAD, T_GRID, T_COUNTERS, T_SCHED, T_SCRATCH = 0, 1, 2, 3, 4
MAX_LAYERS = 8
N_COUNTERS = 16
SCHED_WORDS = 8
MC_COUNTERS = ["photons", "steps", "rd_exits", "tt_exits", "rr_kills", "rr_survive", "capped",
               "zero_w"]
EXPORTS = ["sr_init", "sr_workspace_bytes", "sr_workspace_region", "sr_run", "sr_tally",
           "sr_finalize", "sr_last_error", "sr_build_info", "sr_last_launch", "sr_math_eval",
           "sr_math_eval_p", "sr_pt_closest", "sr_scene_build", "sr_scene_build_host"]
PT_COUNTERS = ["paths", "rays", "node_visits", "tri_tests"]
FN_LOGF, FN_SIN2PI, FN_COS2PI, FN_EXPENSIVE_1000, FN_EXPENSIVE_2000 = 0, 1, 2, 3, 4
FNP_DIV_XP, FNP_DIV_PX, FNP_SQRT, FNP_HG_COST, FNP_HG_SINT, FNP_DIV2_XP, FNP_FRESNEL = 0, 1, 2, 3, 4, 5, 8


class SRError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"libsr status {code}: {msg}")
        self.code = code


class Layer(C.Structure):
    _fields_ = [("n", C.c_float), ("mua", C.c_float), ("mus", C.c_float), ("g", C.c_float),
                ("d", C.c_float)]


class DivloopParams(C.Structure):
    _fields_ = [("p_u32", C.c_uint32), ("fma_count", C.c_uint32), ("advance_unroll", C.c_uint32),
                ("prolog_batch", C.c_uint32), ("pool_split", C.c_uint32)]


class CommoncallParams(C.Structure):
    _fields_ = [("fma_count", C.c_uint32), ("split_u32", C.c_uint32)]


class MCMLParams(C.Structure):
    _fields_ = [("n_layers", C.c_uint32), ("layers", Layer * MAX_LAYERS), ("n_above", C.c_float),
                ("n_below", C.c_float), ("dr", C.c_float), ("dz", C.c_float), ("nr", C.c_uint32),
                ("nz", C.c_uint32), ("step_cap", C.c_uint32), ("defer_threshold", C.c_uint32),
                ("merge_unroll", C.c_uint32)]


class PathtraceParams(C.Structure):
    _fields_ = [("scene_dev", C.c_void_p), ("scene_bytes", C.c_uint64), ("width", C.c_uint32),
                ("height", C.c_uint32), ("max_depth", C.c_uint32), ("merge_unroll", C.c_uint32),
                ("pool_spp", C.c_uint32)]


class RsbenchParams(C.Structure):
    _fields_ = [("fma_count", C.c_uint32), ("prolog_fma", C.c_uint32),
                ("merge_unroll", C.c_uint32)]


class Workload(C.Structure):
    _fields_ = [("kind", C.c_int32), ("flags", C.c_uint32), ("task_offset", C.c_uint64),
                ("block_threads", C.c_uint32), ("grid_ctas", C.c_uint32),
                ("divloop", DivloopParams), ("commoncall", CommoncallParams),
                ("mcml", MCMLParams), ("pathtrace", PathtraceParams),
                ("rsbench", RsbenchParams)]


_lib = None


def load(path: str | None = None):
    """Load libsr.so (or $SR_LIB, an alternative in-tree build used for
    tuning experiments).  Raises FileNotFoundError if it was not built."""
    global _lib
    if _lib is not None:
        return _lib
    path = path or os.environ.get("SR_LIB") or LIB_PATH
    if not os.path.exists(path):
        raise FileNotFoundError(
            f"{path} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'`"
            " (there is no CPU fallback)")
    L = C.CDLL(path)
    vp, sz, u64, u32 = C.c_void_p, C.c_size_t, C.c_uint64, C.c_uint32
    W = C.POINTER(Workload)
    L.sr_init.argtypes = [C.c_int, vp, vp, sz]
    L.sr_workspace_bytes.argtypes = [W, u64]; L.sr_workspace_bytes.restype = sz
    L.sr_workspace_region.argtypes = [W, u64, C.c_int, C.POINTER(sz), C.POINTER(sz)]
    L.sr_run.argtypes = [W, u64, u32, u64, C.c_int, u32]
    L.sr_tally.argtypes = [C.c_int, vp, sz, C.POINTER(sz)]
    L.sr_finalize.argtypes = []
    L.sr_last_error.restype = C.c_char_p
    L.sr_build_info.restype = C.c_char_p
    L.sr_last_launch.argtypes = [C.POINTER(C.c_uint32)]
    L.sr_math_eval.argtypes = [C.c_int, vp, vp, u64]
    L.sr_math_eval.restype = C.c_int
    L.sr_math_eval_p.argtypes = [C.c_int, C.c_float, vp, vp, u64]
    L.sr_math_eval_p.restype = C.c_int
    L.sr_pt_closest.argtypes = [vp, vp, vp, vp, u64]
    L.sr_pt_closest.restype = C.c_int
    fp, up = C.POINTER(C.c_float), C.POINTER(C.c_uint32)
    L.sr_scene_build.argtypes = [fp, up, u32, fp, u32, fp, vp, sz, C.POINTER(sz)]
    L.sr_scene_build_host.argtypes = [fp, up, u32, fp, u32, fp, vp, sz, C.POINTER(sz)]
    for name in ("sr_init", "sr_workspace_region", "sr_run", "sr_tally", "sr_finalize",
                 "sr_last_launch", "sr_scene_build", "sr_scene_build_host"):
        getattr(L, name).restype = C.c_int
    _lib = L
    return L


def _check(rc: int) -> int:
    if rc < 0:
        raise SRError(rc, load().sr_last_error().decode())
    return rc


# ------------------------------------------------------------------ the C ABI, 1:1
def sr_init(device: int, stream: int | None, workspace_ptr: int, workspace_bytes: int) -> None:
    _check(load().sr_init(device, stream, workspace_ptr, workspace_bytes))


def sr_workspace_bytes(w: Workload, n_threads: int) -> int:
    return load().sr_workspace_bytes(C.byref(w), n_threads)


def sr_workspace_region(w: Workload, n_threads: int, what: int) -> tuple[int, int]:
    off, nb = C.c_size_t(), C.c_size_t()
    _check(load().sr_workspace_region(C.byref(w), n_threads, what, C.byref(off), C.byref(nb)))
    return off.value, nb.value


def sr_run(w: Workload, n_threads: int, iters: int, seed: int, mode: int, threshold: int) -> None:
    _check(load().sr_run(C.byref(w), n_threads, iters, seed & 0xFFFFFFFFFFFFFFFF, mode, threshold))


def sr_tally(what: int, dst_ptr: int, dst_bytes: int) -> int:
    written = C.c_size_t()
    _check(load().sr_tally(what, dst_ptr, dst_bytes, C.byref(written)))
    return written.value


def sr_finalize() -> None:
    _check(load().sr_finalize())


def sr_last_error() -> str:
    return load().sr_last_error().decode()


def sr_build_info() -> str:
    return load().sr_build_info().decode()


def sr_math_eval(fn: int, x_ptr: int, out_ptr: int, n: int) -> None:
    _check(load().sr_math_eval(fn, x_ptr, out_ptr, n))


def sr_math_eval_p(fn: int, p: float, x_ptr: int, out_ptr: int, n: int) -> None:
    _check(load().sr_math_eval_p(fn, p, x_ptr, out_ptr, n))


def sr_pt_closest(scene_ptr: int, rays_ptr: int, hit_ptr: int, t_ptr: int, n: int) -> None:
    _check(load().sr_pt_closest(scene_ptr, rays_ptr, hit_ptr, t_ptr, n))


def sr_last_launch() -> dict:
    out = (C.c_uint32 * 4)()
    _check(load().sr_last_launch(out))
    return {"grid": out[0], "block": out[1], "smem": out[2], "kernels": out[3]}


def sr_scene_build(tris, mat, mats, cam, dst_ptr: int | None, dst_bytes: int,
                   host: bool = False) -> int:
    """numpy float32 tris[n,9], uint32 mat[n], float32 mats[m,8], float32 cam[14];
    dst_ptr: device address (sr_scene_build) or, with host=True, a host address
    (sr_scene_build_host).  Returns the bytes needed / written."""
    import numpy as np
    tris = np.ascontiguousarray(tris, np.float32); mat = np.ascontiguousarray(mat, np.uint32)
    mats = np.ascontiguousarray(mats, np.float32); cam = np.ascontiguousarray(cam, np.float32)
    fp, up = C.POINTER(C.c_float), C.POINTER(C.c_uint32)
    needed = C.c_size_t()
    fn = load().sr_scene_build_host if host else load().sr_scene_build
    _check(fn(tris.ctypes.data_as(fp), mat.ctypes.data_as(up), len(mat), mats.ctypes.data_as(fp),
              len(mats), cam.ctypes.data_as(fp), dst_ptr, dst_bytes, C.byref(needed)))
    return needed.value


def scene_image_host(tris, mat, mats, cam):
    """The scene image built on the host (numpy uint8), for inspection."""
    import numpy as np
    need = sr_scene_build(tris, mat, mats, cam, None, 0, host=True)
    img = np.zeros(need, np.uint8)
    used = sr_scene_build(tris, mat, mats, cam, img.ctypes.data, need, host=True)
    return img[:used]


# ------------------------------------------------------------------ workload builders
def divloop_workload(p_u32=1 << 29, fma_count=1000, task_offset=0, flags=0, block=0,
                     advance=0, batch=0, split=0) -> Workload:
    w = Workload(kind=WL_DIVLOOP, flags=flags, task_offset=task_offset, block_threads=block)
    w.divloop = DivloopParams(p_u32, fma_count, advance, batch, split)
    return w


def rsbench_workload(fma_count=64, task_offset=0, flags=0, block=0, prolog_fma=0,
                     unroll=0) -> Workload:
    w = Workload(kind=WL_RSBENCH, flags=flags, task_offset=task_offset, block_threads=block)
    w.rsbench = RsbenchParams(fma_count, prolog_fma, unroll)
    return w


def commoncall_workload(fma_count=2000, split_u32=1 << 31, task_offset=0, flags=0,
                        block=0) -> Workload:
    w = Workload(kind=WL_COMMONCALL, flags=flags, task_offset=task_offset, block_threads=block)
    w.commoncall = CommoncallParams(fma_count, split_u32)
    return w


def mcml_workload(layers, n_above=1.0, n_below=1.0, dr=0.01, dz=0.002, nr=256, nz=255,
                  step_cap=100000, task_offset=0, flags=0, block=0, grid=0,
                  defer=0, unroll=0) -> Workload:
    w = Workload(kind=WL_MCML, flags=flags, task_offset=task_offset, block_threads=block,
                 grid_ctas=grid)
    m = MCMLParams()
    m.n_layers = len(layers)
    for i, (n_, mua, mus, g, d) in enumerate(layers):
        m.layers[i] = Layer(n_, mua, mus, g, d)
    m.n_above, m.n_below, m.dr, m.dz = n_above, n_below, dr, dz
    m.nr, m.nz, m.step_cap = nr, nz, step_cap
    m.defer_threshold = defer
    m.merge_unroll = unroll
    w.mcml = m
    return w


def upload_scene(tris, mat, mats, cam, device: int = 0):
    """Build the BVH scene image (sr_scene_build) into a torch-owned device
    buffer; returns (buffer, bytes)."""
    import torch
    need = sr_scene_build(tris, mat, mats, cam, None, 0)
    buf = torch.empty(need, dtype=torch.uint8, device=f"cuda:{device}")
    used = sr_scene_build(tris, mat, mats, cam, buf.data_ptr(), need)
    return buf, used


def pathtrace_workload(scene_ptr: int, scene_bytes: int, width: int, height: int, max_depth=8,
                       flags=0, block=0, unroll=0, pool_spp=0) -> Workload:
    """pool_spp: with F_POOL, the most samples per pixel a run may use"""
    w = Workload(kind=WL_PATHTRACE, flags=flags, block_threads=block)
    w.pathtrace = PathtraceParams(scene_ptr, scene_bytes, width, height, max_depth, unroll,
                                  pool_spp)
    return w


@dataclass
class Context:
    """A torch-owned workspace bound to libsr on the current CUDA stream."""
    device: int
    workspace: object   # torch.uint8 CUDA tensor
    stream: object

    @classmethod
    def create(cls, device: int, nbytes: int, stream=None):
        import torch
        torch.cuda.set_device(device)
        ws = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=f"cuda:{device}")
        st = stream if stream is not None else torch.cuda.current_stream(device)
        sr_init(device, st.cuda_stream, ws.data_ptr(), ws.numel())
        return cls(device, ws, st)

    def ensure(self, nbytes: int):
        if self.workspace.numel() < nbytes:
            import torch
            # kernels enqueued by libsr on self.stream may still use the old block;
            # the caching allocator could hand it out again once it is dropped
            self.stream.synchronize()
            self.workspace = torch.empty(nbytes, dtype=torch.uint8, device=f"cuda:{self.device}")
            sr_init(self.device, self.stream.cuda_stream, self.workspace.data_ptr(), nbytes)

    def region(self, w: Workload, n_threads: int, what: int, dtype):
        """A zero-copy torch view of one workspace region of the last layout."""
        off, nb = sr_workspace_region(w, n_threads, what)
        self.stream.synchronize()  # the library works on self.stream, not torch's current one
        return self.workspace[off:off + nb].view(dtype)
