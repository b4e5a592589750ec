"""GPU checks of the C ABI's own contract (include/sr.h), not of the arithmetic:

* the workspace regions bound every byte a run writes (sentinel bytes after
  sr_workspace_bytes stay intact), including schedule records with a CTA much
  larger than n_threads (partial last CTA);
* sr_run is stream-ordered and capturable: a PATHTRACE run captured in a CUDA
  graph replays bit-exactly (sr.h: "does not synchronize");
* a scene image copied in by the caller (not written by sr_scene_build) still
  runs, and is refused -- not read -- while the stream is capturing.
"""
import numpy as np
import pytest

from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import sr

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

SENTINEL = 0xA5


@pytest.fixture(scope="module")
def ctx():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    c = sr.Context.create(0, 1 << 20)
    yield c
    torch.cuda.synchronize()
    sr.sr_finalize()


def run_guarded(ctx, w, n, iters, mode, T, pad=1 << 16):
    """Run with a workspace of exactly sr_workspace_bytes + pad sentinel bytes."""
    need = sr.sr_workspace_bytes(w, n)
    ws = torch.full((need + pad,), SENTINEL, dtype=torch.uint8, device="cuda")
    sr.sr_init(ctx.device, ctx.stream.cuda_stream, ws.data_ptr(), need)
    try:
        sr.sr_run(w, n, iters, I.PRIMARY_SEED, mode, T)
        ctx.stream.synchronize()
    finally:
        sr.sr_init(ctx.device, ctx.stream.cuda_stream, ctx.workspace.data_ptr(),
                   ctx.workspace.numel())
    tail = ws[need:].cpu().numpy()
    return ws, need, tail


@pytest.mark.parametrize("kind", ["divloop", "rsbench", "commoncall", "mcml"])
@pytest.mark.parametrize("n", [1, 33, 1000])
@pytest.mark.parametrize("block", [1024, 96])
def test_sched_records_stay_inside_workspace(ctx, kind, n, block):
    m = I.C3
    if kind == "divloop":
        w = sr.divloop_workload(flags=sr.F_SCHED, block=block, advance=8)
        modes = ((sr.PDOM, 0), (sr.SPEC_LOOP, 16))
        iters = 8
    elif kind == "rsbench":
        w = sr.rsbench_workload(flags=sr.F_SCHED, block=min(block, 256), unroll=4)
        modes = ((sr.PDOM, 0), (sr.SPEC_LOOP, 24))
        iters = 3
    elif kind == "commoncall":
        w = sr.commoncall_workload(fma_count=64, flags=sr.F_SCHED, block=block)
        modes = ((sr.PDOM, 0), (sr.SPEC_CALL, 0))
        iters = 1
    else:
        if block > 640:
            block = 640   # the MC kernels' launch bound
        w = sr.mcml_workload(m.layers, flags=sr.F_SCHED, block=block)
        modes = ((sr.PDOM, 0), (sr.SPEC_LOOP, 32))
        iters = 2
    for mode, T in modes:
        _, _, tail = run_guarded(ctx, w, n, iters, mode, T)
        assert (tail == SENTINEL).all(), (kind, n, block, mode, np.nonzero(tail != SENTINEL)[0][:4])


def test_sched_region_covers_launched_warps(ctx):
    """One record per launched warp: ceil(n / block) CTAs of block/32 warps."""
    for block, n in ((1024, 1), (96, 100), (64, 1000)):
        w = sr.divloop_workload(flags=sr.F_SCHED, block=block)
        assert sr.sr_workspace_region(w, n, sr.T_SCHED)[1] == \
            -(-n // block) * (block // 32) * sr.SCHED_WORDS * 4


def _pt_workload(cfg, buf, used, flags=0):
    return sr.pathtrace_workload(buf.data_ptr(), used, cfg.width, cfg.height, cfg.max_depth,
                                 flags=flags)


@pytest.mark.parametrize("mode,T,flags", [(sr.PDOM, 0, 0), (sr.SPEC_LOOP, 12, 0),
                                          (sr.SPEC_LOOP, 16, sr.F_COARSE)])
def test_pathtrace_run_captures_in_cuda_graph(ctx, mode, T, flags):
    cfg = I.C4_SMALL
    tris, mat, mats, cam = I.cornell_scene(cfg)
    buf, used = sr.upload_scene(tris, mat, mats, cam)
    w = _pt_workload(cfg, buf, used, flags)
    n = cfg.width * cfg.height
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, cfg.spp, I.PRIMARY_SEED, mode, T)
    ref = ctx.region(w, n, sr.T_PERTHREAD, torch.float32).clone()
    ref_cnt = ctx.region(w, n, sr.T_COUNTERS, torch.int64).clone()
    ctx.workspace.zero_()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    cap = torch.cuda.Stream()
    sr.sr_init(ctx.device, cap.cuda_stream, ctx.workspace.data_ptr(), ctx.workspace.numel())
    try:
        with torch.cuda.graph(g, stream=cap):
            sr.sr_run(w, n, cfg.spp, I.PRIMARY_SEED, mode, T)
        for _ in range(2):
            ctx.workspace.zero_()
            g.replay()
            torch.cuda.synchronize()
            off, nb = sr.sr_workspace_region(w, n, sr.T_PERTHREAD)
            got = ctx.workspace[off:off + nb].view(torch.float32)
            assert torch.equal(got.view(torch.int32), ref.view(torch.int32))
            off, nb = sr.sr_workspace_region(w, n, sr.T_COUNTERS)
            assert torch.equal(ctx.workspace[off:off + nb].view(torch.int64), ref_cnt)
    finally:
        sr.sr_init(ctx.device, ctx.stream.cuda_stream, ctx.workspace.data_ptr(),
                   ctx.workspace.numel())


def test_pathtrace_caller_copied_scene(ctx):
    """An image built on the host and copied by the caller: runs (header read once), gives the
    same pixels as the registered image, and is refused during stream capture."""
    cfg = I.C4_SMALL
    tris, mat, mats, cam = I.cornell_scene(cfg)
    buf, used = sr.upload_scene(tris, mat, mats, cam)
    n = cfg.width * cfg.height
    w = _pt_workload(cfg, buf, used)
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, cfg.spp, I.PRIMARY_SEED, sr.SPEC_LOOP, 12)
    ref = ctx.region(w, n, sr.T_PERTHREAD, torch.float32).clone()
    img = torch.from_numpy(sr.scene_image_host(tris, mat, mats, cam))
    dev = img.cuda()
    w2 = sr.pathtrace_workload(dev.data_ptr(), dev.numel(), cfg.width, cfg.height, cfg.max_depth)
    g = torch.cuda.CUDAGraph()
    cap = torch.cuda.Stream()
    sr.sr_init(ctx.device, cap.cuda_stream, ctx.workspace.data_ptr(), ctx.workspace.numel())
    try:
        with pytest.raises(sr.SRError):
            with torch.cuda.graph(g, stream=cap):
                sr.sr_run(w2, n, cfg.spp, I.PRIMARY_SEED, sr.SPEC_LOOP, 12)
    except RuntimeError:
        pass   # the aborted capture may also surface as a torch error; either way it refused
    finally:
        torch.cuda.synchronize()
        sr.sr_init(ctx.device, ctx.stream.cuda_stream, ctx.workspace.data_ptr(),
                   ctx.workspace.numel())
    sr.sr_run(w2, n, cfg.spp, I.PRIMARY_SEED, sr.SPEC_LOOP, 12)
    got = ctx.region(w2, n, sr.T_PERTHREAD, torch.float32)
    assert torch.equal(got.view(torch.int32), ref.view(torch.int32))
