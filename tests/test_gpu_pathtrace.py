"""GPU parity of config 4 (path tracer) through the C ABI vs the oracle.

BVH closest hit == brute force (exact index and t bits), rendered pixels
bit-exact in every mode/threshold, and at the full 1M-triangle 1024^2 x 16
spp configuration: PDOM == SPEC bit for bit plus sampled pixels vs the oracle.
"""
import numpy as np
import pytest

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import sr

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    c = sr.Context.create(0, 1 << 24)
    yield c
    torch.cuda.synchronize()
    sr.sr_finalize()


_scenes = {}


def scene(cfg):
    key = (cfg.subdiv, cfg.n_spheres, cfg.scene_seed, cfg.fov_deg, cfg.width, cfg.height)
    if key not in _scenes:
        tris, mat, mats, cam = I.cornell_scene(cfg)
        buf, used = sr.upload_scene(tris, mat, mats, cam)
        _scenes[key] = (tris, mat, mats, cam, buf, used)
    return _scenes[key]


def random_rays(n, seed):
    rng = np.random.default_rng(seed)
    o = rng.uniform(0.03, 0.97, (n, 3))
    d = rng.normal(size=(n, 3))
    d /= np.linalg.norm(d, axis=1, keepdims=True)
    return np.concatenate([o, d], 1).astype(np.float32)


@pytest.mark.parametrize("cfg,n", [(I.C4_SMALL, 20000), (I.C4, 1500)])
def test_bvh_closest_hit_equals_brute_force(ctx, cfg, n):
    tris, mat, mats, cam, buf, used = scene(cfg)
    rays = random_rays(n, 11)
    rd = torch.from_numpy(rays).cuda()
    hit = torch.empty(n, dtype=torch.int64, device="cuda")
    t = torch.empty(n, dtype=torch.float32, device="cuda")
    sr.sr_pt_closest(buf.data_ptr(), rd.data_ptr(), hit.data_ptr(), t.data_ptr(), n)
    ctx.stream.synchronize()
    hit, t = hit.cpu().numpy(), t.cpu().numpy()
    sc = oracle.pt_scene(tris, mat, mats, cam)
    for i in range(n):
        j, tj = oracle.pt_closest(sc, rays[i, :3], rays[i, 3:])
        assert hit[i] == j and np.float32(t[i]).view(np.uint32) == np.float32(tj).view(np.uint32), i


def render(ctx, cfg, mode, T, flags=0, block=0, pool_spp=None):
    tris, mat, mats, cam, buf, used = scene(cfg)
    n = cfg.width * cfg.height
    if pool_spp is None:
        pool_spp = cfg.spp if flags & sr.F_POOL else 0
    w = sr.pathtrace_workload(buf.data_ptr(), used, cfg.width, cfg.height, cfg.max_depth,
                              flags=flags, block=block, pool_spp=pool_spp)
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, cfg.spp, I.PRIMARY_SEED, mode, T)
    rgb = ctx.region(w, n, sr.T_PERTHREAD, torch.float32).view(-1, 3).cpu().numpy().copy()
    cnt = ctx.region(w, n, sr.T_COUNTERS, torch.int64).cpu().numpy()[:4].copy()
    return rgb, cnt


@pytest.mark.parametrize("mode,T", [(sr.PDOM, 0), (sr.SPEC_LOOP, 1), (sr.SPEC_LOOP, 8),
                                    (sr.SPEC_LOOP, 32)])
@pytest.mark.parametrize("block", [32, 128])
@pytest.mark.parametrize("flags", [0, sr.F_COARSE, sr.F_NOSPLIT, sr.F_MATGROUP, sr.F_POOL])
def test_render_bit_exact_small(ctx, mode, T, block, flags):
    cfg = I.C4_SMALL
    tris, mat, mats, cam, buf, used = scene(cfg)
    ref, rc = oracle.pt_render(oracle.pt_scene(tris, mat, mats, cam), cfg.width, cfg.height,
                               cfg.spp, cfg.max_depth, I.PRIMARY_SEED)
    rgb, cnt = render(ctx, cfg, mode, T, block=block, flags=flags)
    assert np.array_equal(rgb.view(np.uint32), ref.view(np.uint32))
    assert cnt[0] == rc["paths"] and cnt[1] == rc["rays"]


def test_render_full_config_invariants_and_sampled_pixels(ctx):
    cfg = I.C4
    a, ca = render(ctx, cfg, sr.SPEC_LOOP, 32)
    b, cb = render(ctx, cfg, sr.PDOM, 0)
    c, cc = render(ctx, cfg, sr.SPEC_LOOP, 16, flags=sr.F_COARSE)
    d, cd = render(ctx, cfg, sr.SPEC_LOOP, 8, flags=sr.F_NOSPLIT)
    e, ce = render(ctx, cfg, sr.SPEC_LOOP, cfg.threshold, flags=sr.F_MATGROUP)
    f, cf = render(ctx, cfg, sr.SPEC_LOOP, cfg.threshold, flags=sr.F_POOL)
    assert np.array_equal(a.view(np.uint32), e.view(np.uint32)) and np.array_equal(ca, ce)
    assert np.array_equal(a.view(np.uint32), f.view(np.uint32)) and np.array_equal(ca, cf)
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    assert np.array_equal(a.view(np.uint32), c.view(np.uint32))
    assert np.array_equal(a.view(np.uint32), d.view(np.uint32))
    # rays, node visits and triangle tests too: every schedule runs each
    # lane's traversal in the same order
    assert np.array_equal(ca, cb) and np.array_equal(ca, cc) and np.array_equal(ca, cd)
    assert ca[0] == cfg.n_pixels * cfg.spp
    tris, mat, mats, cam, buf, used = scene(cfg)
    pix = np.array([0, 1023, 512 * 1024 + 512, 700 * 1024 + 300, 1024 * 1024 - 1, 123457],
                   np.uint32)
    ref, _ = oracle.pt_render(oracle.pt_scene(tris, mat, mats, cam), cfg.width, cfg.height,
                              cfg.spp, cfg.max_depth, I.PRIMARY_SEED, pixels=pix)
    assert np.array_equal(a[pix].view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("mode,T,pool", [(sr.PDOM, 0, False), (sr.SPEC_LOOP, 12, False),
                                         (sr.SPEC_LOOP, 32, False), (sr.SPEC_LOOP, 1, False),
                                         (sr.SPEC_LOOP, 12, True), (sr.SPEC_LOOP, 1, True),
                                         (sr.SPEC_LOOP, 32, True)])
def test_schedule_matches_simulator(ctx, mode, T, pool):
    """per-warp schedule counters of the instrumented kernels (split merge, U = 8;
    with and without the warp's path pool) == the path-tracer warp simulator
    replaying the oracle's work-item streams"""
    cfg = I.C4_SMALL
    tris, mat, mats, cam, buf, used = scene(cfg)
    n = cfg.width * cfg.height
    w = sr.pathtrace_workload(buf.data_ptr(), used, cfg.width, cfg.height, cfg.max_depth,
                              flags=sr.F_SCHED | (sr.F_POOL if pool else 0),
                              pool_spp=cfg.spp if pool else 0)
    ctx.ensure(sr.sr_workspace_bytes(w, n))
    sr.sr_run(w, n, cfg.spp, I.PRIMARY_SEED, mode, T)
    sched = ctx.region(w, n, sr.T_SCHED, torch.int32).view(-1, sr.SCHED_WORDS).cpu().numpy()
    cnt = ctx.region(w, n, sr.T_COUNTERS, torch.int64).cpu().numpy()
    img = sr.scene_image_host(tris, mat, mats, cam)
    ops, off, _ = oracle.pt_trace(img, cfg.width, cfg.height, cfg.spp, cfg.max_depth,
                                  I.PRIMARY_SEED, pixels=I.pt_lane_pixels(cfg.width, cfg.height))
    node = (ops & 0xE000) == 0
    leaf = (ops & 0x8000) != 0
    assert cnt[2] == int(node.sum()) and cnt[3] == int(leaf.sum())   # node visits, tests
    for wi in range(n // 32):
        o = off[32 * wi:32 * wi + 33]
        s = oracle.ws_pt(ops[o[0]:o[-1]], o - o[0],
                         oracle.PDOM if mode == sr.PDOM else
                         (oracle.SPEC_LOOP_POOL if pool else oracle.SPEC_LOOP), T, 8)
        g = sched[wi]
        if mode == sr.PDOM:
            assert (g[1], g[2]) == s["BOUNCE"], wi
            assert g[0] == s["OUTER"][0] and g[4] == s["LAUNCH"][1], wi
        else:
            assert g[0] == s["rounds"], wi
            assert (g[1], g[2]) == s["NREL"] and (g[5], g[6]) == s["LREL"], wi
            assert (g[3], g[4]) == s["ADV"], wi


@pytest.mark.parametrize("T", [1, 12, 32])
def test_pool_ragged_frame_bit_exact(ctx, T):
    """the path pool on a frame whose last warp is partial (315 pixels: 9 full warps
    and 27 lanes), with pool_spp above the run's spp: pixels and counters equal the
    oracle's; a run asking for more samples than pool_spp is refused"""
    import dataclasses
    cfg = dataclasses.replace(I.C4_SMALL, width=45, height=7, spp=3)
    tris, mat, mats, cam, buf, used = scene(cfg)
    ref, rc = oracle.pt_render(oracle.pt_scene(tris, mat, mats, cam), cfg.width, cfg.height,
                               cfg.spp, cfg.max_depth, I.PRIMARY_SEED)
    rgb, cnt = render(ctx, cfg, sr.SPEC_LOOP, T, flags=sr.F_POOL, pool_spp=5)
    assert np.array_equal(rgb.view(np.uint32), ref.view(np.uint32))
    assert cnt[0] == rc["paths"] and cnt[1] == rc["rays"]
    w = sr.pathtrace_workload(buf.data_ptr(), used, cfg.width, cfg.height, cfg.max_depth,
                              flags=sr.F_POOL, pool_spp=2)
    with pytest.raises(sr.SRError) as e:
        sr.sr_run(w, cfg.width * cfg.height, cfg.spp, I.PRIMARY_SEED, sr.SPEC_LOOP, T)
    assert e.value.code == sr.SR_E_INVALID and "pool_spp" in str(e.value)
