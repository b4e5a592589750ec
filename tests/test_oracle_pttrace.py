"""Pins of the path tracer's work-item oracle (oracle/pttrace.c, oracle part 2):
the BVH-traversal replay renders the brute-force oracle's image bit for bit, its
streams count exactly the rays / paths the renderer reports, and the PDOM and
split-merge schedules replay every work item exactly once (conservation), with
the merge's releases bounded by the closed forms of its rule."""
import numpy as np
import pytest

import oracle
from oracle import PDOM, SPEC_LOOP, SPEC_LOOP_POOL
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import sr


@pytest.fixture(scope="module")
def small():
    c = I.C4_SMALL
    tris, mat, mats, cam = I.cornell_scene(c)
    img = sr.scene_image_host(tris, mat, mats, cam)
    ops, off, rgb = oracle.pt_trace(img, c.width, c.height, c.spp, c.max_depth, I.PRIMARY_SEED)
    ref, rc = oracle.pt_render(oracle.pt_scene(tris, mat, mats, cam), c.width, c.height, c.spp,
                               c.max_depth, I.PRIMARY_SEED)
    return c, ops, off, rgb, ref, rc


def _kinds(ops):
    node = (ops & 0xE000) == 0
    leaf = (ops & 0x8000) != 0
    shade = (ops & 0xC000) == 0x4000
    path = (ops & 0xE000) == 0x2000
    return node, leaf, shade, path


def test_bvh_replay_renders_the_brute_force_image(small):
    c, ops, off, rgb, ref, rc = small
    assert np.array_equal(rgb.view(np.uint32), ref.view(np.uint32))
    node, leaf, shade, path = _kinds(ops)
    assert int(shade.sum()) == rc["rays"] and int(path.sum()) == rc["paths"]
    # every node op's queued leaf tests follow it, then the next node / shade op
    n_q = (ops & 15) + ((ops >> 4) & 15)
    assert int(leaf.sum()) == int(n_q[node].sum())
    # every ray's traversal ends exactly once, right before its shading op
    ends = node & ((ops & 0x400) != 0)
    assert int(ends.sum()) == int(shade.sum())
    # a path ends exactly once (its last shading op)
    assert int((shade & ((ops & 16) != 0)).sum()) == rc["paths"]


@pytest.mark.parametrize("T,U", [(1, 1), (12, 8), (32, 1), (32, 8), (4, 3)])
def test_schedules_replay_every_work_item_once(small, T, U):
    c, ops, off, rgb, ref, rc = small
    node, leaf, shade, path = _kinds(ops)
    for w in range(0, c.width * c.height, 32 * 17):   # a spread of warps
        o = off[w:w + 33]
        seg = ops[o[0]:o[-1]]
        nd, lf, sh, pa = _kinds(seg)
        for mode, t, u in ((PDOM, 0, 1), (SPEC_LOOP, T, U), (SPEC_LOOP_POOL, T, U)):
            s = oracle.ws_pt(seg, o - o[0], mode, t, u)
            assert s["NODE"][1] == int(nd.sum()) and s["LEAF"][1] == int(lf.sum())
            assert s["SH"][1] == int(sh.sum()) and s["LAUNCH"][1] == int(pa.sum())
            assert s["TT"] == s["LEAF"]
            assert s["TT_UPD"][1] == int((seg[lf] & 7 == 5).sum())
        if True:
            s = oracle.ws_pt(seg, o - o[0], SPEC_LOOP, T, U)
            # a release runs one group: node releases carry the node visits, leaf
            # releases the tests, at most U items per lane per release
            assert s["REL"][0] == s["NREL"][0] + s["LREL"][0]
            assert s["STEP"][1] == s["NODE"][1] and s["NREL"][0] * U >= s["STEP"][0] // 32
            assert s["rounds"] == s["REL"][0] + s["ADV"][0]
            # every ray starts in an advance round
            assert s["TBEGIN"][1] == int(sh.sum())


def test_pdom_schedule_closed_form(small):
    """PDOM: one outer trip per sample (every lane), a bounce iteration per
    bounce of the warp's longest path, one traversal step per node visit of the
    warp's longest traversal"""
    c, ops, off, rgb, ref, rc = small
    o = off[0:33]
    seg = ops[o[0]:o[-1]]
    s = oracle.ws_pt(seg, o - o[0], PDOM)
    assert s["OUTER"] == (c.spp, 32 * c.spp) and s["LAUNCH"] == (c.spp, 32 * c.spp)
    # per sample, bounce iterations = the longest path's rays
    rays_per_path = []
    for l in range(32):
        lane = ops[off[l]:off[l + 1]]
        _, _, sh, pa = _kinds(lane)
        starts = np.flatnonzero(pa)
        bounds = list(starts) + [len(lane)]
        rays_per_path.append([int(sh[bounds[i]:bounds[i + 1]].sum()) for i in range(len(starts))])
    rp = np.array(rays_per_path)            # [lane, sample]
    assert s["BOUNCE"][0] == int(rp.max(0).sum()) and s["BOUNCE"][1] == int(rp.sum())


@pytest.mark.parametrize("T,U", [(1, 1), (12, 8), (32, 8)])
def test_pool_reduces_to_fixed_pixels(small, T, U):
    """the path pool claims path q = (sample q / 32 of pixel q % 32) in lane order:
    (a) with one sample per pixel the first 32 claims give lane l its own pixel,
    (b) with 32 identical pixels every lane finishes a sample together with the
    others and claims its own pixel's next one -- in both cases the schedule is the
    fixed-pixel one, count for count"""
    c, ops, off, rgb, ref, rc = small
    _, _, _, path = _kinds(ops)
    for w in range(0, c.width * c.height, 32 * 23):
        o = off[w:w + 33]
        seg = ops[o[0]:o[-1]]
        # (a) the first sample of each pixel only
        lanes = []
        for l in range(32):
            lane = ops[off[w + l]:off[w + l + 1]]
            starts = np.flatnonzero(_kinds(lane)[3])
            lanes.append(lane[:starts[1]] if len(starts) > 1 else lane)
        one = np.concatenate(lanes)
        o1 = np.concatenate([[0], np.cumsum([len(x) for x in lanes])]).astype(np.uint64)
        pooled = oracle.ws_pt(one, o1, SPEC_LOOP_POOL, T, U)
        assert pooled.pop("PSUM") == (1, 32)        # then one in-order sum per pixel
        assert pooled == {k: v for k, v in oracle.ws_pt(one, o1, SPEC_LOOP, T, U).items()
                          if k != "PSUM"}
        # (b) 32 copies of pixel w's stream
        lane0 = ops[off[w]:off[w + 1]]
        same = np.tile(lane0, 32)
        o2 = (np.arange(33) * len(lane0)).astype(np.uint64)
        pooled = oracle.ws_pt(same, o2, SPEC_LOOP_POOL, T, U)
        assert pooled.pop("PSUM") == (c.spp, 32 * c.spp)
        assert pooled == {k: v for k, v in oracle.ws_pt(same, o2, SPEC_LOOP, T, U).items()
                          if k != "PSUM"}


def test_pool_balances_unequal_pixels(small):
    """a warp whose pixels carry very different work: with the pool the warp needs
    fewer rounds and its releases run with more lanes (idle lanes take other pixels'
    samples instead of waiting for the longest pixel)"""
    c, ops, off, rgb, ref, rc = small
    # lane l gets pixel w's stream (long) for l < 4, else pixel v's first sample only
    node, _, _, _ = _kinds(ops)
    work = np.array([int(node[off[i]:off[i + 1]].sum()) for i in range(len(off) - 1)])
    w, v = int(np.argmax(work)), int(np.argmin(work))
    lv = ops[off[v]:off[v + 1]]
    starts = np.flatnonzero(_kinds(lv)[3])
    short = lv[:starts[1]] if len(starts) > 1 else lv
    lanes = [ops[off[w]:off[w + 1]]] * 4 + [short] * 28
    seg = np.concatenate(lanes)
    o = np.concatenate([[0], np.cumsum([len(x) for x in lanes])]).astype(np.uint64)
    fixed = oracle.ws_pt(seg, o, SPEC_LOOP, 12, 8)
    pooled = oracle.ws_pt(seg, o, SPEC_LOOP_POOL, 12, 8)
    assert pooled["NODE"][1] == fixed["NODE"][1] and pooled["LEAF"][1] == fixed["LEAF"][1]
    assert pooled["rounds"] < fixed["rounds"]
    assert pooled["NODE"][1] / pooled["NODE"][0] > fixed["NODE"][1] / fixed["NODE"][0]
