"""Host logic of the path tracer's scene builder (sr_scene_build_host, no GPU):
the image layout of csrc/pt_scene.h, every triangle referenced exactly once,
every child box enclosing its subtree (the conservativeness the kernels' exact
closest hit relies on, reading R7), the recorded traversal-stack
bound equal to the tree's, the per-triangle edge vectors equal to the binary32
subtractions the oracle performs, and input validation."""
import numpy as np
import pytest

from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import sr

HDR = np.dtype([("magic", "<u4"), ("n_nodes", "<u4"), ("n_tris", "<u4"), ("n_mats", "<u4"),
                ("off_nodes", "<u8"), ("off_tris", "<u8"), ("off_mats", "<u8"), ("bytes", "<u8"),
                ("cam", "<f4", 16), ("stack_need", "<u4"), ("pad", "<u4", 3)])
NODE = np.dtype([("lo", "<f4", (3, 2)), ("hi", "<f4", (3, 2)),   # [axis][child]
                 ("ref0", "<i4"), ("cnt0", "<i4"), ("ref1", "<i4"), ("cnt1", "<i4")])
TRI = np.dtype([("v0", "<f4", 3), ("e1", "<f4", 3), ("e2", "<f4", 3), ("id", "<u4"),
                ("mat", "<u4"), ("pad", "<u4")])


def parse(img):
    h = np.frombuffer(img[:HDR.itemsize], HDR)[0]
    nodes = np.frombuffer(img[h["off_nodes"]:h["off_tris"]], NODE)
    tris = np.frombuffer(img[h["off_tris"]:h["off_mats"]], TRI)
    mats = np.frombuffer(img[h["off_mats"]:h["bytes"]], np.float32).reshape(-1, 8)
    return h, nodes, tris, mats


@pytest.fixture(scope="module", params=["small", "full"])
def scene(request):
    cfg = I.C4_SMALL if request.param == "small" else I.C4
    t, m, mats, cam = I.cornell_scene(cfg)
    return t, m, mats, cam, parse(sr.scene_image_host(t, m, mats, cam))


def test_layout_and_triangles(scene):
    t, m, mats, cam, (h, nodes, tris, M) = scene
    assert h["magic"] == 0x53525054 and h["n_tris"] == len(t) and h["n_mats"] == len(mats)
    assert h["n_nodes"] == len(nodes) and h["off_nodes"] == HDR.itemsize
    assert np.array_equal(h["cam"][:14], cam[:14]) and np.array_equal(M, mats)
    # a permutation of the input, with the oracle's binary32 edge vectors
    assert np.array_equal(np.sort(tris["id"]), np.arange(len(t)))
    src = t.reshape(-1, 3, 3)[tris["id"]]
    assert np.array_equal(tris["v0"], src[:, 0])
    assert np.array_equal(tris["e1"], (src[:, 1] - src[:, 0]).astype(np.float32))
    assert np.array_equal(tris["e2"], (src[:, 2] - src[:, 0]).astype(np.float32))
    assert np.array_equal(tris["mat"], m[tris["id"]])


def test_tree_covers_every_triangle_once_and_boxes_enclose(scene):
    t, m, mats, cam, (h, nodes, tris, M) = scene
    src = t.reshape(-1, 3, 3)[tris["id"]]
    tlo, thi = src.min(axis=1), src.max(axis=1)
    seen = np.zeros(len(tris), np.int64)
    depth_need = 0
    # iterative DFS over (node, pushed-entries-on-the-path)
    stack = [(0, 0)]
    while stack:
        i, d = stack.pop()
        depth_need = max(depth_need, d)
        nd = nodes[i]
        inner = [(nd["ref0"], nd["cnt0"], nd["lo"][:, 0], nd["hi"][:, 0]),
                 (nd["ref1"], nd["cnt1"], nd["lo"][:, 1], nd["hi"][:, 1])]
        both = all(r >= 0 and c == 0 for r, c, _, _ in inner)
        for r, c, lo, hi in inner:
            if r < 0:
                continue
            if c > 0:                      # leaf: its triangles inside the (padded) box
                assert 1 <= c <= 8
                seen[r:r + c] += 1
                assert np.all(tlo[r:r + c] >= lo) and np.all(thi[r:r + c] <= hi)
            else:
                assert 0 < r < len(nodes)  # pre-order: children after the parent
                ch = nodes[r]
                for k in (0, 1):           # a child's boxes lie inside its parent's box
                    if ch[f"ref{k}"] >= 0:
                        assert np.all(ch["lo"][:, k] >= lo) and np.all(ch["hi"][:, k] <= hi)
                stack.append((r, d + (1 if both else 0)))
    assert np.all(seen == 1)
    assert h["stack_need"] == depth_need
    assert 0 < h["stack_need"] <= 256


def test_deterministic_and_validated():
    t, m, mats, cam = I.cornell_scene(I.C4_SMALL)
    a = sr.scene_image_host(t, m, mats, cam)
    b = sr.scene_image_host(t, m, mats, cam)
    assert np.array_equal(a, b)
    bad = t.copy()
    bad[3, 4] = np.nan
    with pytest.raises(sr.SRError, match="non-finite"):
        sr.scene_image_host(bad, m, mats, cam)
    mm = m.copy()
    mm[0] = len(mats)
    with pytest.raises(sr.SRError, match="material id"):
        sr.scene_image_host(t, mm, mats, cam)
    img = np.zeros(16, np.uint8)
    with pytest.raises(sr.SRError, match="dst_bytes"):
        sr.sr_scene_build(t, m, mats, cam, img.ctypes.data, 16, host=True)


def test_pt_lane_pixels_layout():
    """the kernels' lane -> pixel layout: a permutation of the frame; with 8 x 4 tiles
    every warp's 32 pixels form one tile; otherwise the identity"""
    w, h = 64, 48
    m = I.pt_lane_pixels(w, h)
    assert m.dtype == np.uint32 and np.array_equal(np.sort(m), np.arange(w * h))
    for wi in range(w * h // 32):
        px, py = m[32 * wi:32 * wi + 32] % w, m[32 * wi:32 * wi + 32] // w
        assert px.max() - px.min() == 7 and py.max() - py.min() == 3
        assert px.min() == 8 * (wi % (w // 8)) and py.min() == 4 * (wi // (w // 8))
    assert np.array_equal(I.pt_lane_pixels(45, 7), np.arange(45 * 7))
    assert np.array_equal(I.pt_lane_pixels(64, 6), np.arange(64 * 6))
