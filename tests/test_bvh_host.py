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
NODE = np.dtype([("lox", "<f4", 4), ("loy", "<f4", 4), ("loz", "<f4", 4),
                 ("hix", "<f4", 4), ("hiy", "<f4", 4), ("hiz", "<f4", 4),
                 ("ref", "<i4", 4), ("cnt", "<i4", 4)])
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
    assert h["magic"] == 0x34525054 and h["n_tris"] == len(t) and h["n_mats"] == len(mats)
    assert h["n_nodes"] == len(nodes) and h["off_nodes"] == HDR.itemsize
    assert np.array_equal(h["cam"][:14], cam[:14]) and np.array_equal(M, mats)
    # a permutation of the input, with the oracle's binary32 edge vectors
    assert np.array_equal(np.sort(tris["id"]), np.arange(len(t)))
    src = t.reshape(-1, 3, 3)[tris["id"]]
    assert np.array_equal(tris["v0"], src[:, 0])
    assert np.array_equal(tris["e1"], (src[:, 1] - src[:, 0]).astype(np.float32))
    assert np.array_equal(tris["e2"], (src[:, 2] - src[:, 0]).astype(np.float32))
    assert np.array_equal(tris["mat"], m[tris["id"]])


def _box(nd, k):
    return (np.array([nd["lox"][k], nd["loy"][k], nd["loz"][k]]),
            np.array([nd["hix"][k], nd["hiy"][k], nd["hiz"][k]]))


def test_tree_covers_every_triangle_once_and_boxes_enclose(scene):
    """four-wide nodes: every triangle in exactly one leaf of <= 8, every child box
    encloses its subtree, children stored after their parent, empty slots empty,
    and the recorded stack bound = max over root paths of sum (children - 1)"""
    t, m, mats, cam, (h, nodes, tris, M) = scene
    src = t.reshape(-1, 3, 3)[tris["id"]]
    tlo, thi = src.min(axis=1), src.max(axis=1)
    seen = np.zeros(len(tris), np.int64)
    need = {}
    order = []
    stack = [0]
    while stack:                       # DFS, then the bound bottom-up
        i = stack.pop()
        order.append(i)
        nd = nodes[i]
        for k in range(4):
            r, c = nd["ref"][k], nd["cnt"][k]
            lo, hi = _box(nd, k)
            if r < 0:
                assert c == 0 and np.all(lo == np.inf) and np.all(hi == -np.inf)
                continue
            if c > 0:                  # leaf: its triangles inside the (padded) box
                assert 1 <= c <= 8
                seen[r:r + c] += 1
                assert np.all(tlo[r:r + c] >= lo) and np.all(thi[r:r + c] <= hi)
            else:
                assert i < r < len(nodes)   # children after the parent
                ch = nodes[r]
                for kk in range(4):         # a child's boxes lie inside its parent's box
                    if ch["ref"][kk] >= 0:
                        clo, chi = _box(ch, kk)
                        assert np.all(clo >= lo) and np.all(chi <= hi)
                stack.append(r)
    for i in reversed(order):
        nd = nodes[i]
        kids = [nd["ref"][k] for k in range(4) if nd["ref"][k] >= 0 and nd["cnt"][k] == 0]
        nch = int((nd["ref"] >= 0).sum())
        need[i] = max(nch - 1, 0) + max([need[k] for k in kids], default=0)
    assert np.all(seen == 1)
    assert len(order) == len(nodes)    # every node reachable once
    assert h["stack_need"] == need[0]
    assert 0 < h["stack_need"] <= 256
    # four-wide: most nodes are full
    assert (nodes["ref"] >= 0).sum() >= 2.5 * len(nodes)


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
