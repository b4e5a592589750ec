"""Pins of the oracle's path tracer (config 4): closest hit against an
independent float64 plane/barycentric intersection, an all-emitter box
(exact), the white furnace (closed form Le * sum_k rho^k, RR unbiased), and
pixel-subset consistency."""
import math

import numpy as np
import pytest

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I


def box_tris():
    """Closed unit box, 12 triangles, inward-agnostic (the tracer flips normals)."""
    q = I._quad
    faces = [q([0, 0, 0], [1, 0, 0], [1, 0, 1], [0, 0, 1]), q([0, 1, 0], [0, 1, 1], [1, 1, 1], [1, 1, 0]),
             q([0, 0, 1], [1, 0, 1], [1, 1, 1], [0, 1, 1]), q([0, 0, 0], [0, 1, 0], [1, 1, 0], [1, 0, 0]),
             q([0, 0, 0], [0, 0, 1], [0, 1, 1], [0, 1, 0]), q([1, 0, 0], [1, 1, 0], [1, 1, 1], [1, 0, 1])]
    return np.concatenate(faces).reshape(-1, 9).astype(np.float32)


def camera(w, h, fov=65.0):
    cam = np.zeros(16, np.float32)
    cam[:12] = [0.5, 0.5, 0.02, 0, 0, 1, 1, 0, 0, 0, 1, 0]
    cam[12] = math.tan(math.radians(fov) / 2)
    cam[13] = w / h
    return cam


def hit64(tris, o, d):
    """Independent reference: plane intersection + barycentric inside test in
    float64 (not Moller-Trumbore).  Returns (index, t, margin) where margin is
    the smallest barycentric coordinate (how far inside the triangle)."""
    v0, v1, v2 = (tris[:, 0:3].astype(np.float64), tris[:, 3:6].astype(np.float64),
                  tris[:, 6:9].astype(np.float64))
    n = np.cross(v1 - v0, v2 - v0)
    den = n @ d
    with np.errstate(divide="ignore", invalid="ignore"):
        t = ((v0 - o) * n).sum(1) / den
    p = o + t[:, None] * d
    area = np.einsum("ij,ij->i", n, n)
    b0 = np.einsum("ij,ij->i", np.cross(v1 - p, v2 - p), n) / area
    b1 = np.einsum("ij,ij->i", np.cross(v2 - p, v0 - p), n) / area
    b2 = 1 - b0 - b1
    margin = np.minimum(np.minimum(b0, b1), b2)
    ok = (t > 1e-4) & (margin >= 0) & np.isfinite(t)
    if not ok.any():
        return -1, math.inf, 0.0
    i = int(np.argmin(np.where(ok, t, np.inf)))
    return i, float(t[i]), float(margin[i])


def test_closest_hit_matches_independent_intersection():
    tris, mat, mats, cam = I.cornell_scene(I.C4_SMALL)
    sc = oracle.pt_scene(tris, mat, mats, cam)
    rng = np.random.default_rng(7)
    agree = checked = 0
    for _ in range(400):
        o = rng.uniform(0.05, 0.95, 3)
        d = rng.normal(size=3)
        d /= np.linalg.norm(d)
        i, t = oracle.pt_closest(sc, o.astype(np.float32), d.astype(np.float32))
        j, t64, margin = hit64(tris, o.astype(np.float32).astype(np.float64),
                               d.astype(np.float32).astype(np.float64))
        if margin < 1e-5:      # grazing an edge: float32 and float64 may legitimately differ
            continue
        checked += 1
        agree += (i == j)
        assert i == j, (o, d, i, j)
        assert abs(t - t64) <= 1e-5 * max(1.0, t64)
    assert checked > 350


def test_all_emitter_box_is_exact():
    tris = box_tris()
    w, h, spp = 16, 12, 3
    mats = np.array([[3, 0, 0, 0, 1, 1, 1, 1]], np.float32)
    sc = oracle.pt_scene(tris, np.zeros(len(tris), np.uint32), mats, camera(w, h))
    rgb, cnt = oracle.pt_render(sc, w, h, spp, 8, 1)
    assert np.all(rgb == spp)                 # every camera ray hits a light of Le = 1
    assert cnt == dict(paths=w * h * spp, rays=w * h * spp)


@pytest.mark.parametrize("rho", [0.5, 0.8])
def test_white_furnace(rho):
    # every surface diffuse with albedo rho and emission Le: E[L] = Le sum_{k<D} rho^k
    tris = box_tris()
    D, Le = 8, 1.0
    mats = np.array([[0, rho, rho, rho, Le, Le, Le, 1]], np.float32)
    w, h, spp = 32, 32, 8
    sc = oracle.pt_scene(tris, np.zeros(len(tris), np.uint32), mats, camera(w, h))
    rgb, cnt = oracle.pt_render(sc, w, h, spp, D, 3)
    per_pixel = rgb[:, 0] / spp
    expect = Le * sum(rho**k for k in range(D))
    sigma = per_pixel.std() / math.sqrt(len(per_pixel))
    assert abs(per_pixel.mean() - expect) < 5 * sigma + 1e-6
    assert np.all(rgb[:, 0] == rgb[:, 1]) and np.all(rgb[:, 1] == rgb[:, 2])
    assert cnt["paths"] == w * h * spp


def test_pixel_subset_matches_full_render():
    c = I.C4_SMALL
    tris, mat, mats, cam = I.cornell_scene(c)
    sc = oracle.pt_scene(tris, mat, mats, cam)
    w, h = 16, 8
    full, _ = oracle.pt_render(sc, w, h, 2, c.max_depth, 5)
    pix = np.array([0, 17, 100, w * h - 1], np.uint32)
    sub, cnt = oracle.pt_render(sc, w, h, 2, c.max_depth, 5, pixels=pix)
    assert np.array_equal(sub, full[pix])
    assert cnt["paths"] == 2 * len(pix)


def test_scene_shape_matches_config():
    c = I.C4
    assert 20 * 4**c.subdiv * c.n_spheres + 14 == 1_044_494
