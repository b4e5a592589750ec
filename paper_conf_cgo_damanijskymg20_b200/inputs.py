"""Seeded synthetic inputs shared by the CUDA path and the oracle.

This module holds ONLY workload descriptions -- parameter tables, sizes,
seeds -- and no arithmetic of the method.  Both sides derive everything else
(Philox draws, derived physical constants, bins) themselves.  The recipe is
stated in DESIGN.md ("Input recipe"); the paper gives no workload parameters
for any of the shapes in BASELINE.json, so these are ours.
"""
from __future__ import annotations

from dataclasses import dataclass, field

SEEDS = (20200222, 1, 0xFFFFFFFFFFFFFFFF)   # primary seed first
PRIMARY_SEED = SEEDS[0]


@dataclass(frozen=True)
class DivLoop:
    """Config 1 (BASELINE.json configs[0]): Fig. 2(a) / Listing 1 microbench."""
    n_threads: int = 32768
    iters: int = 64
    p_u32: int = 1 << 29        # P(branch) = 1/8 exactly
    fma_count: int = 1000       # Expensive() = 1000 FMAs
    threshold: int = 16
    advance_unroll: int = 8     # iterations a run-ahead lane may take per round, tuned on B200
    pool_split: int = 4         # warp task pool (SR_F_POOL): warps per 32 threads, tuned on B200


@dataclass(frozen=True)
class CommonCall:
    """Config 2 (BASELINE.json configs[1]): Fig. 2(c) microbench."""
    n_threads: int = 1 << 20
    iters: int = 1
    split_u32: int = 1 << 31    # 50/50 thread-varying split
    fma_count: int = 2000


@dataclass(frozen=True)
class RSBench:
    """NEXT-1: RSBench-shaped nested trip-count loop (Fig. 3).
    Materials / nuclide counts / selection probabilities: DESIGN.md R8."""
    n_threads: int = 131072
    iters: int = 32             # lookups per thread (thread coarsening)
    fma_count: int = 64         # FMAs of the per-nuclide body
    threshold: int = 32         # best of the sweep with the warp task pool (r02e; the
                                # static assignment's best was 24, profiles/threshold_sweep_*.md)
    prolog_fma: int = 0         # FMAs of the lookup prolog (expensive task fetch)
    merge_unroll: int = 12      # inner iterations per release, tuned on B200


NEXT1 = RSBench()
# Fig. 9's XSBench case: an expensive task fetch (2048 FMAs per
# lookup prolog, ~0.6x the mean inner-loop work of a lookup) -- refilling idle
# lanes often no longer pays, the best threshold drops
NEXT1_FETCH = RSBench(prolog_fma=2048, threshold=20)   # best of the pool sweep r02h (static: 12)


# (n, mua [1/cm], mus [1/cm], g, d [cm]) -- a synthetic 3-layer tissue slab
THREE_LAYER = ((1.4, 4.0, 96.0, 0.80, 0.01),
               (1.4, 1.0, 199.0, 0.90, 0.10),
               (1.4, 2.0, 98.0, 0.75, 0.40))


@dataclass(frozen=True)
class MCML:
    """Configs 3 / 5: MC photon transport in a multi-layered slab."""
    layers: tuple = THREE_LAYER
    n_above: float = 1.0
    n_below: float = 1.0
    dr: float = 0.01
    dz: float = 0.002
    nr: int = 256
    nz: int = 255
    step_cap: int = 100000
    n_threads: int = 156250     # lanes
    iters: int = 64             # photons per lane (thread coarsening)
    threshold: int = 32
    merge_unroll: int = 4       # photon steps per release, tuned on B200

    @property
    def n_photons(self) -> int:
        return self.n_threads * self.iters


# Pins with closed forms / published values (tests only use these through
# the oracle): Beer-Lambert slab, no scattering, matched boundaries.
BEER_LAMBERT = MCML(layers=((1.0, 10.0, 0.0, 0.0, 0.1),), nz=100, dz=0.001)
# mua = 0: no absorption, no roulette -> exact weight conservation
NO_ABSORPTION = MCML(layers=((1.4, 0.0, 50.0, 0.9, 0.02),))
# classic MCML validation slab (n=1, mua=10, mus=90, g=0.75, d=0.02 cm)
VAN_DE_HULST = MCML(layers=((1.0, 10.0, 90.0, 0.75, 0.02),))
# index-mismatched absorbing slab in air, no scattering: a normally incident
# pencil beam bounces between the two faces (Fresnel r = ((n-1)/(n+1))^2 at
# each), so Rd, Tt and A follow the multiple-reflection series in closed form
MISMATCHED_ABSORBER = MCML(layers=((1.4, 5.0, 0.0, 0.0, 0.1),), nz=100, dz=0.001)

C1 = DivLoop()
C2 = CommonCall()
C3 = MCML()
# configs[4]: 10^9 photons of C3 in total, sharded over 1/2/4/8 GPUs (strong scaling)
C5_TOTAL_PHOTONS = 10**9


# ---------------------------------------------------------------- config 4 scene
# Materials: (kind, r, g, b, er, eg, eb, ior); kind 0 diffuse, 1 mirror,
# 2 dielectric, 3 emissive-only (light).
MAT_DIFFUSE, MAT_MIRROR, MAT_GLASS, MAT_LIGHT = 0, 1, 2, 3


@dataclass(frozen=True)
class PathTrace:
    """Config 4 (BASELINE.json configs[3]): Cornell box + icospheres, BVH."""
    width: int = 1024
    height: int = 1024
    spp: int = 16
    max_depth: int = 8
    n_spheres: int = 51
    subdiv: int = 5          # 20 * 4^5 = 20480 triangles per sphere; 51 -> 1,044,494 total
    fov_deg: float = 65.0
    scene_seed: int = 20200222
    threshold: int = 12      # best of the tools/exp_pt_minb.sh sweep (split merge, unroll 8)

    @property
    def n_pixels(self) -> int:
        return self.width * self.height


C4 = PathTrace()
C4_SMALL = PathTrace(width=64, height=48, spp=4, subdiv=1)   # oracle-sized parity case


def pt_lane_pixels(width: int, height: int):
    """Launch layout of the path-tracing kernels (not the method): the pixel of
    lane slot i = 32 w + l.  When the frame splits into 8 x 4 tiles, warp w
    covers tile w (tiles row-major, lanes row-major inside a tile); otherwise
    slot i is pixel i.  uint32 array of width * height entries; the warp
    simulator replays warp w's lanes as entries [32 w, 32 w + 32)."""
    import numpy as np
    n = width * height
    i = np.arange(n, dtype=np.int64)
    if width % 8 or height % 4:
        return i.astype(np.uint32)
    w, l = i >> 5, i & 31
    tpr = width // 8
    return (((w // tpr) * 4 + (l >> 3)) * width + (w % tpr) * 8 + (l & 7)).astype(np.uint32)


def _icosphere(subdiv: int):
    """Unit icosphere as a float64 triangle soup [n, 3, 3]; midpoints are
    computed from the two endpoint values only, so shared edges stay shared."""
    import numpy as np
    t = (1.0 + 5.0 ** 0.5) / 2.0
    v = np.array([[-1, t, 0], [1, t, 0], [-1, -t, 0], [1, -t, 0], [0, -1, t], [0, 1, t],
                  [0, -1, -t], [0, 1, -t], [t, 0, -1], [t, 0, 1], [-t, 0, -1], [-t, 0, 1]],
                 np.float64)
    v /= np.linalg.norm(v, axis=1, keepdims=True)
    f = np.array([[0, 11, 5], [0, 5, 1], [0, 1, 7], [0, 7, 10], [0, 10, 11], [1, 5, 9],
                  [5, 11, 4], [11, 10, 2], [10, 7, 6], [7, 1, 8], [3, 9, 4], [3, 4, 2],
                  [3, 2, 6], [3, 6, 8], [3, 8, 9], [4, 9, 5], [2, 4, 11], [6, 2, 10],
                  [8, 6, 7], [9, 8, 1]])
    tri = v[f]                                           # [20, 3, 3]
    for _ in range(subdiv):
        a, b, c = tri[:, 0], tri[:, 1], tri[:, 2]
        ab, bc, ca = (a + b), (b + c), (c + a)
        ab /= np.linalg.norm(ab, axis=1, keepdims=True)
        bc /= np.linalg.norm(bc, axis=1, keepdims=True)
        ca /= np.linalg.norm(ca, axis=1, keepdims=True)
        tri = np.stack([np.stack([a, ab, ca], 1), np.stack([ab, b, bc], 1),
                        np.stack([ca, bc, c], 1), np.stack([ab, bc, ca], 1)], 1).reshape(-1, 3, 3)
    return tri


def _quad(p0, p1, p2, p3):
    """Two triangles of the quad p0-p1-p2-p3 (counter-clockwise)."""
    import numpy as np
    return np.array([[p0, p1, p2], [p0, p2, p3]], np.float64)


def cornell_scene(cfg: PathTrace = C4):
    """Seeded synthetic scene.  Returns (tris float32 [n, 9], mat uint32 [n],
    mats float32 [m, 8], cam float32 [12]).

    Closed unit Cornell box with the camera just inside its front wall, a small
    emissive ceiling quad, and cfg.n_spheres non-overlapping icospheres: 50 % diffuse, 20 %
    mirror, 20 % glass (ior 1.5), 10 % emissive.  cam = {eye, forward, right,
    up, tan(fov/2), aspect, 0} as floats (an orthonormal basis, float64 -> f32).
    """
    import numpy as np
    rng = np.random.default_rng(cfg.scene_seed)
    mats = [(MAT_DIFFUSE, .73, .73, .73, 0, 0, 0, 1.0),   # 0 white walls
            (MAT_DIFFUSE, .65, .05, .05, 0, 0, 0, 1.0),   # 1 red wall
            (MAT_DIFFUSE, .12, .45, .15, 0, 0, 0, 1.0),   # 2 green wall
            (MAT_LIGHT, 0, 0, 0, 15.0, 15.0, 15.0, 1.0)]  # 3 ceiling light
    tris, mat = [], []

    def add(t, m):
        tris.append(t)
        mat.extend([m] * len(t))
    add(_quad([0, 0, 0], [1, 0, 0], [1, 0, 1], [0, 0, 1]), 0)          # floor
    add(_quad([0, 1, 0], [0, 1, 1], [1, 1, 1], [1, 1, 0]), 0)          # ceiling
    add(_quad([0, 0, 1], [1, 0, 1], [1, 1, 1], [0, 1, 1]), 0)          # back
    add(_quad([0, 0, 0], [0, 1, 0], [1, 1, 0], [1, 0, 0]), 0)          # front (behind camera)
    add(_quad([0, 0, 0], [0, 0, 1], [0, 1, 1], [0, 1, 0]), 1)          # left, red
    add(_quad([1, 0, 0], [1, 1, 0], [1, 1, 1], [1, 0, 1]), 2)          # right, green
    add(_quad([.4, .999, .4], [.4, .999, .6], [.6, .999, .6], [.6, .999, .4]), 3)  # light
    unit = _icosphere(cfg.subdiv)
    centres = []
    kinds = rng.permutation([MAT_DIFFUSE] * 50 + [MAT_MIRROR] * 20 + [MAT_GLASS] * 20 +
                            [MAT_LIGHT] * 10)
    while len(centres) < cfg.n_spheres:
        r = rng.uniform(0.035, 0.075)
        c = rng.uniform(r + 0.01, 1 - r - 0.01, 3)
        c[2] = max(c[2], 0.25 + r)          # keep the spheres off the camera
        if all(np.linalg.norm(c - c2) > r + r2 + 0.005 for c2, r2 in centres):
            centres.append((c, r))
    for i, (c, r) in enumerate(centres):
        kind = int(kinds[i % len(kinds)])
        col = rng.uniform(0.2, 0.9, 3)
        if kind == MAT_LIGHT:
            mats.append((MAT_LIGHT, 0, 0, 0, *(4.0 * col), 1.0))
        elif kind == MAT_GLASS:
            mats.append((MAT_GLASS, 1, 1, 1, 0, 0, 0, 1.5))
        elif kind == MAT_MIRROR:
            mats.append((MAT_MIRROR, *(0.5 + 0.5 * col), 0, 0, 0, 1.0))
        else:
            mats.append((MAT_DIFFUSE, *col, 0, 0, 0, 1.0))
        add(unit * r + c, len(mats) - 1)
    tris = np.concatenate(tris).reshape(-1, 9).astype(np.float32)
    mat = np.array(mat, np.uint32)
    eye = np.array([0.5, 0.5, 0.02])
    fwd = np.array([0.5, 0.5, 0.5]) - eye
    fwd /= np.linalg.norm(fwd)
    right = np.cross(np.array([0.0, 1.0, 0.0]), fwd)
    right /= np.linalg.norm(right)
    up = np.cross(fwd, right)
    cam = np.concatenate([eye, fwd, right, up,
                          [np.tan(np.radians(cfg.fov_deg) / 2), cfg.width / cfg.height, 0.0]])
    return tris, mat, np.array(mats, np.float32), cam.astype(np.float32)
