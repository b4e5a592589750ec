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


@dataclass(frozen=True)
class CommonCall:
    """Config 2 (BASELINE.json configs[1]): Fig. 2(c) microbench."""
    n_threads: int = 1 << 20
    iters: int = 1
    split_u32: int = 1 << 31    # 50/50 thread-varying split
    fma_count: int = 2000


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

C1 = DivLoop()
C2 = CommonCall()
C3 = MCML()
