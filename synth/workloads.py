"""Benchmark table and seeded input recipe.

Stencil shapes follow PAPER.md Table 3 (L328-L338): Heat-1D (3 points), Heat-2D
(5-point star), Box-2D9P, Heat-3D (7-point star), Box-3D27P; plus the large-radius
2D stencils of BASELINE.json configs[2] (Star-2D13P, r=3 star; Box-2D49P, 7x7 box).
The paper gives no coefficients (reading Q14) and no input distribution, so:

  weights  = shape mask x U(0.5, 1.5) from numpy default_rng(20250301), normalised
             to sum 1 (asymmetric, complex spectrum; the "seeded" set);
  classic  = the textbook symmetric set (Heat-1D 1/4,1/2,1/4; Heat-2D centre 1/2 and
             4 x 1/8; Heat-3D centre 0.4 and 6 x 0.1; boxes uniform 1/P; Star-2D13P
             centre 0.4 and 12 x 0.05);
  grid     = numpy default_rng(1234 + cfg_id).random(extents), float64 U[0,1).

Sizes are BASELINE.json's (not Table 3's 512M / 16K^2 / 768^3, reading Q16).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

WEIGHT_SEED = 20250301
GRID_SEED_BASE = 1234


def mask(shape: str, ndim: int, radius: int) -> np.ndarray:
    """Boolean offset cube [(2r+1)]*ndim: 'star' = axis-aligned arms, 'box' = full cube."""
    w = 2 * radius + 1
    if shape == "box":
        return np.ones((w,) * ndim, dtype=bool)
    if shape == "star":
        m = np.zeros((w,) * ndim, dtype=bool)
        for idx in np.ndindex(*m.shape):
            nz = sum(1 for i in idx if i != radius)
            m[idx] = nz <= 1
        return m
    raise ValueError(shape)


def seeded_weights(shape: str, ndim: int, radius: int, seed: int = WEIGHT_SEED) -> np.ndarray:
    m = mask(shape, ndim, radius)
    rng = np.random.default_rng(seed)
    w = rng.uniform(0.5, 1.5, size=m.shape) * m
    return (w / w.sum()).astype(np.float64)


def classic_weights(shape: str, ndim: int, radius: int) -> np.ndarray:
    m = mask(shape, ndim, radius)
    P = int(m.sum())
    if shape == "box":
        return (m / P).astype(np.float64)
    w = np.zeros(m.shape, dtype=np.float64)
    centre = (radius,) * ndim
    if ndim == 1 and radius == 1:
        return np.array([0.25, 0.5, 0.25])
    if radius == 1:
        c = {2: 0.5, 3: 0.4}[ndim]
    else:
        c = 0.4
    arm = (1.0 - c) / (P - 1)
    w[m] = arm
    w[centre] = c
    return w


def signed_weights(shape: str, ndim: int, radius: int, seed: int = WEIGHT_SEED + 1,
                   abs_sum: float = 1.6) -> np.ndarray:
    """Signed, un-normalised weights: shape mask x U(-1, 1), scaled so sum|w| = abs_sum; the
    centre tap is made positive and the largest (so the symbol's modulus can exceed 1 and
    the field may grow: SURVEY reading Q19 "other weights are allowed")."""
    m = mask(shape, ndim, radius)
    rng = np.random.default_rng(seed)
    w = rng.uniform(-1.0, 1.0, size=m.shape) * m
    c = (radius,) * ndim
    w[c] = np.abs(w).max() + 0.25
    return (w * (abs_sum / np.abs(w).sum())).astype(np.float64)


def gain_weights(shape: str, ndim: int, radius: int, gain: float = 1.2) -> np.ndarray:
    """The seeded set scaled to sum w = gain (> 1): the symbol's modulus peaks at gain at
    theta = 0, so a constant field grows by gain per step."""
    return (seeded_weights(shape, ndim, radius) * gain).astype(np.float64)


def stencil_weights(shape: str, ndim: int, radius: int, kind: str = "seeded") -> np.ndarray:
    if kind == "seeded":
        return seeded_weights(shape, ndim, radius)
    if kind == "signed":
        return signed_weights(shape, ndim, radius)
    if kind == "signed_unit":      # signed, sum|w| = 1 (bounded growth for long runs)
        return signed_weights(shape, ndim, radius, abs_sum=1.0)
    if kind == "gain":
        return gain_weights(shape, ndim, radius)
    return classic_weights(shape, ndim, radius)


def grid(extents, cfg_id: int = 0) -> np.ndarray:
    rng = np.random.default_rng(GRID_SEED_BASE + cfg_id)
    return rng.random(tuple(int(e) for e in extents))


def signed_grid(extents, cfg_id: int = 0) -> np.ndarray:
    """float64 U(-1, 1) input (signed values; the benchmark grids are U[0, 1))."""
    rng = np.random.default_rng(GRID_SEED_BASE + 7919 + cfg_id)
    return rng.uniform(-1.0, 1.0, tuple(int(e) for e in extents))


@dataclass(frozen=True)
class Workload:
    cfg_id: int
    name: str
    shape: str          # 'star' | 'box'
    ndim: int
    radius: int
    extents: tuple
    T: int              # fused depth requested (0 = auto)
    bench_steps: int
    parity_steps: int = 0   # 0 -> 2T+3
    notes: str = ""
    extras: dict = field(default_factory=dict)

    @property
    def points(self) -> int:
        return int(mask(self.shape, self.ndim, self.radius).sum())

    def weights(self, kind: str = "seeded") -> np.ndarray:
        return stencil_weights(self.shape, self.ndim, self.radius, kind)

    def grid(self, extents=None) -> np.ndarray:
        return grid(self.extents if extents is None else extents, self.cfg_id)


# BASELINE.json configs; cfg ids match SURVEY §8(d).
CONFIGS = {
    "heat1d": Workload(0, "Heat-1D", "star", 1, 1, (4096,), 8, 64, 64,
                       "configs[0]: N=4096, T=8, 64 steps"),
    "heat2d": Workload(1, "Heat-2D", "star", 2, 1, (10240, 10240), 0, 1000,
                       notes="configs[1]: 10240^2, T swept 1..16"),
    "box2d9p": Workload(2, "Box-2D9P", "box", 2, 1, (10240, 10240), 0, 1000,
                        notes="configs[1]: 10240^2, T swept 1..16"),
    "star2d13p": Workload(3, "Star-2D13P", "star", 2, 3, (10240, 10240), 0, 1000,
                          notes="configs[2]"),
    "box2d49p": Workload(4, "Box-2D49P", "box", 2, 3, (10240, 10240), 0, 1000,
                         notes="configs[2]"),
    "heat3d": Workload(5, "Heat-3D", "star", 3, 1, (1024, 1024, 1024), 0, 100,
                       notes="configs[3]"),
    "box3d27p": Workload(6, "Box-3D27P", "box", 3, 1, (1024, 1024, 1024), 0, 100,
                         notes="configs[3]"),
    # PAPER.md Table 3's 1D sizes (512M = 2^29 cells, reading Q16) for a meaningful 1D roofline
    "heat1d_512m": Workload(9, "Heat-1D 512M", "star", 1, 1, (1 << 29,), 0, 1000, notes="Table 3 L332"),
    "1d5p_512m": Workload(10, "1D5P 512M", "star", 1, 2, (1 << 29,), 0, 1000, notes="Table 3 L333"),
    "1d7p_512m": Workload(11, "1D7P 512M", "star", 1, 3, (1 << 29,), 0, 1000, notes="Table 3 L334"),
    "box2d9p_weak": Workload(7, "Box-2D9P weak", "box", 2, 1, (5120, 40960), 0, 1000,
                             notes="configs[4]: per-GPU slab; global (5120 g) x 40960"),
    "heat3d_weak": Workload(8, "Heat-3D weak", "star", 3, 1, (256, 1024, 1024), 0, 100,
                            notes="configs[4]: per-GPU slab; global (256 g) x 1024^2"),
}
