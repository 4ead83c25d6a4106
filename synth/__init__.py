"""Seeded synthetic inputs shared by the oracle, the tests and bench.py.

This module holds NO arithmetic of the method (no covariance, no norms, no
factorisation): only the recipes that produce the inputs of one log-likelihood
evaluation, so both the CPU oracle (`oracle/`) and the CUDA path
(`paper_conf_cluster_caoalgkb23_b200`) can be fed identical data.

Recipe (readings C1/C2):
  * locations: jittered sqrt(n) x sqrt(n) grid on [0,1]^2,
      x = (i + 0.5 + U(-0.4, 0.4)) / side,  y = (j + 0.5 + U(-0.4, 0.4)) / side,
    drawn with numpy.random.default_rng(seed), then sorted by the Morton
    (z-order) key of (floor(65535 x), floor(65535 y)).  The paper only says
    "synthetic locations" (§VII-B); the spatial ordering is
    what makes tile norms decay away from the diagonal (§V).
  * observations: a seeded standard-normal vector e (default_rng(seed)).
    The measurement vector Z = L(theta_true) e is formed by whoever owns a
    Cholesky factor (the oracle in tests); for timing, Z = e is used because
    the cost of one evaluation does not depend on Z.
"""
from __future__ import annotations

import math

import numpy as np

__all__ = [
    "grid_side",
    "jittered_grid",
    "morton_keys",
    "morton_sort",
    "locations",
    "uniform_locations",
    "collinear_locations",
    "normal_vector",
]


def grid_side(n: int) -> int:
    side = math.isqrt(n)
    if side * side != n:
        raise ValueError(f"n={n} is not a perfect square (jittered-grid recipe needs side^2 points)")
    return side


def jittered_grid(n: int, seed: int = 0) -> tuple[np.ndarray, np.ndarray]:
    """Unsorted jittered grid, row-major over (i, j)."""
    side = grid_side(n)
    rng = np.random.default_rng(seed)
    jx = rng.uniform(-0.4, 0.4, size=n)
    jy = rng.uniform(-0.4, 0.4, size=n)
    i = np.repeat(np.arange(side, dtype=np.float64), side)
    j = np.tile(np.arange(side, dtype=np.float64), side)
    x = (i + 0.5 + jx) / side
    y = (j + 0.5 + jy) / side
    return x, y


def _part1by1(v: np.ndarray) -> np.ndarray:
    v = v.astype(np.uint64) & np.uint64(0xFFFF)
    v = (v | (v << np.uint64(8))) & np.uint64(0x00FF00FF)
    v = (v | (v << np.uint64(4))) & np.uint64(0x0F0F0F0F)
    v = (v | (v << np.uint64(2))) & np.uint64(0x33333333)
    v = (v | (v << np.uint64(1))) & np.uint64(0x55555555)
    return v


def morton_keys(x: np.ndarray, y: np.ndarray) -> np.ndarray:
    ix = np.floor(65535.0 * np.clip(x, 0.0, 1.0)).astype(np.uint64)
    iy = np.floor(65535.0 * np.clip(y, 0.0, 1.0)).astype(np.uint64)
    return _part1by1(ix) | (_part1by1(iy) << np.uint64(1))


def morton_sort(x: np.ndarray, y: np.ndarray) -> tuple[np.ndarray, np.ndarray]:
    order = np.argsort(morton_keys(x, y), kind="stable")
    return np.ascontiguousarray(x[order]), np.ascontiguousarray(y[order])


def locations(n: int, seed: int = 0) -> tuple[np.ndarray, np.ndarray]:
    """The benchmark/test locations: jittered grid, Morton order (float64 [n] each)."""
    return morton_sort(*jittered_grid(n, seed))


def uniform_locations(n: int, seed: int = 0) -> tuple[np.ndarray, np.ndarray]:
    """Uniform random points in [0,1]^2 (any n), Morton-sorted; for small brute-force cases."""
    rng = np.random.default_rng(seed)
    return morton_sort(rng.uniform(0.0, 1.0, n), rng.uniform(0.0, 1.0, n))


def collinear_locations(n: int, delta: float) -> tuple[np.ndarray, np.ndarray]:
    """x_i = i * delta, y_i = 0: with nu = 1/2 the covariance is Kac-Murdock-Szego."""
    return np.arange(n, dtype=np.float64) * delta, np.zeros(n, dtype=np.float64)


def normal_vector(n: int, seed: int = 1) -> np.ndarray:
    return np.random.default_rng(seed).standard_normal(n)
