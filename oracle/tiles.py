"""Tiling, tile generation and tile norms.  Oracle: test infrastructure only.

Tile layout (§VII-A "tile size ... 2048"; reading C18): NT = ceil(n/nb);
tile (m, k) covers rows [m*nb, min(n, (m+1)*nb)) and columns [k*nb, min(n,
(k+1)*nb)); the last tile row/column is ragged (no padding in the oracle).
Only the lower triangle (m >= k) is generated, as the factorisation only
touches it (Alg. 1).

Tile norms (§V): ||A_mk||_F.  Readings:
  C8  the global norm ||A||_F is over the whole symmetric matrix (both
      triangles), real entries only:  S = sum_k s_kk + 2 * sum_{m>k} s_mk,
      with s_mk = ||A_mk||_F^2.
  O4  every sum of squares is the correctly rounded sum of the (rounded)
      squares (math.fsum), and S is formed as fsum(diag) + 2 * fsum(off).
"""
from __future__ import annotations

import math

import numpy as np

from .matern import covariance, distance, matern


def num_tiles(n: int, nb: int) -> int:
    return -(-n // nb)


def tile_range(i: int, n: int, nb: int) -> tuple[int, int]:
    return i * nb, min(n, (i + 1) * nb)


def gen_tile(x, y, theta, m: int, k: int, nb: int, kernel: str = "matern") -> np.ndarray:
    """Sigma_ij = C(||s_i - s_j||; theta) for i in tile row m, j in tile column k."""
    n = x.shape[0]
    r0, r1 = tile_range(m, n, nb)
    c0, c1 = tile_range(k, n, nb)
    h = distance(x[r0:r1, None], y[r0:r1, None], x[None, c0:c1], y[None, c0:c1])
    return covariance(h, theta, kernel)


def gen_lower_tiles(x, y, theta, nb: int, kernel: str = "matern") -> dict:
    """All lower tiles {(m, k): ndarray} of Sigma(theta)."""
    nt = num_tiles(x.shape[0], nb)
    return {(m, k): gen_tile(x, y, theta, m, k, nb, kernel) for k in range(nt) for m in range(k, nt)}


def dense_covariance(x, y, theta) -> np.ndarray:
    """The full n x n Sigma(theta) (small n only)."""
    sigma2, beta, nu = theta
    h = distance(x[:, None], y[:, None], x[None, :], y[None, :])
    return matern(h, sigma2, beta, nu)


def tile_sqnorm(t: np.ndarray) -> float:
    """s = ||t||_F^2 as the correctly rounded sum of the squares (reading O4)."""
    return math.fsum((t * t).ravel().tolist())


def tile_sqnorms(tiles: dict, nt: int) -> np.ndarray:
    """NT x NT array, s[m, k] = ||A_mk||_F^2 for m >= k, 0 above the diagonal."""
    s = np.zeros((nt, nt), dtype=np.float64)
    for (m, k), t in tiles.items():
        s[m, k] = tile_sqnorm(t)
    return s


def global_sqnorm(s: np.ndarray) -> float:
    """S = ||A||_F^2 of the whole symmetric matrix (reading C8): fsum(s_kk) + 2*fsum(s_mk, m>k)."""
    nt = s.shape[0]
    diag = math.fsum(float(s[k, k]) for k in range(nt))
    off = math.fsum(float(s[m, k]) for k in range(nt) for m in range(k + 1, nt))
    return diag + 2.0 * off


def assemble(tiles: dict, n: int, nb: int) -> np.ndarray:
    """Dense lower-triangular-tile matrix from a tile dict (upper tiles zero)."""
    out = np.zeros((n, n), dtype=np.float64)
    for (m, k), t in tiles.items():
        r0, r1 = tile_range(m, n, nb)
        c0, c1 = tile_range(k, n, nb)
        out[r0:r1, c0:c1] = t
    return out
