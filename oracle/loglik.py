"""Gaussian log-likelihood, Eq. (1) (§III-A).  Oracle: test infrastructure only.

    l(theta) = -(n/2) log(2 pi) - 1/2 log|Sigma(theta)| - 1/2 Z^T Sigma(theta)^{-1} Z

From the tile factor Sigma = L L^T (the paper does not spell out these steps):
    log|Sigma| = 2 * sum_i log L_ii                     (diagonal tiles, FP64)
    y = L^{-1} Z by tile forward substitution:
        y_k = L_kk^{-1} (z_k - sum_{j<k} L_kj y_j)
    Z^T Sigma^{-1} Z = y^T y
Reading C15: L is read at whatever precision it is stored in; all of this
arithmetic is FP64.  Sums over the n entries are correctly rounded (math.fsum).
"""
from __future__ import annotations

import math

import numpy as np
import scipy.linalg

from .cholesky import tile_cholesky
from .tiles import gen_lower_tiles, num_tiles, tile_range


def logdet(factor: dict, nt: int) -> float:
    """log|Sigma| = 2 sum log diag(L)."""
    return 2.0 * math.fsum(v for k in range(nt) for v in np.log(np.diag(factor[k, k])).tolist())


def forward_solve(factor: dict, z: np.ndarray, nt: int, nb: int) -> np.ndarray:
    """y = L^{-1} z by tiles."""
    n = z.shape[0]
    y = np.zeros(n, dtype=np.float64)
    for k in range(nt):
        r0, r1 = tile_range(k, n, nb)
        rhs = z[r0:r1].copy()
        for j in range(k):
            c0, c1 = tile_range(j, n, nb)
            rhs -= factor[k, j] @ y[c0:c1]
        y[r0:r1] = scipy.linalg.solve_triangular(factor[k, k], rhs, lower=True, check_finite=False)
    return y


def loglik_from_factor(factor: dict, z: np.ndarray, nt: int, nb: int) -> tuple[float, float, float]:
    """(l, log|Sigma|, Z^T Sigma^-1 Z) per Eq. (1)."""
    n = z.shape[0]
    ld = logdet(factor, nt)
    y = forward_solve(factor, z, nt, nb)
    q = math.fsum((y * y).tolist())
    ll = -0.5 * n * math.log(2.0 * math.pi) - 0.5 * ld - 0.5 * q
    return ll, ld, q


def loglik(x, y, z, theta, nb: int, maps=None, kernel: str = "matern") -> dict:
    """One full evaluation: generate tiles, factor (Alg. 1), Eq. (1).

    maps=None -> the FP64 definition; maps=(kernel, storage, comm) -> MP emulation."""
    n = x.shape[0]
    nt = num_tiles(n, nb)
    tiles = gen_lower_tiles(x, y, theta, nb, kernel)
    if maps is None:
        fac = tile_cholesky(tiles, nt, nb)
    else:
        kmap, _smap, cmap = maps
        fac = tile_cholesky(tiles, nt, nb, kernel=kmap, comm=cmap)
    ll, ld, q = loglik_from_factor(fac, z, nt, nb)
    return {"loglik": ll, "logdet": ld, "quad": q, "factor": fac, "tiles": tiles}
