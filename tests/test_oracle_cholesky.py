"""Pins for oracle/cholesky.py + oracle/loglik.py (Alg. 1, Eq. (1)).

* Kac-Murdock-Szego: collinear equispaced points with nu = 1/2 give
  Sigma_ij = sigma^2 rho^|i-j|, rho = exp(-delta/beta), whose Cholesky factor,
  log-determinant and quadratic form have closed forms (any n, ragged tiles).
* mpmath brute force (50 digits) on random 2D points, n <= 48, general nu.
* residual ||A - L L^T||_F / ||A||_F <= 1e-13 on the config-1 matrix.
* non-SPD -> NotSPDError with the LAPACK 1-based global column.
"""
import math

import mpmath
import numpy as np
import pytest

import synth
from oracle.cholesky import NotSPDError, residual, tile_cholesky
from oracle.loglik import loglik, loglik_from_factor
from oracle.tiles import assemble, gen_lower_tiles, num_tiles, tile_range


def kms_closed_form(n, sigma2, rho, z):
    """Closed forms for Sigma = sigma^2 rho^|i-j| (1-based formulas in the docstring above)."""
    s = math.sqrt(sigma2)
    c = math.sqrt(1.0 - rho * rho)
    L = np.zeros((n, n))
    for i in range(n):
        L[i, 0] = s * rho**i
        for j in range(1, i + 1):
            L[i, j] = s * rho ** (i - j) * c
    logdet = n * math.log(sigma2) + (n - 1) * math.log(1.0 - rho * rho)
    quad = (z[0] ** 2 + z[-1] ** 2 + (1 + rho * rho) * float(np.sum(z[1:-1] ** 2))
            - 2 * rho * float(np.sum(z[:-1] * z[1:]))) / (sigma2 * (1 - rho * rho))
    ll = -0.5 * n * math.log(2 * math.pi) - 0.5 * logdet - 0.5 * quad
    return L, logdet, quad, ll


@pytest.mark.parametrize("n,nb,delta,beta", [(37, 8, 0.01, 0.05), (300, 64, 0.002, 0.1), (129, 32, 0.05, 0.03)])
def test_kms_closed_form(n, nb, delta, beta):
    sigma2 = 1.7
    x, y = synth.collinear_locations(n, delta)
    z = synth.normal_vector(n, 5)
    rho = math.exp(-delta / beta)
    Lref, ld_ref, q_ref, ll_ref = kms_closed_form(n, sigma2, rho, z)
    out = loglik(x, y, z, (sigma2, beta, 0.5), nb)
    L = np.tril(assemble(out["factor"], n, nb))
    assert np.max(np.abs(L - Lref)) <= 1e-13 * math.sqrt(sigma2)
    assert abs(out["logdet"] - ld_ref) <= 1e-12 * abs(ld_ref)
    assert abs(out["quad"] - q_ref) <= 1e-12 * abs(q_ref)
    assert abs(out["loglik"] - ll_ref) <= 1e-12 * abs(ll_ref)


def mp_loglik(x, y, z, theta):
    mpmath.mp.dps = 50
    sigma2, beta, nu = (mpmath.mpf(v) for v in theta)
    n = len(x)
    S = mpmath.matrix(n, n)
    for i in range(n):
        for j in range(n):
            h = mpmath.sqrt((mpmath.mpf(x[i]) - mpmath.mpf(x[j])) ** 2 + (mpmath.mpf(y[i]) - mpmath.mpf(y[j])) ** 2)
            if h == 0:
                S[i, j] = sigma2
            else:
                r = h / beta
                S[i, j] = sigma2 * 2 ** (1 - nu) / mpmath.gamma(nu) * r**nu * mpmath.besselk(nu, r)
    Z = mpmath.matrix([mpmath.mpf(v) for v in z])
    det = mpmath.det(S)
    sol = mpmath.lu_solve(S, Z)
    quad = sum(Z[i] * sol[i] for i in range(n))
    ll = -mpmath.mpf(n) / 2 * mpmath.log(2 * mpmath.pi) - mpmath.log(det) / 2 - quad / 2
    return float(ll), float(mpmath.log(det)), float(quad)


@pytest.mark.parametrize("theta,nb", [((1.0, 0.2, 0.5), 7), ((1.3, 0.15, 0.8), 16), ((0.7, 0.1, 1.5), 48)])
def test_mpmath_brute_force(theta, nb):
    n = 40
    x, y = synth.uniform_locations(n, seed=11)
    z = synth.normal_vector(n, 12)
    ll_ref, ld_ref, q_ref = mp_loglik(x, y, z, theta)
    out = loglik(x, y, z, theta, nb)
    assert abs(out["logdet"] - ld_ref) <= 1e-11 * max(1.0, abs(ld_ref))
    assert abs(out["quad"] - q_ref) <= 1e-11 * abs(q_ref)
    assert abs(out["loglik"] - ll_ref) <= 1e-11 * abs(ll_ref)


def test_residual_config1():
    n, nb = 1600, 400
    x, y = synth.locations(n, 0)
    tiles = gen_lower_tiles(x, y, (1.0, 0.1, 0.5), nb)
    fac = tile_cholesky(tiles, num_tiles(n, nb), nb)
    assert residual(tiles, fac, n, nb) <= 1e-13


def test_tile_factor_equals_dense_factor_ragged():
    n, nb = 529, 100
    x, y = synth.locations(n, 2)
    tiles = gen_lower_tiles(x, y, (1.0, 0.05, 1.0), nb)
    fac = tile_cholesky(tiles, num_tiles(n, nb), nb)
    a = assemble(tiles, n, nb)
    a = np.tril(a) + np.tril(a, -1).T
    ref = np.linalg.cholesky(a)
    assert np.max(np.abs(np.tril(assemble(fac, n, nb)) - ref)) <= 1e-13


def test_not_spd_reports_lapack_info():
    n, nb = 50, 16
    a = np.eye(n)
    a[37, 37] = -1.0
    tiles = {}
    for k in range(num_tiles(n, nb)):
        for m in range(k, num_tiles(n, nb)):
            r0, r1 = tile_range(m, n, nb)
            c0, c1 = tile_range(k, n, nb)
            tiles[m, k] = a[r0:r1, c0:c1].copy()
    with pytest.raises(NotSPDError) as e:
        tile_cholesky(tiles, num_tiles(n, nb), nb)
    assert e.value.info == 38


def test_loglik_from_factor_identity():
    # Sigma = I: l = -(n/2) log 2pi - |z|^2/2
    n, nb = 10, 4
    fac = {}
    for k in range(3):
        for m in range(k, 3):
            r0, r1 = tile_range(m, n, nb)
            c0, c1 = tile_range(k, n, nb)
            fac[m, k] = np.eye(n)[r0:r1, c0:c1]
    z = np.arange(n, dtype=float)
    ll, ld, q = loglik_from_factor(fac, z, 3, nb)
    assert ld == 0.0 and q == float(np.sum(z * z))
    assert ll == -0.5 * n * math.log(2 * math.pi) - 0.5 * q
