"""Independent pins of the oracle parts the round-1 review found unpinned (CPU).

* tile_sqnorm / global_sqnorm (§V, readings C8/O4): against the dense ||A||_F^2 of the whole
  symmetric matrix, and against closed forms of the Kac-Murdock-Szego matrix
  Sigma_ij = sigma^2 rho^|i-j| (collinear equispaced points, nu = 1/2):
      diagonal tile of size b:   sigma^4 [ b + 2 q/(1-q) ((b-1) - q (1 - q^(b-1))/(1-q)) ],
      off-diagonal tile (rows [r0,r1) below columns [c0,c1)):
                                 sigma^4 q^(r0-c1+1) (1-q^R)(1-q^C)/(1-q)^2,
  with q = rho^2, R = r1-r0, C = c1-c0 (geometric sums, derived by hand; no tile loop).
* band_map (reading C21): hand-built norms with a known band b, checked on both sides (the band is
  neither too narrow nor too wide).
* storage_map: literal expected table for a literal kernel map.
* residual: a hand-computed 2 x 2 example (both triangles of A enter the norm).
"""
import math

import numpy as np
import pytest

import synth
from oracle import FP16, FP32, FP64
from oracle.cholesky import residual
from oracle.matern import matern
from oracle.precision import band_map, kernel_map, storage_map
from oracle.tiles import (dense_covariance, gen_lower_tiles, global_sqnorm, num_tiles, tile_range, tile_sqnorm,
                          tile_sqnorms)


@pytest.mark.parametrize("n,nb,theta", [(529, 100, (1.0, 0.05, 0.5)), (400, 64, (1.7, 0.2, 1.3))])
def test_tile_norms_sum_to_dense_frobenius(n, nb, theta):
    x, y = synth.locations(n, 3)
    tiles = gen_lower_tiles(x, y, theta, nb)
    s = tile_sqnorms(tiles, num_tiles(n, nb))
    a = dense_covariance(x, y, theta)
    dense = float(np.sum(a * a))
    assert abs(global_sqnorm(s) - dense) <= 1e-13 * dense
    # a diagonal tile counts both of its triangles: its norm is the dense diagonal block's
    r0, r1 = tile_range(1, n, nb)
    blk = a[r0:r1, r0:r1]
    assert abs(s[1, 1] - float(np.sum(blk * blk))) <= 1e-14 * s[1, 1]


def kms_tile_closed_form(sigma2, q, r0, r1, c0, c1):
    """sum over the tile of (sigma^2 rho^|i-j|)^2 = sigma^4 sum q^|i-j|, q = rho^2 (module docstring)."""
    s4 = sigma2 * sigma2
    if (r0, r1) == (c0, c1):
        b = r1 - r0
        return s4 * (b + 2.0 * q / (1.0 - q) * ((b - 1) - q * (1.0 - q ** (b - 1)) / (1.0 - q)))
    R, C = r1 - r0, c1 - c0
    return s4 * q ** (r0 - c1 + 1) * (1.0 - q**R) * (1.0 - q**C) / (1.0 - q) ** 2


@pytest.mark.parametrize("n,nb,delta,beta", [(300, 64, 0.002, 0.1), (130, 32, 0.01, 0.03)])
def test_tile_norms_kms_closed_form(n, nb, delta, beta):
    sigma2 = 1.3
    x, y = synth.collinear_locations(n, delta)
    theta = (sigma2, beta, 0.5)
    tiles = gen_lower_tiles(x, y, theta, nb)
    nt = num_tiles(n, nb)
    s = tile_sqnorms(tiles, nt)
    # rho^|i-j| with rho = exp(-delta/beta): the distance is |i-j| delta up to the rounding of i*delta
    q = math.exp(-2.0 * delta / beta)
    for k in range(nt):
        for m in range(k, nt):
            r0, r1 = tile_range(m, n, nb)
            c0, c1 = tile_range(k, n, nb)
            ref = kms_tile_closed_form(sigma2, q, r0, r1, c0, c1)
            assert abs(s[m, k] - ref) <= 1e-11 * ref, (m, k, s[m, k], ref)
    # the whole matrix: sigma^4 [n + 2 sum_{d=1}^{n-1} (n-d) q^d]
    ref = kms_tile_closed_form(sigma2, q, 0, n, 0, n)
    assert abs(global_sqnorm(s) - ref) <= 1e-11 * ref


def test_tile_sqnorm_is_correctly_rounded():
    # squares 1 and four times 2^-54: the exact sum 1 + 2^-52 is a double; a running float sum
    # would stay at 1 (each 1 + 2^-54 rounds back to 1)
    e = 2.0**-27
    assert tile_sqnorm(np.array([[1.0, e, e], [e, e, 0.0]])) == 1.0 + 2.0**-52
    # squares 2^54, 1, 1, 1: exact 2^54 + 3, correctly rounded to 2^54 + 4 (a running sum gives 2^54)
    assert tile_sqnorm(np.array([[2.0**27, 1.0], [1.0, 1.0]])) == 2.0**54 + 4.0


def test_band_map_handbuilt():
    """NT = 6, u_req = 2^-30 (thr32 = 2^-7): only tile (3,0) exceeds the FP32 threshold, so the
    narrowest band holding it is b = 4: FP64 iff m - k < 4."""
    nt = 6
    s = np.zeros((nt, nt))
    for k in range(nt):
        s[k, k] = 1024.0
    s[3, 0] = 1.0          # r = 1 * 6 / sqrt(6146) = 0.0765 > 2^-7: FP64 under the two-level rule
    s[5, 4] = 2.0**-40     # r ~ 7.7e-14: FP32
    s[4, 0] = 2.0**-40     # distance 4: must stay outside the band
    assert abs(global_sqnorm(s) - 6146.0) < 1e-9
    km = band_map(s, 2.0**-30)
    for k in range(nt):
        for m in range(k, nt):
            want = FP64 if m - k < 4 else FP32
            assert km[m, k] == want, (m, k, km[m, k])
    # moving the far tile one step further widens the band by one (not too narrow)
    s[3, 0], s[4, 0] = 2.0**-40, 1.0
    km = band_map(s, 2.0**-30)
    assert km[4, 0] == FP64 and km[5, 0] == FP32 and km[5, 1] == FP64
    # no FP64 tile off the diagonal: the band is the diagonal itself
    s[4, 0] = 2.0**-40
    km = band_map(s, 2.0**-30)
    assert all(km[m, k] == (FP64 if m == k else FP32) for k in range(nt) for m in range(k, nt))


def test_storage_map_literal():
    km = np.full((4, 4), 255, np.uint8)
    km[np.tril_indices(4)] = [FP64,
                              FP16, FP64,
                              FP32, FP64, FP64,
                              FP16, FP32, FP16, FP64]
    expect = np.full((4, 4), 255, np.uint8)
    expect[np.tril_indices(4)] = [FP64,
                                  FP32, FP64,
                                  FP32, FP64, FP64,
                                  FP32, FP32, FP32, FP64]
    assert np.array_equal(storage_map(km), expect)


def test_residual_handbuilt():
    """A = [[4, 2], [2, 5]] (tiles of size 1), L = [[2, 0], [1 + d, 2]]:
    L L^T - A = [[0, 2d], [2d, 2d + d^2]], ||A||_F = 7, so the residual is
    sqrt(8 d^2 + (2d + d^2)^2) / 7 (an A missing its upper triangle would give sqrt(45))."""
    tiles = {(0, 0): np.array([[4.0]]), (1, 0): np.array([[2.0]]), (1, 1): np.array([[5.0]])}
    exact = {(0, 0): np.array([[2.0]]), (1, 0): np.array([[1.0]]), (1, 1): np.array([[2.0]])}
    assert residual(tiles, exact, 2, 1) == 0.0
    d = 2.0**-20
    fac = dict(exact)
    fac[1, 0] = np.array([[1.0 + d]])
    ref = math.sqrt(8 * d * d + (2 * d + d * d) ** 2) / 7.0
    assert abs(residual(tiles, fac, 2, 1) - ref) <= 1e-15 * ref
    # an upper-triangle entry of a factor tile is ignored (L is lower triangular)
    fac[1, 1] = np.array([[2.0]])
    fac[0, 0] = np.array([[2.0]])
    big = {(0, 0): np.array([[4.0, 2.0], [2.0, 5.0]])}
    lbig = {(0, 0): np.array([[2.0, 123.0], [1.0, 2.0]])}
    assert residual(big, lbig, 2, 2) == 0.0


def test_kernel_map_rule_single_tile_by_hand():
    """One off-diagonal tile at a chosen ratio r = sqrt(s) NT / sqrt(S) on each side of both
    thresholds (u_req = 2^-30: thr16 = 2^-20, thr32 = 2^-7)."""
    nt = 2
    for r, want in [(2.0**-21, FP16), (2.0**-19, FP32), (2.0**-8, FP32), (2.0**-6, FP64)]:
        s = np.array([[1.0, 0.0], [0.0, 0.0]])
        # S = 1 + 2 s10 (s11 = 0); choose s10 = (r/2)^2 S -> s10 = r^2/4 (1 + 2 s10) -> s10 = r^2 / (4 - 2 r^2)
        s10 = r * r / (4.0 - 2.0 * r * r)
        s[1, 0] = s10
        km = kernel_map(s, 2.0**-30)
        assert km[1, 0] == want, (r, km[1, 0])
