"""CPU pins of the test-side checkers in tests/gpu_helpers.py (they judge the GPU results, so they must
themselves be pinned): the tile-wise residual equals the oracle's dense residual, and the backward-error
bound accepts valid mixed-precision factors (the oracle's emulation) while rejecting corrupted ones."""
import numpy as np

import synth
from oracle.cholesky import residual, tile_cholesky
from oracle.loglik import loglik as oracle_loglik
from oracle.precision import all_fp64_maps, precision_maps
from oracle.tiles import gen_lower_tiles, num_tiles, tile_sqnorms
from tests.gpu_helpers import mp_backward_check, residual_tiles


def test_residual_tiles_equals_dense_residual():
    n, nb = 700, 128
    x, y = synth.locations(900, 0)
    x, y = x[:n], y[:n]
    tiles = gen_lower_tiles(x, y, (1.0, 0.1, 0.5), nb)
    nt = num_tiles(n, nb)
    fac = tile_cholesky(tiles, nt, nb)
    fac[3, 1] = fac[3, 1] * (1 + 1e-9)  # a non-trivial residual
    r0, r1 = residual(tiles, fac, n, nb), residual_tiles(tiles, fac, nt)
    assert r0 > 1e-11 and abs(r0 - r1) <= 1e-6 * r0


def test_backward_bound_accepts_emulated_mp_and_rejects_corruption():
    n, nb, theta = 2304, 256, (1.0, 0.03, 0.5)
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ref = oracle_loglik(x, y, z, theta, nb)
    nt = num_tiles(n, nb)
    s = tile_sqnorms(ref["tiles"], nt)
    km, sm, cm = precision_maps(s, 1e-9)
    assert {0, 1, 2} <= set(km[np.tril_indices(nt, -1)].tolist())
    emu = oracle_loglik(x, y, z, theta, nb, maps=(km, sm, cm))
    worst, _ = mp_backward_check(ref["tiles"], emu["factor"], ref["factor"], km, sm, cm, nt, nb, lowp_trsm=False,
                                  scaled_fp16=False)  # the emulation rounds FP16 operands plainly
    assert worst <= 1.0, worst
    # the FP64 factor passes the FP64 bound, and a relative 1e-6 error in one FP64-class tile does not
    k64, s64, c64 = all_fp64_maps(nt)
    worst64, _ = mp_backward_check(ref["tiles"], ref["factor"], ref["factor"], k64, s64, c64, nt, nb)
    assert worst64 <= 1.0
    bad = dict(ref["factor"])
    bad[5, 4] = bad[5, 4] * (1 + 1e-6)
    worst_bad, _ = mp_backward_check(ref["tiles"], bad, ref["factor"], k64, s64, c64, nt, nb)
    assert worst_bad > 1.0
