"""MP-emulation mode of oracle/cholesky.py (prediction only; see oracle/__init__.py)."""
import numpy as np

import synth
from oracle.loglik import loglik
from oracle.precision import all_fp64_maps, extreme_map, comm_map, precision_maps, storage_map
from oracle.tiles import gen_lower_tiles, num_tiles, tile_sqnorms
from oracle import FP16


def test_all_fp64_emulation_is_the_definition():
    n, nb = 900, 128
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    th = (1.0, 0.1, 0.5)
    a = loglik(x, y, z, th, nb)
    b = loglik(x, y, z, th, nb, maps=all_fp64_maps(num_tiles(n, nb)))
    assert a["loglik"] == b["loglik"]


def test_adaptive_map_error_small_extreme_map_error_large():
    n, nb = 4096, 256
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    th = (1.0, 0.03, 0.5)
    ref = loglik(x, y, z, th, nb)
    s = tile_sqnorms(ref["tiles"], num_tiles(n, nb))
    mp = loglik(x, y, z, th, nb, maps=precision_maps(s, 1e-9))
    err = abs(mp["loglik"] - ref["loglik"]) / abs(ref["loglik"])
    assert err <= 1e-8  # survey-measured 5e-11 .. 7e-10 at u_req = 1e-9
    km = extreme_map(num_tiles(n, nb), FP16)
    ex = loglik(x, y, z, th, nb, maps=(km, storage_map(km), comm_map(km)))
    err_ex = abs(ex["loglik"] - ref["loglik"]) / abs(ref["loglik"])
    assert err_ex > err
