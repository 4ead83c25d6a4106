"""C-ABI library: loads on a GPU-less host, exports every declared symbol, and its pure-host
entry points (mp_precision_map, the exact sum) match the oracle bit for bit."""
import math
import os
import re

import numpy as np
import pytest

import synth
from oracle import precision as oprec
from oracle.tiles import gen_lower_tiles, num_tiles, tile_sqnorms
from oracle import FP16

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    names = set()
    for hdr in ("mpgeo.h", "mpgeo_test.h"):
        txt = open(os.path.join(ROOT, "include", hdr)).read()
        txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
        names |= set(re.findall(r"\b(mp\w+)\s*\(", txt))
    return names


def test_library_loads_and_exports_every_declared_symbol():
    from paper_conf_cluster_caoalgkb23_b200._lib import lib
    syms = declared_symbols()
    assert {"mp_init", "mp_matern_gen", "mp_precision_map", "mp_tile_potrf", "mp_loglik", "mp_eval"} <= syms
    for s in syms:
        assert hasattr(lib, s), s
    assert b"sm_100a" in lib.mp_version()


def test_exact_sum_matches_fsum():
    from paper_conf_cluster_caoalgkb23_b200 import exact_sum
    rng = np.random.default_rng(0)
    for trial in range(20):
        v = rng.standard_normal(1000) * 10.0 ** rng.integers(-30, 30, 1000)
        v = np.abs(v) if trial % 2 else v
        assert exact_sum(v) == math.fsum(v.tolist())
    v = np.array([1.0, 1e100, 1.0, -1e100])
    assert exact_sum(v) == 2.0


def _matern_norms(n, nb, beta, nu=0.5, seed=0):
    x, y = synth.locations(n, seed)
    tiles = gen_lower_tiles(x, y, (1.0, beta, nu), nb)
    return tile_sqnorms(tiles, num_tiles(n, nb))


@pytest.mark.parametrize("beta,u_req,policy", [(0.03, 1e-9, 1), (0.1, 1e-9, 1), (0.03, 1e-6, 0), (0.3, 1e-4, 1)])
def test_precision_map_bit_exact_vs_oracle(beta, u_req, policy):
    from paper_conf_cluster_caoalgkb23_b200 import precision_map
    s = _matern_norms(6400, 256, beta)
    km, sm, cm = precision_map(s, u_req, policy=policy)
    okm, osm, ocm = oprec.precision_maps(s, u_req, policy=policy)
    nt = s.shape[0]
    low = np.tril(np.ones((nt, nt), bool))
    assert np.array_equal(km[low], okm[low])
    assert np.array_equal(sm[low], osm[low])
    assert np.array_equal(cm[low], ocm[low])


def test_precision_map_handbuilt_golden():
    from paper_conf_cluster_caoalgkb23_b200 import precision_map
    from tests.test_oracle_precision import load_handbuilt
    s, expect = load_handbuilt()
    km, _, _ = precision_map(s, 2.0**-30)
    for (m, k), e in expect.items():
        assert km[m, k] == e


def test_precision_map_user_maps_and_extreme_stc():
    from paper_conf_cluster_caoalgkb23_b200 import precision_map
    nt = 9
    ext = oprec.extreme_map(nt, FP16)
    km, sm, cm = precision_map(None, kernel_prec=ext)
    ocm = oprec.comm_map(ext)
    low = np.tril(np.ones((nt, nt), bool))
    assert np.array_equal(cm[low], ocm[low])
    assert all(cm[m, k] == FP16 for k in range(nt) for m in range(k + 1, nt))


def test_precision_map_rejects_bad_input():
    from paper_conf_cluster_caoalgkb23_b200 import precision_map, MpError
    with pytest.raises(MpError):
        precision_map(np.full((3, 3), -1.0))
    bad = oprec.extreme_map(4, FP16)
    bad[2, 2] = FP16  # diagonal must be FP64
    with pytest.raises(MpError):
        precision_map(None, kernel_prec=bad)
