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


def test_config_defaults_and_unique_id_on_cpu():
    """mp_config_default fills the documented defaults (include/mpgeo.h); mp_get_unique_id gives 128
    bytes with fresh randomness per call and this host's name (no GPU needed for either)."""
    import socket
    import paper_conf_cluster_caoalgkb23_b200 as mp
    cfg = mp.default_config()
    assert cfg == {"fp64_engine": mp.MP_F64_CRT16, "fp32_engine": mp.MP_F32_3XFP16, "fp16_tensor": 1, "lookahead": 1,
                   "reserve_pairs": 6, "lowp_trsm_product": 1, "matern_table": 1, "f16x3_persistent": 0,
                   "crt_phase_lock": 1, "fp16_storage": 0}
    a, b = mp.unique_id(), mp.unique_id()
    assert len(a) == len(b) == 128 and a != b and a[:32] != b[:32]
    assert a[48:48 + len(socket.gethostname().encode()[:79])] == socket.gethostname().encode()[:79]


def test_multirank_init_requires_the_communicator_id():
    """nranks > 1 without the id of mp_get_unique_id is an argument error (checked before any CUDA call)."""
    import ctypes as C
    from paper_conf_cluster_caoalgkb23_b200._lib import lib, MP_ERR_ARG
    h = C.c_void_p()
    assert lib.mp_init(0, 0, 2, 1, 2, None, None, C.byref(h)) == MP_ERR_ARG
    assert lib.mp_init(0, 0, 16, 4, 4, None, None, C.byref(h)) != 0  # more ranks than MAX_PEERS


@pytest.mark.parametrize("beta,u_req,policy", [(0.03, 1e-9, 1), (0.1, 1e-9, 1), (0.03, 1e-6, 0)])
def test_precision_map4_bit_exact_vs_oracle(beta, u_req, policy):
    from paper_conf_cluster_caoalgkb23_b200 import MP_EPS_FP16_32, precision_map
    s = _matern_norms(6400, 256, beta)
    eps4 = (2.0**-52, 2.0**-23, MP_EPS_FP16_32, 2.0**-10)
    km, sm, cm = precision_map(s, u_req, policy=policy, levels=4)  # eps = NULL: the library default
    okm, osm, ocm = oprec.precision_maps(s, u_req, eps=eps4, policy=policy)
    nt = s.shape[0]
    low = np.tril(np.ones((nt, nt), bool))
    assert np.array_equal(km[low], okm[low])
    assert np.array_equal(sm[low], osm[low])
    assert np.array_equal(cm[low], ocm[low])


def test_precision_map4_handbuilt_golden():
    from paper_conf_cluster_caoalgkb23_b200 import precision_map
    from tests.test_oracle_precision import EPS4_GOLDEN, load_handbuilt4
    s, expect = load_handbuilt4()
    km, _, _ = precision_map(s, 2.0**-30, eps=EPS4_GOLDEN, levels=4)
    for (m, k), e in expect.items():
        assert km[m, k] == e
    # a three-level call rejects a user map holding the four-level class; the four-level call takes it
    from paper_conf_cluster_caoalgkb23_b200 import MpError
    user = km.copy()
    with pytest.raises(MpError):
        precision_map(None, kernel_prec=user)
    _, sm, cm = precision_map(None, kernel_prec=user, levels=4)
    assert sm[1, 0] == 1 and cm[1, 0] <= 2
