"""Pins for oracle/precision.py: the tile rule, storage map, Algorithm 2."""
import numpy as np
import pytest

import synth
from oracle import FP16, FP32, FP64
from oracle.precision import (COMM_AUTO, COMM_TTC, all_fp64_maps, band_map, comm_map, extreme_map,
                              kernel_map, precision_maps, storage_map)
from oracle.tiles import gen_lower_tiles, global_sqnorm, num_tiles, tile_sqnorms

import os

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "map_handbuilt.txt")


def load_handbuilt():
    nt = 4
    s = np.zeros((nt, nt))
    expect = {}
    for line in open(GOLDEN):
        if line.startswith("#") or not line.strip():
            continue
        m, k, v, e = line.split()[:4]
        s[int(m), int(k)] = float.fromhex(v)
        expect[int(m), int(k)] = int(e)
    s[0, 0] = 14.0 - 2.0**-12 - 2.0**-29 - 2.0**-39
    return s, expect


def test_handbuilt_map():
    s, expect = load_handbuilt()
    assert global_sqnorm(s) == 16.0
    km = kernel_map(s, 2.0**-30)
    for k in range(4):
        assert km[k, k] == FP64
    for (m, k), e in expect.items():
        assert km[m, k] == e, (m, k, km[m, k], e)


def small_norms(beta=0.03, n=4096, nb=256):
    x, y = synth.locations(n, 0)
    tiles = gen_lower_tiles(x, y, (1.0, beta, 0.5), nb)
    return tile_sqnorms(tiles, num_tiles(n, nb))


def test_rule_invariants_on_matern():
    s = small_norms()
    nt = s.shape[0]
    prev = None
    for u in [1e-12, 1e-9, 1e-6, 1e-3]:
        km = kernel_map(s, u)
        assert all(km[k, k] == FP64 for k in range(nt))
        if prev is not None:  # monotone: a looser u_req never raises a tile's precision
            for k in range(nt):
                for m in range(k, nt):
                    assert km[m, k] >= prev[m, k]
        prev = km
    km = kernel_map(s, 1e-9)
    assert {FP64, FP32, FP16} <= set(np.unique(km[np.tril_indices(nt, -1)]).tolist())


def test_storage_map():
    s = small_norms()
    km = kernel_map(s, 1e-9)
    sm = storage_map(km)
    nt = s.shape[0]
    for k in range(nt):
        for m in range(k, nt):
            assert sm[m, k] == (FP64 if km[m, k] == FP64 else FP32)


def test_comm_all_fp64():
    nt = 6
    km = all_fp64_maps(nt)[0]
    cm = comm_map(km, COMM_AUTO)
    for k in range(nt):
        for m in range(k + 1, nt):
            assert cm[m, k] == FP64
        if k < nt - 1:
            assert cm[k, k] == FP64
    assert cm[nt - 1, nt - 1] == FP32  # Alg. 2 line 7 literal; the last POTRF has no consumer


def test_comm_extreme_map_all_stc():
    """with FP64 diagonal / FP16(_32) off-diagonal 'all communications can employ STC'."""
    nt = 7
    cm = comm_map(extreme_map(nt, FP16), COMM_AUTO)
    for k in range(nt):
        assert cm[k, k] == FP32  # POTRF sends below its FP64 kernel precision
        for m in range(k + 1, nt):
            assert cm[m, k] == FP16  # below storage FP32: sender-side conversion


def test_comm_ttc_policy():
    s = small_norms()
    km, sm, cm = precision_maps(s, 1e-9, policy=COMM_TTC)
    nt = s.shape[0]
    for k in range(nt):
        assert cm[k, k] == FP64
        for m in range(k + 1, nt):
            assert cm[m, k] == sm[m, k]


def test_comm_handbuilt_successors():
    # NT = 4: tile (2,0) is FP16; its successors are GEMM(2,1,0) (kernel(2,1)) and GEMM(3,2,0) (kernel(3,2))
    km = extreme_map(4, FP16)
    cm = comm_map(km)
    assert cm[2, 0] == FP16
    km[3, 2] = FP32  # a column-broadcast successor runs in FP32 -> TTC at storage FP32
    assert comm_map(km)[2, 0] == FP32
    km = extreme_map(4, FP16)
    km[2, 1] = FP64  # row-broadcast successor FP64 -> capped at storage (FP32)
    assert comm_map(km)[2, 0] == FP32
    km = extreme_map(4, FP16)
    km[1, 0] = FP64  # TRSM(1,0) runs FP64 -> POTRF(0,0) must send FP64
    assert comm_map(km)[0, 0] == FP64 and comm_map(km)[1, 1] == FP32
    # comm never exceeds storage and never undercuts the tile's own kernel precision
    s = small_norms(0.03)
    km, sm, cm = precision_maps(s, 1e-9)
    nt = s.shape[0]
    for k in range(nt):
        for m in range(k + 1, nt):
            assert sm[m, k] <= cm[m, k] <= km[m, k]


def test_band_map():
    s = small_norms(0.1)
    bm = band_map(s, 1e-9)
    nt = s.shape[0]
    two = kernel_map(s, 1e-9, (2.0**-52, 2.0**-23, 1e300))
    for k in range(nt):
        for m in range(k, nt):
            if two[m, k] == FP64:
                assert bm[m, k] == FP64
    assert set(np.unique(bm[np.tril_indices(nt)]).tolist()) <= {FP64, FP32}


# ---------------------------------------------------------------- four-level maps
GOLDEN4 = os.path.join(os.path.dirname(__file__), "golden", "map4_handbuilt.txt")
EPS4_GOLDEN = (2.0**-52, 2.0**-23, 2.0**-13, 2.0**-10)


def load_handbuilt4():
    nt = 4
    s = np.zeros((nt, nt))
    expect = {}
    for line in open(GOLDEN4):
        if line.startswith("#") or not line.strip():
            continue
        m, k, v, e = line.split()[:4]
        s[int(m), int(k)] = float.fromhex(v)
        expect[int(m), int(k)] = int(e)
    s[0, 0] = 14.0 - 2.0**-13 - 2.0**-33 - 2.0**-35 - 2.0**-39 - 2.0**-49
    return s, expect


def test_handbuilt_map_four_levels():
    from oracle import FP16H
    s, expect = load_handbuilt4()
    assert global_sqnorm(s) == 16.0
    km = kernel_map(s, 2.0**-30, EPS4_GOLDEN)
    for k in range(4):
        assert km[k, k] == FP64
    for (m, k), e in expect.items():
        assert km[m, k] == e, (m, k, km[m, k], e)
    assert sorted(set(expect.values())) == [FP64, FP32, FP16, FP16H]  # every class appears


def test_four_level_refines_three_level():
    """Invariants of the four-level rule on Matérn norms: a tile is FP16 (pure) only if the three-level rule
    with the same FP16 epsilon already makes it FP16(_32); FP64 / FP32 are unchanged; with
    eps[FP16_32] = eps[FP16] the FP16_32 band is empty; storage is FP32 for every non-FP64 class; Algorithm 2
    gives an FP16H tile's successors FP16 data (no comm code above FP16)."""
    from oracle import FP16H
    s = small_norms(0.03, 4096, 256)
    u = 1e-9
    k3 = kernel_map(s, u, (2.0**-52, 2.0**-23, 2.0**-10))
    k4 = kernel_map(s, u, (2.0**-52, 2.0**-23, 2.0**-13, 2.0**-10))
    nt = s.shape[0]
    low = np.tril(np.ones((nt, nt), bool), -1)
    assert np.array_equal(k4[low] == FP64, k3[low] == FP64)
    assert np.array_equal(k4[low] == FP16H, k3[low] == FP16)
    assert ((k4[low] == FP16) <= (k3[low] == FP32)).all()
    assert (k4[low] == FP16).any() and (k4[low] == FP16H).any()
    same = kernel_map(s, u, (2.0**-52, 2.0**-23, 2.0**-10, 2.0**-10))
    assert not (same[low] == FP16).any()
    sm = storage_map(k4)
    assert np.array_equal(sm[low] == FP64, k4[low] == FP64) and set(np.unique(sm[low])) <= {FP64, FP32}
    cm = comm_map(k4)
    assert int(cm[np.tril(np.ones((nt, nt), bool))].max()) <= FP16
    # an all-FP16H map behaves like the extreme FP16 map for communication: every tile STC in FP16
    ext = extreme_map(nt, FP16H)
    ce = comm_map(ext)
    for k in range(nt - 1):
        for m in range(k + 1, nt):
            assert ce[m, k] == FP16
