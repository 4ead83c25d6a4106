"""Config 2 of BASELINE.json at the bench tile size (n = 40,000 = 200^2, nb = 2048, NT = 20, ragged last
tile of 1088 rows) against the CPU oracle, through the C ABI (mp_eval), on the default engines:
  * all-FP64 map: factor entrywise <= 1e-12 sigma^2 vs the oracle's FP64 factor, residual <= 1e-13,
    l <= 1e-10 (north-star FP64 tolerances);
  * adaptive map (u_req = 1e-9): maps bit-exact vs the oracle's maps from its own tile norms (near-tie
    guard), l <= 1e-8 vs the FP64 oracle (north star 1e-5), backward error within the maps' bound;
  * band FP64/FP32 map (reading C21): map equal to the oracle's band map, l <= 1e-8;
  * extreme FP64/FP16 map under AUTO (all STC) and TTC: backward error within the bound.
The oracle at this size takes ~2-3 minutes on the GPU box's host cores (computed once per module)."""
import numpy as np
import pytest

import synth
from oracle import FP16
from oracle.loglik import loglik as oracle_loglik
from oracle.precision import all_fp64_maps, band_map, comm_map, extreme_map, precision_maps
from oracle.tiles import num_tiles, tile_sqnorms
from tests.gpu_helpers import mp_backward_check, near_tie_guard, residual_tiles

pytestmark = pytest.mark.gpu

N, NB, THETA, U_REQ = 40000, 2048, (1.0, 0.03, 0.5), 1e-9


@pytest.fixture(scope="module")
def c2():
    import torch
    assert torch.cuda.is_available()
    import paper_conf_cluster_caoalgkb23_b200 as mp
    x, y = synth.locations(N, 0)
    z = synth.normal_vector(N, 1)
    ref = oracle_loglik(x, y, z, THETA, NB)
    nt = num_tiles(N, NB)
    s = tile_sqnorms(ref["tiles"], nt)
    ev = mp.Evaluator(N, NB)
    assert ev.M.engines()["fp64"] == mp.MP_F64_CRT16  # the bench engines
    return {"mp": mp, "x": x, "y": y, "z": z, "ref": ref, "nt": nt, "s": s, "ev": ev}


def gpu_tiles(c):
    ref = c["ref"]
    return {key: c["ev"].M.tile(*key)[: t.shape[0], : t.shape[1]] for key, t in ref["tiles"].items()}


def test_c2_fp64_vs_oracle(c2):
    mp, ref, nt = c2["mp"], c2["ref"], c2["nt"]
    r = c2["ev"].eval(c2["x"], c2["y"], c2["z"], THETA, mode=mp.MP_MAP_FP64)
    L = gpu_tiles(c2)
    worst = max(float(np.max(np.abs(np.tril(L[key]) - np.tril(ref["factor"][key])))) for key in L)
    assert worst <= 1e-12 * THETA[0], worst
    res = residual_tiles(ref["tiles"], L, nt)
    assert res <= 1e-13, res
    assert abs(r.loglik - ref["loglik"]) <= 1e-10 * abs(ref["loglik"])
    assert abs(r.logdet - ref["logdet"]) <= 1e-10 * abs(ref["logdet"])


def test_c2_adaptive_maps_and_loglik(c2):
    mp, ref, nt, s = c2["mp"], c2["ref"], c2["nt"], c2["s"]
    near_tie_guard(s, nt, U_REQ)
    maps = precision_maps(s, U_REQ)
    r = c2["ev"].eval(c2["x"], c2["y"], c2["z"], THETA, u_req=U_REQ)
    km, sm, cm = c2["ev"].M.maps()
    low = np.tril(np.ones((nt, nt), bool))
    for g, o in zip((km, sm, cm), maps):
        assert np.array_equal(g[low], o[low])
    assert r.tiles[0] > 0 and r.tiles[1] > 0 and r.tiles[2] > 0
    assert abs(r.loglik - ref["loglik"]) <= 1e-8 * abs(ref["loglik"])
    worst, _ = mp_backward_check(ref["tiles"], gpu_tiles(c2), ref["factor"], km, sm, cm, nt, NB)
    assert worst <= 1.0, worst


def test_c2_band_map(c2):
    mp, ref, nt, s = c2["mp"], c2["ref"], c2["nt"], c2["s"]
    r = c2["ev"].eval(c2["x"], c2["y"], c2["z"], THETA, u_req=U_REQ, mode=mp.MP_MAP_BAND)
    km, sm, cm = c2["ev"].M.maps()
    low = np.tril(np.ones((nt, nt), bool))
    assert np.array_equal(km[low], band_map(s, U_REQ)[low])
    assert abs(r.loglik - ref["loglik"]) <= 1e-8 * abs(ref["loglik"])


@pytest.mark.parametrize("policy", ["auto", "ttc"])
def test_c2_extreme_map(c2, policy):
    mp, ref, nt = c2["mp"], c2["ref"], c2["nt"]
    pol = mp.MP_COMM_AUTO if policy == "auto" else mp.MP_COMM_TTC
    r = c2["ev"].eval(c2["x"], c2["y"], c2["z"], THETA, mode=mp.MP_MAP_EXTREME, policy=pol)
    km, sm, cm = c2["ev"].M.maps()
    low = np.tril(np.ones((nt, nt), bool))
    ekm = extreme_map(nt, FP16)
    assert np.array_equal(km[low], ekm[low]) and np.array_equal(cm[low], comm_map(ekm, pol)[low])
    assert r.stc_tiles == (nt * (nt - 1) // 2 if policy == "auto" else 0)
    worst, _ = mp_backward_check(ref["tiles"], gpu_tiles(c2), ref["factor"], km, sm, cm, nt, NB)
    assert worst <= 1.0, worst
    assert np.isfinite(r.loglik)
