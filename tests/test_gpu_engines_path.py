"""Every engine combination of mp_config must meet the all-FP64 tolerances through the whole path
(residual <= 1e-13, l relative error <= 1e-10 vs the oracle's FP64 definition) and the MP regression
bound (l <= 1e-8 vs the FP64 oracle at u_req = 1e-9):
  crt-f16x3  FP64 class CRT-16 on INT8 tcgen05 + FP32 class 3xFP16 (the defaults, C13c);
  crt-tf32x3 FP64 class CRT-16 + FP32 class 3xTF32 (reading C13);
  crt-ref    FP64 class CRT-16, FP32/FP16 classes on DMMA with rounded operands, FP64 TRSM everywhere;
  dmma       FP64 class on DMMA (native FP64), default FP32/FP16 classes;
  nolook     the defaults without the panel lookahead (one stream, strict Algorithm 1 order)."""
import numpy as np
import pytest

import synth
from oracle.cholesky import residual
from oracle.loglik import loglik as oracle_loglik
from oracle.precision import all_fp64_maps
from oracle.tiles import num_tiles
from tests.gpu_helpers import to_dev

pytestmark = pytest.mark.gpu

CONFIGS = {
    "crt-f16x3": {},
    "crt-tf32x3": {"fp32_engine": 1},
    "crt-ref": {"fp32_engine": 2, "fp16_tensor": 0, "lowp_trsm_product": 0},
    "dmma": {"fp64_engine": 1},
    "nolook": {"lookahead": 0},
}


@pytest.fixture(scope="module", params=list(CONFIGS), ids=list(CONFIGS))
def engine_handle(request):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    h = mp.Handle(0, config=CONFIGS[request.param])
    cfg = h.config()
    for k, v in CONFIGS[request.param].items():
        assert cfg[k] == v
    return h


@pytest.mark.parametrize("n,nb,theta", [(4900, 512, (1.0, 0.1, 0.5)), (8192, 1024, (1.0, 0.3, 0.5)),
                                         (3600, 512, (1.2, 0.05, 1.5))])
def test_fp64_path_engines(engine_handle, n, nb, theta):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    x, y = synth.locations(n, 0) if int(np.sqrt(n)) ** 2 == n else synth.uniform_locations(n, 0)
    z = synth.normal_vector(n, 1)
    nt = num_tiles(n, nb)
    M = mp.Matrix(engine_handle, n, nb, None)
    eng = M.engines()
    cfg = engine_handle.config()
    assert eng["fp64"] == cfg["fp64_engine"] and eng["fp32"] == cfg["fp32_engine"]  # nb % 256 == 0 here
    dx, dy, dz = to_dev(x), to_dev(y), to_dev(z)
    km, sm, cm = all_fp64_maps(nt)
    M.matern_gen(dx, dy, theta, sm)
    assert M.potrf(km, cm) == 0
    ll, ld, q = M.loglik(dz)
    ref = oracle_loglik(x, y, z, theta, nb)
    res = residual(ref["tiles"], {key: M.tile(*key)[: t.shape[0], : t.shape[1]] for key, t in ref["tiles"].items()},
                   n, nb)
    assert res <= 1e-13, res
    assert abs(ll - ref["loglik"]) <= 1e-10 * abs(ref["loglik"])


def test_mixed_precision_path_engines(engine_handle):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    n, nb, theta = 10000, 512, (1.0, 0.03, 0.5)
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ref = oracle_loglik(x, y, z, theta, nb)
    ev = mp.Evaluator(n, nb, handle=engine_handle)
    r = ev.eval(x, y, z, theta, u_req=1e-9)
    assert r.tiles[1] > 0 and r.tiles[2] > 0  # all three classes present
    assert abs(r.loglik - ref["loglik"]) <= 1e-8 * abs(ref["loglik"])


def test_engines_fall_back_when_nb_not_multiple_of_256():
    """the engines a matrix reports follow nb (C1's nb = 400 runs DMMA everywhere)."""
    import paper_conf_cluster_caoalgkb23_b200 as mp
    h = mp.Handle(0)
    M = mp.Matrix(h, 1600, 400, None)
    e = M.engines()
    assert e == {"fp64": mp.MP_F64_DMMA, "fp32": mp.MP_F32_DMMA, "fp16_tensor": 0, "lowp_trsm_product": 0}
    M2 = mp.Matrix(h, 4096, 512, None)
    assert M2.engines() == {"fp64": mp.MP_F64_CRT16, "fp32": mp.MP_F32_3XFP16, "fp16_tensor": 1,
                            "lowp_trsm_product": 1}
