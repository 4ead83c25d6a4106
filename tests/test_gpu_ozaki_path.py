"""All FP64-class engines — CRT modular emulation (MPGEO_OZAKI=16) and the 8-slice Ozaki split
(MPGEO_OZAKI=8), both on INT8 tensor cores, and DMMA FP64 (MPGEO_OZAKI=0) — must meet the all-FP64 tolerances: residual <= 1e-13, l relative error <= 1e-10."""
import os

import numpy as np
import pytest

import synth
from oracle.cholesky import residual
from oracle.loglik import loglik as oracle_loglik
from oracle.precision import all_fp64_maps
from oracle.tiles import num_tiles
from tests.gpu_helpers import to_dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", params=["16", "16t", "16f", "8", "0"],
                ids=["crt", "crt-tf32x3", "crt-f16x3", "ozaki", "dmma"])
def engine_handle(request):
    """crt: CRT FP64 class + CRT-8 FP32 class (MPGEO_CRT32=1); crt-tf32x3: CRT FP64 class + 3xTF32
    (MPGEO_F16X3=0); crt-f16x3: CRT FP64 class + 3xFP16 (the default engines)."""
    import paper_conf_cluster_caoalgkb23_b200 as mp
    eng = request.param.rstrip("tf")
    os.environ["MPGEO_OZAKI"] = eng
    os.environ["MPGEO_CRT32"] = "0" if request.param[-1] in "tf" else "1"  # crt: the CRT-8 FP32 class (opt-in)
    os.environ["MPGEO_F16X3"] = "0" if request.param.endswith("t") else "1"
    try:
        h = mp.Handle(0)
    finally:
        del os.environ["MPGEO_OZAKI"], os.environ["MPGEO_CRT32"], os.environ["MPGEO_F16X3"]
    oz = h.config()["ozaki"]
    assert oz % 100 == int(eng)
    assert (oz >= 200) == (request.param == "16")
    return h


@pytest.mark.parametrize("n,nb,theta", [(4900, 512, (1.0, 0.1, 0.5)), (8192, 1024, (1.0, 0.3, 0.5)),
                                         (3600, 512, (1.2, 0.05, 1.5))])
def test_fp64_path_engines(engine_handle, n, nb, theta):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    x, y = synth.locations(n, 0) if int(np.sqrt(n)) ** 2 == n else synth.uniform_locations(n, 0)
    z = synth.normal_vector(n, 1)
    nt = num_tiles(n, nb)
    M = mp.Matrix(engine_handle, n, nb, None)
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
    assert abs(r.loglik - ref["loglik"]) <= 1e-8 * abs(ref["loglik"])
