"""theta recovery (north star: MP estimates within 1e-3 of the FP64 estimates on the same data, same
optimiser and start).  Z = L(theta_true) e with L from the CPU oracle's dense factor."""
import numpy as np
import pytest

import synth
from oracle.tiles import dense_covariance

pytestmark = pytest.mark.gpu


def test_theta_mp_vs_fp64():
    import paper_conf_cluster_caoalgkb23_b200 as mp
    from paper_conf_cluster_caoalgkb23_b200.mle import fit
    from tests.gpu_helpers import to_dev

    n, nb = 6400, 512
    theta_true = (1.0, 0.03, 0.5)
    x, y = synth.locations(n, 7)
    L = np.linalg.cholesky(dense_covariance(x, y, theta_true))
    z = L @ synth.normal_vector(n, 8)
    ev = mp.Evaluator(n, nb)
    dx, dy, dz = to_dev(x), to_dev(y), to_dev(z)
    r64 = fit(ev, dx, dy, dz, mode=mp.MP_MAP_FP64, maxfev=400)
    rmp = fit(ev, dx, dy, dz, mode=mp.MP_MAP_ADAPTIVE, u_req=1e-9, maxfev=400)
    rep = ev.eval(x, y, z, tuple(rmp.theta))
    assert rep.tiles[1] + rep.tiles[2] > 0, "the adaptive map should use low precision here"
    print("FP64", r64.theta, r64.nfev, "MP", rmp.theta, rmp.nfev)
    assert np.max(np.abs(rmp.theta - r64.theta)) <= 1e-3
    # the estimate is statistically close to the truth (loose: one realisation)
    assert abs(r64.theta[1] - theta_true[1]) < 0.02 and abs(r64.theta[2] - theta_true[2]) < 0.2
