"""Parity at BASELINE.json's full single-GPU size (config 3: n = 160,000, nb = 2048), in the launch
configuration bench.py times (mp_eval, adaptive map, lookahead, default engines).  The oracle cannot
factor n = 160,000 on the host, so the checks are (a) sampled outputs the oracle computes one by
one (covariance entries, whole-tile norms incl. the ragged tile) and (b) properties that hold at any
size: the Kac-Murdock-Szego closed form of l at n = 160,000 (FP64 map <= 1e-10, adaptive MP map
<= 1e-5), the map is the rule applied to the norms, and MP vs FP64 agree to the north-star 1e-5."""
import math

import numpy as np
import pytest

import synth
from oracle.matern import distance, matern
from oracle.precision import precision_maps
from oracle.tiles import gen_tile, tile_sqnorm
from tests.gpu_helpers import to_dev

pytestmark = pytest.mark.gpu

N, NB = 160000, 2048


@pytest.fixture(scope="module")
def ev():
    import paper_conf_cluster_caoalgkb23_b200 as mp
    return mp.Evaluator(N, NB)


def test_config3_sampled_generation_and_norms(ev):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    theta = (1.0, 0.03, 0.5)
    x, y = synth.locations(N, 0)
    M = ev.M
    s = M.matern_gen(to_dev(x), to_dev(y), theta)
    nt = M.nt
    # whole-tile norms for a sample of tiles, including the ragged last row/column
    for (m, k) in [(0, 0), (5, 3), (nt - 1, 0), (nt - 1, nt - 1), (40, 39), (77, 12)]:
        ref = tile_sqnorm(gen_tile(x, y, theta, m, k, NB))
        assert abs(s[m, k] - ref) <= 1e-13 * ref, (m, k)
    # the maps are the rule applied to these norms (oracle rule = library rule, bit for bit)
    km, sm, cm = mp.precision_map(s, 1e-9)
    okm, osm, ocm = precision_maps(s, 1e-9)
    low = np.tril(np.ones((nt, nt), bool))
    assert np.array_equal(km[low], okm[low]) and np.array_equal(cm[low], ocm[low])
    # sampled covariance entries after the storage-precision write (workspace sized for this map)
    if M.bytes_for(sm) > M.nbytes:
        M.attach(M.bytes_for(sm))
    M.bind(sm)
    M.matern_gen(to_dev(x), to_dev(y), theta, sm)
    rng = np.random.default_rng(5)
    for _ in range(12):
        k = int(rng.integers(0, nt))
        m = int(rng.integers(k, nt))
        t = M.tile(m, k)
        i = int(rng.integers(0, min(NB, N - m * NB)))
        j = int(rng.integers(0, min(NB, N - k * NB)))
        gi, gj = m * NB + i, k * NB + j
        h = float(distance(x[gi], y[gi], x[gj], y[gj]))
        ref = float(matern(np.array([h]), *theta)[0])
        tol = 2.3e-16 * (2 + h / theta[1]) * abs(ref)  # exp(-r): r = h/beta carries one rounding
        if sm[m, k] == 1:  # FP32-stored tile: one more rounding (to nearest FP32)
            ref = float(np.float32(ref))
            tol = max(tol, 2.0**-24 * abs(ref))
        assert abs(t[i, j] - ref) <= tol + 1e-300, (m, k, i, j, t[i, j], ref)


def test_config3_kms_closed_form_fp64_and_adaptive(ev):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    delta, beta, sigma2 = 1.0 / N, 0.0005, 1.0
    x, y = synth.collinear_locations(N, delta)
    z = synth.normal_vector(N, 9)
    rho = math.exp(-delta / beta)
    ld = N * math.log(sigma2) + (N - 1) * math.log(1 - rho * rho)
    q = (z[0] ** 2 + z[-1] ** 2 + (1 + rho * rho) * float(np.sum(z[1:-1] ** 2))
         - 2 * rho * float(np.sum(z[:-1] * z[1:]))) / (sigma2 * (1 - rho * rho))
    ll = -0.5 * N * math.log(2 * math.pi) - 0.5 * ld - 0.5 * q
    dx, dy, dz = to_dev(x), to_dev(y), to_dev(z)
    r64 = ev.eval(dx, dy, dz, (sigma2, beta, 0.5), mode=mp.MP_MAP_FP64)
    assert abs(r64.loglik - ll) <= 1e-10 * abs(ll)
    rmp = ev.eval(dx, dy, dz, (sigma2, beta, 0.5), u_req=1e-9)
    assert rmp.tiles[1] + rmp.tiles[2] > 0
    assert abs(rmp.loglik - ll) <= 1e-5 * abs(ll)


def test_config3_mp_vs_fp64(ev):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    theta = (1.0, 0.03, 0.5)
    x, y = synth.locations(N, 0)
    z = synth.normal_vector(N, 1)
    dx, dy, dz = to_dev(x), to_dev(y), to_dev(z)
    rmp = ev.eval(dx, dy, dz, theta, u_req=1e-9)
    r64 = ev.eval(dx, dy, dz, theta, mode=mp.MP_MAP_FP64)
    assert rmp.tiles[1] + rmp.tiles[2] > 0
    assert abs(rmp.loglik - r64.loglik) <= 1e-5 * abs(r64.loglik)
    assert abs(rmp.loglik - r64.loglik) <= 1e-8 * abs(r64.loglik)  # regression bound
