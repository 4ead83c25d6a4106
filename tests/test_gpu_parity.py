"""Parity of the CUDA path (through the C ABI) against the CPU oracle.

Tolerances (BASELINE.json north_star):
  all-FP64: ||A - L L^T||_F / ||A||_F <= 1e-13, l relative error <= 1e-10;
  mixed precision: l relative error <= 1e-5 vs the FP64 oracle; precision maps bit-exact.
"""
import math

import numpy as np
import pytest

import synth
from oracle import FP16, FP64
from oracle.cholesky import residual, tile_cholesky
from oracle.loglik import loglik as oracle_loglik, loglik_from_factor
from oracle.precision import all_fp64_maps, comm_map, extreme_map, precision_maps, storage_map
from oracle.tiles import assemble, gen_lower_tiles, num_tiles, tile_range, tile_sqnorms
from tests.gpu_helpers import (gpu_factor_dense, loglik_perturbation_bound, mp_backward_check, near_tie_guard,
                               to_dev)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def mp():
    import torch
    assert torch.cuda.is_available(), "the -m gpu tests need a GPU"
    import paper_conf_cluster_caoalgkb23_b200 as mp
    return mp


@pytest.fixture(scope="module")
def handle(mp):
    return mp.Handle(0)


def stepwise(mp, handle, x, y, z, theta, nb, maps=None, u_req=1e-9):
    """gen pass 1 -> map -> bind -> gen pass 2 -> potrf -> loglik through the four ABI calls."""
    n = x.shape[0]
    M = mp.Matrix(handle, n, nb, None)
    dx, dy, dz = to_dev(x), to_dev(y), to_dev(z)
    s = M.matern_gen(dx, dy, theta)
    if maps is None:
        km, sm, cm = mp.precision_map(s, u_req)
    else:
        km, sm, cm = maps
    M.bind(sm)
    M.matern_gen(dx, dy, theta, sm)
    info = M.potrf(km, cm)
    assert info == 0
    ll = M.loglik(dz)
    return M, s, (km, sm, cm), ll


@pytest.mark.parametrize("n,nb,theta", [(1600, 400, (1.0, 0.1, 0.5)), (2500, 384, (1.3, 0.05, 0.8)),
                                         (900, 256, (0.7, 0.2, 1.5))])
def test_generation_tiles_and_norms(mp, handle, n, nb, theta):
    x, y = synth.locations(n, 0)
    M = mp.Matrix(handle, n, nb, None)
    dx, dy = to_dev(x), to_dev(y)
    s = M.matern_gen(dx, dy, theta)
    nt = num_tiles(n, nb)
    tiles = gen_lower_tiles(x, y, theta, nb)
    so = tile_sqnorms(tiles, nt)
    low = np.tril(np.ones((nt, nt), bool))
    assert np.max(np.abs(s[low] - so[low]) / so[low]) <= 1e-13
    M.matern_gen(dx, dy, theta, np.zeros((nt, nt), np.uint8))
    tol = 1e-15 if theta[2] == 0.5 else 2e-13
    for (m, k), t in tiles.items():
        g = M.tile(m, k)
        r = t.shape[0]
        c = t.shape[1]
        assert np.max(np.abs(g[:r, :c] - t)) <= tol * theta[0] * 4
        pad = g.copy()
        pad[:r, :c] = 0
        expect = np.zeros_like(pad)
        if m == k:
            for i in range(r, nb):
                expect[i, i] = 1.0
        assert np.array_equal(pad, expect)


def test_generation_fp32_storage(mp, handle):
    n, nb, theta = 1024, 256, (1.0, 0.05, 0.5)
    x, y = synth.locations(n, 4)
    M = mp.Matrix(handle, n, nb, None)
    nt = M.nt
    sm = np.full((nt, nt), 255, np.uint8)
    for k in range(nt):
        for m in range(k, nt):
            sm[m, k] = 0 if m == k else 1
    M.bind(sm)
    M.matern_gen(to_dev(x), to_dev(y), theta, sm)
    t = gen_lower_tiles(x, y, theta, nb)[3, 1]
    assert np.array_equal(M.tile(3, 1), t.astype(np.float32).astype(np.float64))


def test_map_from_gpu_norms_bit_exact(mp, handle):
    n, nb, u_req = 10000, 512, 1e-9
    x, y = synth.locations(n, 0)
    theta = (1.0, 0.03, 0.5)
    M = mp.Matrix(handle, n, nb, None)
    s = M.matern_gen(to_dev(x), to_dev(y), theta)
    so = tile_sqnorms(gen_lower_tiles(x, y, theta, nb), M.nt)
    near_tie_guard(so, M.nt, u_req)
    got = mp.precision_map(s, u_req)
    ref = precision_maps(so, u_req)
    low = np.tril(np.ones((M.nt, M.nt), bool))
    for g, r in zip(got, ref):
        assert np.array_equal(g[low], r[low])
    assert len(set(got[0][low].tolist())) == 3  # the case exercises all three classes


@pytest.mark.parametrize("n,nb,theta", [(1600, 400, (1.0, 0.1, 0.5)), (4900, 512, (1.0, 0.1, 0.5)),
                                         (3600, 1024, (1.5, 0.07, 1.0))])
def test_fp64_path_vs_oracle(mp, handle, n, nb, theta):
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    nt = num_tiles(n, nb)
    M, _, _, (ll, ld, q) = stepwise(mp, handle, x, y, z, theta, nb, maps=all_fp64_maps(nt))
    ref = oracle_loglik(x, y, z, theta, nb)
    L = gpu_factor_dense(M, n)
    Lo = np.tril(assemble(ref["factor"], n, nb))
    assert np.max(np.abs(L - Lo)) <= 1e-12 * theta[0]
    assert residual(ref["tiles"], {key: M.tile(*key)[: t.shape[0], : t.shape[1]] for key, t in ref["tiles"].items()},
                    n, nb) <= 1e-13
    assert abs(ll - ref["loglik"]) <= 1e-10 * abs(ref["loglik"])
    assert abs(ld - ref["logdet"]) <= 1e-10 * abs(ref["logdet"])
    assert abs(q - ref["quad"]) <= 1e-10 * abs(ref["quad"])


def test_config1_via_mp_eval_host_and_device_inputs(mp, handle):
    """Config 1 (BASELINE.json configs[0]): n=1600, 40x40 grid, theta=(1,0.1,0.5), tile 400, all FP64."""
    n, nb, theta = 1600, 400, (1.0, 0.1, 0.5)
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ref = oracle_loglik(x, y, z, theta, nb)
    ev = mp.Evaluator(n, nb, handle=handle)
    r1 = ev.eval(x, y, z, theta, mode=mp.MP_MAP_FP64)
    r2 = ev.eval(to_dev(x), to_dev(y), to_dev(z), theta, mode=mp.MP_MAP_FP64)
    r3 = ev.eval(x, y, z, theta, mode=mp.MP_MAP_ADAPTIVE)  # the rule also gives all FP64 here
    assert r1.loglik == r2.loglik == r3.loglik  # deterministic, input location irrelevant
    assert abs(r1.loglik - ref["loglik"]) <= 1e-10 * abs(ref["loglik"])
    assert r3.tiles[1] == 0 and r3.tiles[2] == 0
    assert r1.gpu_launches > 0


def test_kms_closed_form_large(mp, handle):
    from tests.test_oracle_cholesky import kms_closed_form
    n, nb, delta, beta, sigma2 = 12000, 1024, 1e-4, 0.02, 1.2
    x, y = synth.collinear_locations(n, delta)
    z = synth.normal_vector(n, 3)
    rho = math.exp(-delta / beta)
    ld_ref = n * math.log(sigma2) + (n - 1) * math.log(1 - rho * rho)
    q_ref = (z[0] ** 2 + z[-1] ** 2 + (1 + rho * rho) * float(np.sum(z[1:-1] ** 2))
             - 2 * rho * float(np.sum(z[:-1] * z[1:]))) / (sigma2 * (1 - rho * rho))
    ll_ref = -0.5 * n * math.log(2 * math.pi) - 0.5 * ld_ref - 0.5 * q_ref
    ev = mp.Evaluator(n, nb, handle=handle)
    r = ev.eval(x, y, z, (sigma2, beta, 0.5), mode=mp.MP_MAP_FP64)
    assert abs(r.logdet - ld_ref) <= 1e-10 * abs(ld_ref)
    assert abs(r.quad - q_ref) <= 1e-10 * abs(q_ref)
    assert abs(r.loglik - ll_ref) <= 1e-10 * abs(ll_ref)


@pytest.mark.parametrize("beta", [0.03, 0.1])
def test_mixed_precision_path(mp, handle, beta):
    n, nb, u_req = 10000, 512, 1e-9
    theta = (1.0, beta, 0.5)
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ref = oracle_loglik(x, y, z, theta, nb)
    nt = num_tiles(n, nb)
    so = tile_sqnorms(ref["tiles"], nt)
    near_tie_guard(so, nt, u_req)
    maps = precision_maps(so, u_req)
    ev = mp.Evaluator(n, nb, handle=handle)
    r = ev.eval(x, y, z, theta, u_req=u_req)
    km, sm, cm = ev.M.maps()
    low = np.tril(np.ones((nt, nt), bool))
    for g, o in zip((km, sm, cm), maps):
        assert np.array_equal(g[low], o[low])
    err = abs(r.loglik - ref["loglik"]) / abs(ref["loglik"])
    assert err <= 1e-5  # north-star MP tolerance
    assert err <= 1e-8  # regression bound (survey emulation: 5e-11 .. 7e-10)
    # the factor's backward error stays within the bound the maps imply (tests/gpu_helpers.py)
    Lhat = {key: ev.M.tile(*key)[: t.shape[0], : t.shape[1]] for key, t in ref["tiles"].items()}
    worst, _ = mp_backward_check(ref["tiles"], Lhat, ref["factor"], km, sm, cm, nt, nb)
    assert worst <= 1.0, worst


@pytest.mark.parametrize("beta", [0.03, 0.1])
def test_four_level_precision_path(mp, handle, beta):
    """Four-level maps (P:113 / P:117 "FP64, FP32, FP16_32, and FP16"; MP_MAP_ADAPTIVE4 with
    the library's default eps = (2^-52, 2^-23, MP_EPS_FP16_32, 2^-10)): maps bit-exact vs the oracle's
    four-level rule, pure-FP16 tiles present and run through the F16-accumulator kernel, l within the
    north-star 1e-5 of the FP64 oracle, and the factor's backward error within the bound the maps imply
    (FP16 accumulation unit 2^-11 for the pure-FP16 class, tests/gpu_helpers.py)."""
    from oracle import FP16H
    n, nb, u_req = 10000, 512, 1e-9
    theta = (1.0, beta, 0.5)
    eps4 = (2.0**-52, 2.0**-23, mp.MP_EPS_FP16_32, 2.0**-10)
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ref = oracle_loglik(x, y, z, theta, nb)
    nt = num_tiles(n, nb)
    so = tile_sqnorms(ref["tiles"], nt)
    near_tie_guard(so, nt, u_req, eps4)
    maps = precision_maps(so, u_req, eps=eps4)
    ev = mp.Evaluator(n, nb, handle=handle)
    r = ev.eval(x, y, z, theta, u_req=u_req, mode=mp.MP_MAP_ADAPTIVE4)
    km, sm, cm = ev.M.maps()
    low = np.tril(np.ones((nt, nt), bool))
    for g, o in zip((km, sm, cm), maps):
        assert np.array_equal(g[low], o[low])
    n16h = int((km[np.tril(np.ones((nt, nt), bool), -1)] == FP16H).sum())
    assert r.tiles_fp16h == n16h and (beta > 0.05 or n16h > 0)
    err = abs(r.loglik - ref["loglik"]) / abs(ref["loglik"])
    print(f"beta {beta}: tiles FP64/FP32/FP16_32/FP16 = {list(r.tiles)} + {r.tiles_fp16h}, l rel. error {err:.2e}")
    assert err <= 1e-5  # north-star MP tolerance
    Lhat = {key: ev.M.tile(*key)[: t.shape[0], : t.shape[1]] for key, t in ref["tiles"].items()}
    worst, _ = mp_backward_check(ref["tiles"], Lhat, ref["factor"], km, sm, cm, nt, nb)
    assert worst <= 1.0, worst


@pytest.mark.parametrize("beta", [0.03, 0.1])
def test_extreme_map_stc_and_ttc(mp, handle, beta):
    """P:294 extreme FP64/FP16 map: AUTO -> every communication STC; TTC keeps storage precision.
    Pass criteria (no emulation): the GPU factor's backward error per tile within the bound the maps
    imply, and l within the first-order perturbation bound of the FP64 oracle given that backward
    error (tests/gpu_helpers.py); STC may not be better than TTC by construction, so both are checked."""
    n, nb, theta = 4096, 512, (1.0, beta, 0.5)
    x, y = synth.locations(n, 2)
    z = synth.normal_vector(n, 1)
    nt = num_tiles(n, nb)
    ref = oracle_loglik(x, y, z, theta, nb)
    a = assemble(ref["tiles"], n, nb)
    a = np.tril(a) + np.tril(a, -1).T
    km = extreme_map(nt, FP16)
    ev = mp.Evaluator(n, nb, handle=handle)
    out = {}
    for pol in (mp.MP_COMM_AUTO, mp.MP_COMM_TTC):
        r = ev.eval(x, y, z, theta, mode=mp.MP_MAP_EXTREME, policy=pol)
        gk, gs, gc = ev.M.maps()
        assert np.array_equal(gc[np.tril_indices(nt)], comm_map(km, pol)[np.tril_indices(nt)])
        Lhat = {key: ev.M.tile(*key)[: t.shape[0], : t.shape[1]] for key, t in ref["tiles"].items()}
        worst, dA = mp_backward_check(ref["tiles"], Lhat, ref["factor"], gk, gs, gc, nt, nb)
        assert worst <= 1.0, (pol, worst)
        bound, rho = loglik_perturbation_bound(a, z, dA)
        assert rho < 1.0  # the perturbation bound applies
        assert abs(r.loglik - ref["loglik"]) <= bound, (pol, abs(r.loglik - ref["loglik"]), bound)
        out[pol] = r
    assert out[mp.MP_COMM_AUTO].stc_tiles == nt * (nt - 1) // 2
    assert out[mp.MP_COMM_TTC].stc_tiles == 0


def test_not_spd_reports_info(mp, handle):
    n, nb = 700, 256
    M = mp.Matrix(handle, n, nb, None)
    nt = M.nt
    a = np.eye(nt * nb)
    a[517, 517] = -2.0
    for k in range(nt):
        for m in range(k, nt):
            M.set_tile(m, k, a[m * nb:(m + 1) * nb, k * nb:(k + 1) * nb])
    km, sm, cm = all_fp64_maps(nt)
    assert M.potrf(km, cm) == 518


def test_user_matrix_factor_matches_lapack(mp, handle):
    """Factor a random SPD matrix given through mp_matrix_set_tile (no Matérn)."""
    n, nb = 1000, 208
    rng = np.random.default_rng(7)
    G = rng.standard_normal((n, n))
    A = G @ G.T / n + np.eye(n)
    M = mp.Matrix(handle, n, nb, None)
    nt = M.nt
    Ap = np.eye(nt * nb)
    Ap[:n, :n] = A
    for k in range(nt):
        for m in range(k, nt):
            M.set_tile(m, k, Ap[m * nb:(m + 1) * nb, k * nb:(k + 1) * nb])
    km, sm, cm = all_fp64_maps(nt)
    assert M.potrf(km, cm) == 0
    L = gpu_factor_dense(M, n)
    assert np.max(np.abs(L - np.linalg.cholesky(A))) <= 1e-12


def test_sqexp_covariance_path(mp, handle):
    """The paper's 2D squared exponential through the same path: tiles and l vs the oracle."""
    n, nb, theta = 1600, 512, (1.0, 0.0003, 0.0)
    x, y = synth.locations(n, 3)
    z = synth.normal_vector(n, 4)
    ref = oracle_loglik(x, y, z, theta, nb, kernel="sqexp")
    M = mp.Matrix(handle, n, nb, None)
    M.set_covariance(mp.MP_COV_SQEXP)
    M.matern_gen(to_dev(x), to_dev(y), theta, np.zeros((M.nt, M.nt), np.uint8))
    for key in [(2, 1), (3, 3), (3, 0)]:
        g = M.tile(*key)
        t = ref["tiles"][key]
        assert np.max(np.abs(g[: t.shape[0], : t.shape[1]] - t)) <= 1e-15
    ev = mp.Evaluator(n, nb, handle=handle, covariance=mp.MP_COV_SQEXP)
    r = ev.eval(x, y, z, theta, mode=mp.MP_MAP_FP64)
    assert abs(r.loglik - ref["loglik"]) <= 1e-10 * abs(ref["loglik"])


@pytest.mark.parametrize("nu", [0.3, 0.8, 1.7, 3.2])
def test_general_nu_tabulated_generation_vs_mpmath(mp, handle, nu):
    """General nu is generated from a per-evaluation piecewise Chebyshev table of the correlation
    (matern.cu): sampled entries against 30-digit mpmath, relative error <= 4e-15 + r 2^-52 (the
    table's floor ~2e-15: the e^r / e^-r factors and Clenshaw each add an ulp; r carries one rounding)."""
    import mpmath
    mpmath.mp.dps = 30
    n, nb, theta = 4096, 512, (1.4, 0.04, nu)
    x, y = synth.locations(n, 6)
    M = mp.Matrix(handle, n, nb, None)
    M.matern_gen(to_dev(x), to_dev(y), theta, np.zeros((M.nt, M.nt), np.uint8))
    rng = np.random.default_rng(int(nu * 10))
    for (m, k) in [(0, 0), (3, 2), (7, 0), (5, 5)]:
        t = M.tile(m, k)
        for _ in range(12):
            i, j = int(rng.integers(0, nb)), int(rng.integers(0, nb))
            gi, gj = m * nb + i, k * nb + j
            if gi == gj:
                continue
            dx, dy = x[gi] - x[gj], y[gi] - y[gj]
            h = float(np.sqrt(dx * dx + dy * dy))
            r = mpmath.mpf(h) / mpmath.mpf(theta[1])
            ref = float(mpmath.mpf(theta[0]) * 2 ** (1 - mpmath.mpf(nu)) / mpmath.gamma(nu) * r**nu
                        * mpmath.besselk(nu, r))
            assert abs(t[i, j] - ref) <= (4e-15 + float(r) * 2.0**-52) * abs(ref) + 1e-300, (nu, m, k, i, j, t[i, j], ref)


def test_gp_sample_matches_dense_factor(mp, handle):
    """mp_gp_sample: z = L e with the library's factor equals the dense Cholesky factor times e."""
    n, nb, theta = 1500, 256, (1.0, 0.1, 0.5)
    x, y = synth.uniform_locations(n, 2)
    e = synth.normal_vector(n, 3)
    M = mp.Matrix(handle, n, nb, None)
    km, sm, cm = all_fp64_maps(M.nt)
    M.matern_gen(to_dev(x), to_dev(y), theta, sm)
    assert M.potrf(km, cm) == 0
    import torch
    dz = torch.zeros(n, dtype=torch.float64, device="cuda")
    M.gp_sample(to_dev(e), dz)
    from oracle.tiles import dense_covariance
    ref = np.linalg.cholesky(dense_covariance(x, y, theta)) @ e
    assert np.max(np.abs(dz.cpu().numpy() - ref)) <= 1e-12 * np.max(np.abs(ref))


def test_fp16_storage_class(mp):
    """SURVEY §8(f)3 FP16 storage class (mp_config.fp16_storage): FP16-class tiles stored as fp16(x 2^t),
    sent in FP16.  Maps: storage and comm FP16 exactly where the kernel map is FP16 (else the paper's
    maps); l within the north-star 1e-5 of the FP64 oracle; the factor's backward error within the bound
    of the maps (FP16 storage rounding included); smaller workspace than the P:152 FP32 storage."""
    n, nb, u_req, theta = 10000, 512, 1e-9, (1.0, 0.03, 0.5)
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ref = oracle_loglik(x, y, z, theta, nb)
    nt = num_tiles(n, nb)
    okm, osm, ocm = precision_maps(tile_sqnorms(ref["tiles"], nt), u_req)
    h16 = mp.Handle(0, config={"fp16_storage": 1})
    ev16 = mp.Evaluator(n, nb, handle=h16)
    r16 = ev16.eval(x, y, z, theta, u_req=u_req)
    km, sm, cm = ev16.M.maps()
    low = np.tril(np.ones((nt, nt), bool), -1)
    assert np.array_equal(km[low], okm[low]) and r16.tiles[2] > 0
    f16 = low & (okm == FP16)
    assert np.all(sm[f16] == FP16) and np.all(cm[f16] == FP16)
    assert np.array_equal(sm[low & ~f16], osm[low & ~f16]) and np.array_equal(cm[low & ~f16], ocm[low & ~f16])
    err = abs(r16.loglik - ref["loglik"]) / abs(ref["loglik"])
    assert err <= 1e-5, err
    Lhat = {key: ev16.M.tile(*key)[: t.shape[0], : t.shape[1]] for key, t in ref["tiles"].items()}
    worst, _ = mp_backward_check(ref["tiles"], Lhat, ref["factor"], km, sm, cm, nt, nb)
    assert worst <= 1.0, worst
    ev32 = mp.Evaluator(n, nb)
    r32 = ev32.eval(x, y, z, theta, u_req=u_req)
    assert r16.workspace_bytes < r32.workspace_bytes
    print(f"FP16 storage: l rel. error {err:.2e} (FP32 storage {abs(r32.loglik - ref['loglik']) / abs(ref['loglik']):.2e}), "
          f"workspace {r16.workspace_bytes / 1e9:.2f} vs {r32.workspace_bytes / 1e9:.2f} GB")
