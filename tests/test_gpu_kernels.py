"""Kernel-level GPU checks through the C-ABI test hooks (include/mpgeo_test.h)."""
import ctypes as C

import mpmath
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lib():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_cluster_caoalgkb23_b200._lib import lib
    return lib


def dev(a):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("nu", [0.3, 0.5, 0.8, 1.0, 1.5, 1.7, 3.7, 12.3])
def test_bessel_k_device_vs_mpmath(lib, nu):
    mpmath.mp.dps = 30
    x = np.concatenate([np.logspace(-5, 2.2, 120), [1.9999999999, 2.0, 2.0000000001]])
    dx = dev(x)
    out = dev(np.zeros_like(x))
    assert lib.mp_test_bessel_k(nu, C.c_void_p(dx.data_ptr()), C.c_void_p(out.data_ptr()), x.size) == 0
    got = out.cpu().numpy()
    for xi, g in zip(x, got):
        ref = float(mpmath.besselk(nu, xi))
        assert abs(g - ref) <= 4e-15 * (1 + xi) * abs(ref), (nu, xi, g, ref)


def run_dgemm(lib, A, B, Cm, lower=0, alpha=-1.0, beta=1.0, rnd=0, cf32=0):
    M, K = A.shape
    N = B.shape[0]
    dA, dB, dC = dev(A), dev(B), dev(Cm)
    st = lib.mp_test_dgemm(C.c_void_p(dA.data_ptr()), C.c_void_p(dB.data_ptr()), C.c_void_p(dC.data_ptr()),
                           M, N, K, K, K, Cm.shape[1], lower, alpha, beta, rnd, cf32)
    assert st == 0
    return dC.cpu().numpy()


@pytest.mark.parametrize("M,N,K", [(128, 128, 16), (300, 200, 144), (2048, 256, 2048), (16, 48, 32)])
def test_dgemm_update_fp64(lib, M, N, K):
    rng = np.random.default_rng(M + N + K)
    A, B, Cm = rng.standard_normal((M, K)), rng.standard_normal((N, K)), rng.standard_normal((M, N))
    got = run_dgemm(lib, A, B, Cm)
    ref = Cm - A @ B.T
    assert np.max(np.abs(got - ref)) <= 1e-15 * K * 8


def test_dgemm_overwrite_and_lower(lib):
    rng = np.random.default_rng(1)
    A, B, Cm = rng.standard_normal((400, 64)), rng.standard_normal((400, 64)), rng.standard_normal((400, 400))
    got = run_dgemm(lib, A, B, Cm, alpha=1.0, beta=0.0)
    assert np.max(np.abs(got - A @ B.T)) <= 1e-13
    got = run_dgemm(lib, A, B, Cm, lower=1)
    ref = Cm - A @ B.T
    for bi in range(4):
        for bj in range(4):
            blk = (slice(bi * 128, (bi + 1) * 128), slice(bj * 128, (bj + 1) * 128))
            if bj <= bi:
                assert np.max(np.abs(got[blk] - ref[blk])) <= 1e-13
            else:
                assert np.array_equal(got[blk], Cm[blk])  # strictly upper CTA tiles untouched


@pytest.mark.parametrize("rnd,npdt", [(1, np.float32), (2, np.float16)])
def test_dgemm_rounded_operands_fp32_c(lib, rnd, npdt):
    rng = np.random.default_rng(rnd)
    A, B = rng.standard_normal((256, 128)), rng.standard_normal((256, 128))
    Cm = rng.standard_normal((256, 256)).astype(np.float32)
    got = run_dgemm(lib, A, B, Cm, rnd=rnd, cf32=1)
    Ar, Br = A.astype(npdt).astype(np.float64), B.astype(npdt).astype(np.float64)
    ref = (Cm.astype(np.float64) - Ar @ Br.T).astype(np.float32)
    assert np.max(np.abs(got.astype(np.float64) - ref)) <= 2 * np.max(np.abs(ref)) * 2.0**-24


def tf32_rna(a32: np.ndarray) -> np.ndarray:
    """cvt.rna.tf32.f32 written out: round the fp32 magnitude to 10 mantissa bits, ties away from zero."""
    b = a32.astype(np.float32).view(np.uint32).astype(np.uint64)
    b = ((b + 0x1000) & 0xFFFFE000).astype(np.uint32)
    return b.view(np.float32)


@pytest.mark.parametrize("scale", [0.1, 4e-8])
def test_tc_gemm_f16_class_row_scaled(lib, scale):
    """FP16 class (P:113 FP16_32): operands are the row-scaled FP16 hi planes, so the
    product keeps FP16 accuracy (11 bits per operand relative to its row, FP32 accumulation) even for
    tiles whose entries lie below FP16's smallest normal (scale 4e-8: the C3 FP16-class magnitude,
    where a plain FP16 conversion underflows to 0-2 bits).  Bound: |err| <= (2^-10 + K 2^-23) |A||B|^T
    entrywise, against the exact product of the FP32-rounded operands."""
    assert lib.mp_tc_available() == 1
    nb, nt = 512, 3
    rng = np.random.default_rng(3)
    P = rng.standard_normal((nt * nb, nb)) * scale * np.exp2(-rng.integers(0, 8, size=(nt * nb, 1)))
    Cm = (rng.standard_normal((nb, nb)) * scale * scale).astype(np.float32)
    dP, dC = dev(P), dev(Cm)
    assert lib.mp_test_tc_gemm_split(0, C.c_void_p(dP.data_ptr()), C.c_void_p(dC.data_ptr()), nb, nt, 2, 0, 0) == 0
    got = dC.cpu().numpy().astype(np.float64)
    A32 = P.astype(np.float32).astype(np.float64)
    A, B = A32[2 * nb:3 * nb], A32[0:nb]
    ref = Cm.astype(np.float64) - A @ B.T
    bound = (2.0**-10 + nb * 2.0**-23) * (np.abs(A) @ np.abs(B).T) + 2.0**-23 * np.abs(ref)
    assert np.all(np.abs(got - ref) <= bound), np.max(np.abs(got - ref) / bound)
    if scale < 1e-4:  # a plain (unscaled) FP16 conversion would lose the product entirely
        plain = A.astype(np.float16).astype(np.float64) @ B.astype(np.float16).astype(np.float64).T
        assert np.linalg.norm(plain - A @ B.T) > 0.1 * np.linalg.norm(A @ B.T)
        assert np.linalg.norm(got - ref) < 1e-2 * np.linalg.norm(A @ B.T)


def test_tc_gemm_tf32x3_matches_sgemm_accuracy(lib):
    """Reading C13 pin: 3xTF32 error vs an FP64 product <= 2x the SGEMM error on the same inputs."""
    nb, nt = 512, 2
    rng = np.random.default_rng(4)
    A32 = rng.standard_normal((nt * nb, nb)).astype(np.float32)
    hi = tf32_rna(A32)
    lo = tf32_rna((A32 - hi).astype(np.float32))
    Cm = np.zeros((nb, nb), np.float32)
    dH, dL, dC = dev(hi), dev(lo), dev(Cm)
    assert lib.mp_test_tc_gemm(1, C.c_void_p(dH.data_ptr()), C.c_void_p(dL.data_ptr()), C.c_void_p(dC.data_ptr()),
                               nb, nt, 1, 0) == 0
    got = -dC.cpu().numpy().astype(np.float64)
    Ad = A32.astype(np.float64)
    exact = Ad[nb:] @ Ad[:nb].T
    sgemm = (A32[nb:] @ A32[:nb].T).astype(np.float64)
    err_tc = np.linalg.norm(got - exact) / np.linalg.norm(exact)
    err_sg = np.linalg.norm(sgemm - exact) / np.linalg.norm(exact)
    single = (hi[nb:].astype(np.float64) @ hi[:nb].astype(np.float64).T)
    err_1x = np.linalg.norm(single - exact) / np.linalg.norm(exact)
    assert err_tc <= 2 * err_sg + 1e-9, (err_tc, err_sg)
    assert err_tc < err_1x / 50  # far better than a single TF32 product


@pytest.mark.parametrize("nb,spread,colspread,persistent", [(512, 0, 0, 0), (512, 30, 0, 0), (2048, 0, 0, 0),
                                                              (2048, 30, 30, 0), (2048, 30, 30, 1)])
def test_tc_gemm_f16x3_matches_sgemm_accuracy(lib, nb, spread, colspread, persistent):
    """Reading C13c pin: 3xFP16 (row-scaled FP16 hi/lo split, kind::f16) error vs the exact product of
    the FP32-rounded operands <= 2x the SGEMM error on the same inputs — at the bench tile size
    nb = 2048 (16 TMEM chunks of K = 128), with row magnitudes spread over 2^-spread .. 1 and, within
    each row, entries spread over 2^-colspread .. 1 (the large within-row range of Cholesky panel rows;
    ADVICE r01), also with the persistent kernel; a zero row gives a zero row of the product."""
    nt = 2
    rng = np.random.default_rng(5 + nb + spread)
    P = rng.standard_normal((nt * nb, nb)) * np.exp2(-rng.integers(0, spread + 1, size=(nt * nb, 1)))
    P *= np.exp2(-rng.uniform(0, colspread, size=(1, nb)))
    P[nb + 3] = 0.0
    Cm = np.zeros((nb, nb), np.float32)
    dP, dC = dev(P), dev(Cm)
    assert lib.mp_test_tc_gemm_split(2, C.c_void_p(dP.data_ptr()), C.c_void_p(dC.data_ptr()), nb, nt, 1, 0,
                                     persistent) == 0
    got = -dC.cpu().numpy().astype(np.float64)
    A32 = P.astype(np.float32)
    Ad = A32.astype(np.float64)
    exact = Ad[nb:] @ Ad[:nb].T
    sgemm = (A32[nb:] @ A32[:nb].T).astype(np.float64)
    # row-wise relative errors (rows of different magnitude must each be accurate)
    rn = np.linalg.norm(exact, axis=1)
    ok = rn > 0
    err_tc = np.max(np.linalg.norm(got - exact, axis=1)[ok] / rn[ok])
    err_sg = np.max(np.linalg.norm(sgemm - exact, axis=1)[ok] / rn[ok])
    print(f"3xFP16 nb={nb} spread={spread}/{colspread} persistent={persistent}: row-wise error {err_tc:.3e}, "
          f"SGEMM {err_sg:.3e}")
    assert err_tc <= 2 * err_sg + 1e-9, (err_tc, err_sg)
    assert np.all(got[3] == 0.0)
    single = (A32[nb:].astype(np.float16).astype(np.float64) @ A32[:nb].astype(np.float16).astype(np.float64).T)
    if spread == 0 and colspread == 0:
        assert err_tc < np.max(np.linalg.norm(single - exact, axis=1)[ok] / rn[ok]) / 50


@pytest.mark.parametrize("nb,nt,m,n,nmod", [(512, 3, 2, 0, 16), (4096, 2, 1, 0, 16), (2048, 3, 1, 2, 16)])
def test_crt_int8_fp64_gemm(lib, nb, nt, m, n, nmod):
    """FP64 GEMM by CRT modular emulation on tcgen05 kind::i8 vs the exact FP64 product: with 16
    moduli the operands keep b = 56 bits (rounded) per row, so |err| <= K 2^-(b+1) max|a_i| max|b_j|
    + the final FP64 rounding — within the FP64-GEMM-level bound 8 K u max|a| max|b|.  nb = 4096 gives 256 pair tiles for 74 persistent CTA pairs (several tiles per pair, both
    accumulator parities, scratch-slot reuse).  Rows of very different scale and an all-zero row."""
    rng = np.random.default_rng(nb + nmod)
    P = rng.standard_normal((nt * nb, nb)) * np.exp(rng.uniform(-3, 3, (nt * nb, 1)))
    P[m * nb + 5] = 0.0
    Cm = rng.standard_normal((nb, nb))
    dP, dC = dev(P), dev(Cm)
    assert lib.mp_test_crt_gemm(C.c_void_p(dP.data_ptr()), C.c_void_p(dC.data_ptr()), nb, nt, m, n, nmod, 0, 0) == 0
    got = dC.cpu().numpy()
    A, B = P[m * nb:(m + 1) * nb], P[n * nb:(n + 1) * nb]
    ref = Cm - A @ B.T
    ma = np.abs(A).max(axis=1)[:, None]
    mb = np.abs(B).max(axis=1)[None, :]
    scale = np.maximum(ma * mb, 1e-300)
    err = np.max(np.abs(got - ref) / (scale + np.abs(ref) * 1e-300))
    bound = 8 * nb * 2.0**-53
    assert err <= bound, (err, bound)
    assert np.array_equal(got[5], Cm[5])  # zero row of A: C row untouched


@pytest.mark.parametrize("nmod", [8, 16])
def test_crt_store_mode_fp64_c(lib, nmod):
    """Store mode (C = P_m P_n^T, the TRSM product X = A_mk W^T with W = L_kk^-1): CRT-8 (the FP32-class
    TRSM, FP64 C) keeps b = 25 bits per operand row, CRT-16 b = 56; C's previous contents are ignored."""
    nb, nt, m, n = 2048, 2, 1, 0
    rng = np.random.default_rng(nmod + 1)
    P = rng.standard_normal((nt * nb, nb)) * np.exp(rng.uniform(-3, 3, (nt * nb, 1)))
    P[n * nb:(n + 1) * nb] = np.tril(P[n * nb:(n + 1) * nb])  # a triangular B operand, like the inverse factor
    Cm = np.full((nb, nb), np.nan)
    dP, dC = dev(P), dev(Cm)
    assert lib.mp_test_crt_gemm(C.c_void_p(dP.data_ptr()), C.c_void_p(dC.data_ptr()), nb, nt, m, n, nmod, 0, 1) == 0
    got = dC.cpu().numpy()
    A, B = P[m * nb:(m + 1) * nb], P[n * nb:(n + 1) * nb]
    ref = A @ B.T
    b = {8: 25, 16: 56}[nmod]
    ma = np.abs(A).max(axis=1)[:, None]
    mb = np.abs(B).max(axis=1)[None, :]
    assert np.all(np.isfinite(got))
    err = np.abs(got - ref) - 2.0**-52 * np.abs(ref)
    assert np.all(err <= nb * 2.0 ** -b * ma * mb), np.max(err / (ma * mb)) / 2.0**-b


def test_crt_int8_syrk_lower(lib):
    """lower = 1 (DSYRK on a diagonal tile): 256 x 256 blocks on or below the diagonal are updated,
    strictly-upper blocks are left untouched."""
    nb, nt = 1024, 2
    rng = np.random.default_rng(3)
    P = rng.standard_normal((nt * nb, nb))
    Cm = rng.standard_normal((nb, nb))
    dP, dC = dev(P), dev(Cm)
    assert lib.mp_test_crt_gemm(C.c_void_p(dP.data_ptr()), C.c_void_p(dC.data_ptr()), nb, nt, 1, 1, 16, 1, 0) == 0
    got = dC.cpu().numpy()
    A = P[nb:]
    ref = Cm - A @ A.T
    for bi in range(nb // 256):
        for bj in range(nb // 256):
            blk = (slice(bi * 256, (bi + 1) * 256), slice(bj * 256, (bj + 1) * 256))
            if bj > bi:
                assert np.array_equal(got[blk], Cm[blk])
            else:
                assert np.max(np.abs(got[blk] - ref[blk])) <= 8 * nb * 2.0**-53 * np.abs(A).max() ** 2


@pytest.mark.parametrize("scale", [1.0, 4e-8])
def test_tc_gemm_pure_fp16_accumulates_in_fp16(lib, scale):
    """Pure FP16 class (four-level maps, "A, B, C, and operation are all in FP16"): row-scaled FP16
    operands (the hs planes) and an F16 TMEM accumulator over the whole K.  Pins: (i) the error against the
    exact product of the FP32-rounded operands stays within the FP16-accumulation bound
    (2^-10 + K 2^-11) |A||B|^T entrywise; (ii) it is the FP16 accumulator that ran: the normwise error is
    several times the FP16_32 kernel's on the same operands (FP32 accumulation), and close to an emulated
    FP16 accumulation; (iii) no overflow at the C3 FP16-class magnitude (scale 4e-8) thanks to the row scale."""
    assert lib.mp_tc_available() == 1
    nb, nt = 2048, 2
    rng = np.random.default_rng(11)
    P = np.abs(rng.standard_normal((nt * nb, nb))) * scale * np.exp2(-rng.integers(0, 6, size=(nt * nb, 1)))
    out = {}
    for kind in (0, 3):
        dP, dC = dev(P), dev(np.zeros((nb, nb), np.float32))
        assert lib.mp_test_tc_gemm_split(kind, C.c_void_p(dP.data_ptr()), C.c_void_p(dC.data_ptr()), nb, nt, 1, 0, 0) == 0
        out[kind] = -dC.cpu().numpy().astype(np.float64)
    A32 = P.astype(np.float32).astype(np.float64)
    A, B = A32[nb:2 * nb], A32[0:nb]
    exact = A @ B.T
    assert np.all(np.isfinite(out[3]))
    bound = (2.0**-10 + nb * 2.0**-11) * (np.abs(A) @ np.abs(B).T)
    assert np.all(np.abs(out[3] - exact) <= bound)
    e3 = np.linalg.norm(out[3] - exact) / np.linalg.norm(exact)
    e0 = np.linalg.norm(out[0] - exact) / np.linalg.norm(exact)
    print(f"scale {scale}: pure FP16 {e3:.3e}, FP16_32 {e0:.3e}, ratio {e3 / e0:.1f}")
    assert e3 > 3 * e0, (e3, e0)   # positive entries: FP16 accumulation error grows with K
    assert e3 < 2.0**-4, e3
