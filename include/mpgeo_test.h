/*
 * mpgeo_test.h — kernel-level test hooks of libmpgeo.so (C ABI, device pointers).
 * Used only by tests/ to check single kernels against the oracle; not part of the path.
 * All return mp_status (0 = OK) and synchronise the default stream.
 */
#ifndef MPGEO_TEST_H
#define MPGEO_TEST_H
#include "mpgeo.h"
#ifdef __cplusplus
extern "C" {
#endif
/* out[i] = K_nu(x[i]) (modified Bessel function of the second kind, device code of K1). */
mp_status mp_test_bessel_k(double nu, const double* d_x, double* d_out, int n);
/* One job of the K5 DMMA GEMM: C = beta*C + alpha*A*B^T (row-major, see kernels.h).
 * round: operand rounding class (0 FP64, 1 FP32, 2 FP16); c_f32: C is float. */
mp_status mp_test_dgemm(const double* d_A, const double* d_B, void* d_C, int M, int N, int K, int lda, int ldb,
                        int ldc, int lower, double alpha, double beta, int round, int c_f32);
/* One job of the tcgen05 GEMMs: C (FP32 nb x nb) -= P_m P_n^T with P the panel cache
 * [nt*nb][nb]: kind 1 = 3xTF32 (panel = hi, panel_lo = lo, float), kind 2 = FP16 (panel = half). */
mp_status mp_test_tc_gemm(int kind, const void* d_panel, const void* d_panel_lo, float* d_C, int nb, int nt, int m,
                          int n);
/* 3xFP16 FP32-class GEMM (reading C13c): splits the nt tiles of the FP64 panel [nt*nb][nb] into
 * row-scaled FP16 hi / lo, then C (FP32 nb x nb) -= P_m P_n^T on tcgen05 kind::f16. */
mp_status mp_test_tc_gemm_f16x3(const double* d_panel, float* d_C, int nb, int nt, int m, int n);
/* Ozaki-split GEMM on INT8 tensor cores: splits the nt tiles of the FP64 panel [nt*nb][nb] into 8
 * int8 slices, then C -= P_m P_n^T using the first S slices: S = 8 (FP64 class, C FP64, lower CTA
 * tiles only if `lower`) or S = 4 (FP32 class, C is FP32). */
mp_status mp_test_ozaki_gemm(const double* d_panel, double* d_C, int nb, int nt, int m, int n, int S, int lower);
/* CRT ("Ozaki scheme II") GEMM on INT8 tensor cores: the nt tiles of the FP64 panel [nt*nb][nb]
 * become nmod int8 residue planes, then C -= P_m P_n^T (lower: only 256 x 256 blocks on or below the
 * diagonal).  nb % 256 == 0; nmod = 16: C is FP64 (FP64 class); nmod = 8: C is FP32 (FP32 class). */
mp_status mp_test_crt_gemm(const double* d_panel, void* d_C, int nb, int nt, int m, int n, int nmod, int lower);
/* The same with the C type and mode explicit: c_f32 (FP32 C, nmod = 8 only), store = 1: C = P_m P_n^T
 * (overwrite; the FP32-class TRSM product), else C -= P_m P_n^T. */
mp_status mp_test_crt_gemm_ex(const double* d_panel, void* d_C, int nb, int nt, int m, int n, int nmod, int lower,
                              int c_f32, int store);
/* Isolated timing of the INT8 engines (engine 8: 8-slice splitting, 16: CRT with nmod moduli — nmod
 * = 16 FP64 C, nmod = 8 the FP32-class instantiation with FP32 C) on njobs batched nb x nb tile-GEMMs over an nt-tile panel; ms[0] = panel split, ms[1] = GEMM
 * launch, milliseconds (mean of reps). */
mp_status mp_bench_fp64_engine(int engine, int nb, int nt, int njobs, int nmod, int reps, float* ms);
/* Host constants of the CRT engine for nmod (even) moduli and inner dimension K: operand bits, the
 * nmod moduli, the split CRT weights w_j = H_j + L_j of the nmod/2 paired moduli m_j = p_2j p_2j+1
 * and M = Mhl[0] + Mhl[1] (host pointers). */
mp_status mp_test_crt_constants(int nmod, int K, int* bits, int* moduli, double* H, double* L, double* Mhl);
/* 1 if the tcgen05 kernels are compiled in, else 0. */
int mp_tc_available(void);
/* Correctly rounded sum of n doubles (host; the S of the precision rule). */
double mpgeo_exact_sum(const double* v, int64_t n);
#ifdef __cplusplus
}
#endif
#endif
