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
/* One job of the 3xTF32 tcgen05 GEMM (kind must be 1): C (FP32 nb x nb) -= P_m P_n^T with the TF32
 * hi / lo panel caches [nt*nb][nb] (float) in d_panel / d_panel_lo. */
mp_status mp_test_tc_gemm(int kind, const void* d_panel, const void* d_panel_lo, float* d_C, int nb, int nt, int m,
                          int n);
/* The row-scaled FP16 tcgen05 GEMMs from an FP64 panel [nt*nb][nb]: split16 (row scale 2^-e_i,
 * FP16 hi / lo), then C (FP32 nb x nb) -= P_m P_n^T.  kind 0: FP16 class (hi only, kind::f16, one
 * product); kind 2: FP32 class as 3xFP16 (reading C13c); persistent: the persistent 3xFP16 kernel. */
mp_status mp_test_tc_gemm_split(int kind, const double* d_panel, float* d_C, int nb, int nt, int m, int n,
                                int persistent);
/* CRT ("Ozaki scheme II") GEMM on INT8 tensor cores: the nt tiles of the FP64 panel [nt*nb][nb]
 * become nmod int8 residue planes, then C (FP64 nb x nb) -= P_m P_n^T (store = 1: C = P_m P_n^T;
 * lower: only 256 x 256 blocks on or below the diagonal).  nb % 256 == 0; nmod = 16 (FP64 class)
 * or 8 (the FP32-class TRSM product). */
mp_status mp_test_crt_gemm(const double* d_panel, double* d_C, int nb, int nt, int m, int n, int nmod, int lower,
                           int store);
/* Isolated timing of the CRT engine with nmod moduli on njobs batched nb x nb tile-GEMMs over an
 * nt-tile panel; ms[0] = panel split, ms[1] = GEMM launch, milliseconds (mean of reps). */
mp_status mp_bench_fp64_engine(int nb, int nt, int njobs, int nmod, int reps, float* ms);
/* Host constants of the CRT engine for nmod (even) moduli and inner dimension K: operand bits, the
 * nmod moduli, the split CRT weights w_j = H_j + L_j of the nmod/2 paired moduli m_j = p_2j p_2j+1
 * and M = Mhl[0] + Mhl[1] (host pointers). */
mp_status mp_test_crt_constants(int nmod, int K, int* bits, int* moduli, double* H, double* L, double* Mhl);
/* The CRT engine's element reconstruction (crt_recon_bits, the same host/device function the GEMM
   epilogue runs), evaluated on the host: R = n x (nmod/2) combined pair residues (row-major), e0[n]
   exponents, neg = 1 for -X; out[n] = FP64 results.  Pinned on CPU against big-integer CRT. */
mp_status mp_test_crt_recon(int nmod, int K, const uint32_t* R, const int* e0, int n, int neg, double* out);
/* 1 if the tcgen05 kernels are compiled in, else 0. */
int mp_tc_available(void);
/* Correctly rounded sum of n doubles (host; the S of the precision rule). */
double mpgeo_exact_sum(const double* v, int64_t n);
#ifdef __cplusplus
}
#endif
#endif
