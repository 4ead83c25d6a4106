// Internal launcher interface between the host engine (engine.cu) and the kernels.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"

namespace mpgeo {

// ---- K5: batched FP64 DMMA GEMM, C = beta*C + alpha*A*B^T (dgemm_dmma.cu)
struct DgemmArgs {
    const GemmJob* jobs;  // device array, one entry per job
    int M, N, K;          // K % 16 == 0
    int lda, ldb, ldc;    // elements; even (16-byte rows)
    int lower;            // compute only CTA tiles on/below the diagonal (M == N)
    double alpha, beta;   // alpha in {-1, +1}; beta in {0, 1}
    // filled by the launcher
    int tiles_m, tiles_n, tiles_per_job;
};
cudaError_t dgemm_nt_launch(DgemmArgs a, int njobs, int round_ops, bool c_f32, cudaStream_t s);

// ---- K3 helpers: diagonal-block Cholesky + inverse, block inverses (potrf.cu)
constexpr int POTRF_IB = 128;  // inner block of the tile POTRF / TRSM
// Factor the jb x jb block at A (lda) in place (lower), write W = L^{-1} (ld POTRF_IB, zero
// upper) to W; on a non-positive pivot atomicMin(info, col0 + c + 1).
cudaError_t potrf_diag_block_launch(double* A, int lda, int jb, double* W, int col0, int* info,
                                    cudaStream_t s);
// For each diagonal block b of the nb x nb lower matrix L (ld nb): W_b = inv(L_bb).
cudaError_t trtri_blocks_launch(const double* L, int nb, double* W, cudaStream_t s);
// Batched over tiles: W[t][b] = inv(L_t,bb) for every 128-block b of every tile t
cudaError_t trtri_batch_launch(const double* const* Ls, int ntiles, int nb, double* W, cudaStream_t s);

// ---- K1: Matérn generation (matern.cu)
struct GenTile {
    int m, k;     // tile coordinates
    int prec;     // storage precision of the destination (P64 / P32 / P16); unused in pass 1
    int scale;    // P16 storage: the tile's exponent t (stored value fp16(x 2^t))
    void* dst;    // nb x nb row-major destination (pass 2)
};
struct MaternArgs {
    const double* x;
    const double* y;
    int64_t n;
    int nb;
    double sigma2, beta, nu;
    int kind;     // 0: nu = 1/2, 1: nu = 3/2, 2: nu = 5/2, 3: general nu, 4: squared exponential
    double coef;  // 2^(1-nu) / Gamma(nu) for the general formula
    // general nu: piecewise Chebyshev table of the normalised correlation in u = log(r) (see matern.cu)
    const double* tab;  // [npieces][MT_DEG + 1] coefficients, null = evaluate K_nu directly
    double u0, inv_w, w;
    int npieces, split;  // pieces p >= split carry rho(r) e^r (r > 2), pieces below carry rho(r)
};
constexpr int MT_DEG = 15;  // Chebyshev degree per piece
// Build the table for kind 3 (one CTA per piece); pieces of width w in u = log r from u0.
cudaError_t matern_table_launch(const MaternArgs& a, double* tab, cudaStream_t s);
constexpr int GEN_ROWS = 16;  // rows per CTA in the generation kernels
// Pass 1: partial sums of squares, partials[t * (nb/GEN_ROWS) + chunk]
cudaError_t matern_norm_launch(const MaternArgs& a, const GenTile* tiles, int ntiles, double* partials,
                               cudaStream_t s);
// Reduce partials (fixed order) into out[t]
cudaError_t reduce_partials_launch(const double* partials, int ntiles, int per_tile, double* out,
                                   cudaStream_t s);
// Pass 2: write tiles in storage precision (padding: identity on diagonal tiles, zero elsewhere)
cudaError_t matern_write_launch(const MaternArgs& a, const GenTile* tiles, int ntiles, cudaStream_t s);
// Device Bessel K_nu for tests: out[i] = K_nu(x[i])
cudaError_t bessel_k_launch(double nu, const double* x, double* out, int n, cudaStream_t s);

// ---- K2: panel conversion (convert.cu)
struct PanelTile {
    void* store;      // the tile in the pool (storage precision)
    double* p64;      // FP64 panel slot
    int store_prec;   // P64 / P32 / P16 (FP16 storage class, scaled by 2^scale)
    int comm_prec;    // precision the tile is sent at (P64 / P32 / P16)
    int scale;        // P16 storage: the tile's exponent
    int pad;
};
struct Tf32Item {     // 3xTF32 operands of one panel tile (FP32 class with MP_F32_3XTF32)
    const double* src;
    float* hi;
    float* lo;
};
// Row-scaled FP16 operands of one FP64 panel tile (split16_kernel, convert.cu)
struct Split16Item {
    const double* src;  // FP64 panel slot (nb x nb)
    __half* hi;         // row-scaled FP16 hi / lo (nb x nb); lo may be null (FP16 class only)
    __half* lo;
    int* exps;          // [nb]: 2^exps undoes row i's scale
    __half* hs = nullptr;  // optional pure-FP16 operand rn(x 2^(s - 13)) (four-level maps)
};
cudaError_t split16_launch(const Split16Item* items, int n, int nb, cudaStream_t s);
// p64 = (double) store
cudaError_t panel_in_launch(const PanelTile* t, int ntiles, int64_t elems, cudaStream_t s);
// store = round(p64, store_prec); p64 = round(p64, comm_prec)
cudaError_t panel_out_launch(const PanelTile* t, int ntiles, int64_t elems, cudaStream_t s);
// hi/lo = 3xTF32 split of fp32(src)
cudaError_t tf32_split_launch(const Tf32Item* t, int ntiles, int64_t elems, cudaStream_t s);
// dst = round(src, prec) elementwise on FP64 arrays
cudaError_t round_copy_launch(const double* src, double* dst, int64_t elems, int prec, cudaStream_t s);
// zero the strictly upper triangle of an nb x nb row-major tile
cudaError_t zero_upper_launch(double* A, int nb, cudaStream_t s);
// A = I (nb x nb FP64); dst = src^T (nb x nb FP64, nb % 32 == 0)
cudaError_t identity_launch(double* A, int nb, cudaStream_t s);
cudaError_t transpose_launch(const double* src, double* dst, int nb, cudaStream_t s);

// ---- K8: solve and reductions (solve.cu)
// y[0..nb) = L^{-1} r[0..nb) for one FP64 lower tile (ld nb), rows >= nreal are identity pads
cudaError_t trsv_tile_launch(const double* L, int nb, const double* r, double* y, cudaStream_t s);
// Blocked TRSV of one FP64 lower tile with its block inverses Wk ([block][128][128]): y = L^{-1} r
// (r is overwritten with intermediate values)
cudaError_t trsv_blocked_launch(const double* L, int nb, const double* Wk, double* r, double* y, cudaStream_t s);
struct GemvTile {
    const void* L;    // tile (m, k), storage precision, nb x nb
    int prec;
    int scale;        // P16 storage: the tile's exponent
    double* r;        // r_m (nb), updated r_m -= L y
};
// r_m -= L_mk y_k for a batch of tiles sharing y
cudaError_t gemv_sub_launch(const GemvTile* t, int ntiles, const double* y, int nb, cudaStream_t s);
// per diagonal tile k: out[k] = sum_{i < nreal_k} log L_kk[i][i]
cudaError_t logdiag_launch(const double* const* diag_tiles, const int* nreal, int ntiles, int nb,
                           double* out, cudaStream_t s);
// dst[i] = a * src[i]
cudaError_t scale_vec_launch(double* dst, const double* src, int64_t n, double a, cudaStream_t s);
// out[b] = sum of squares of v[b*chunk .. min(n, (b+1)*chunk))
cudaError_t sumsq_chunks_launch(const double* v, int64_t n, int chunk, double* out, cudaStream_t s);

}  // namespace mpgeo
