// K3 helpers — FP64 Cholesky and triangular inverse of one <= 128 x 128 diagonal block.  The tile
// DPOTRF of Algorithm 1 ("D" = FP64 on diagonal tiles) and the panel TRSM are
// blocked right-looking loops whose bulk work is the DMMA GEMM (dgemm_dmma.cu); only these small
// sequential pieces live here.  The inverse W = L_bb^{-1} turns each block's triangular solve into a
// 128-wide GEMM (X_b = A_b W^T).  They sit on the panel's critical path (16 per diagonal tile), so the
// O(n^3) work runs from registers with one barrier per column / row step.
#include <math.h>

#include "common.cuh"
#include "kernels.h"

namespace mpgeo {

constexpr int PB = POTRF_IB;  // 128
constexpr int PLD = PB + 1;   // padded smem leading dimension
constexpr int PT = 256;       // threads

// Register blocking.  Thread
// (tx, ty) = (tid % 16, tid / 16) owns the 8 x 8 entries i = ty + 16 r, j = tx + 16 s of the 128 x 128
// block in registers; per column / row step only the column (row) being eliminated goes through shared
// memory (double-buffered, one barrier per step), so the O(n^3) work runs from registers.  Entries
// beyond jb are the identity (their factor and inverse are the identity and never written out).
constexpr int RB = PB / 16;  // 8

// Cholesky (lower, right-looking): a <- L.  The pivot quartet of column c (d, sqrt d, 1/sqrt d, 1/d)
// is computed by the owner of (c, c) right after its last update (end of step c-1).
template <int CS>
__device__ __forceinline__ void reg_cholesky_cols(double (&a)[RB][RB], double* colbuf, double* pv, int jb, int col0,
                                                  int* info) {
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
#pragma unroll 1
    for (int cl = 0; cl < 16; ++cl) {
        const int c = CS * 16 + cl;
        double* cb = colbuf + (c & 1) * PB;
        if (tx == cl) {  // owners of column c publish it (unscaled)
#pragma unroll
            for (int r = CS; r < RB; ++r)
                if (ty + 16 * r >= c) cb[ty + 16 * r] = a[r][CS];
        }
        __syncthreads();
        const double* q = pv + (c & 1) * 4;
        const double d = q[0], sd = q[1], isd = q[2], ip = q[3];
        if (tid == 0 && c < jb && !(d > 0.0)) atomicMin(info, col0 + c + 1);
        double li[RB], lj[RB];
#pragma unroll
        for (int r = CS; r < RB; ++r) li[r] = cb[ty + 16 * r] * ip;
#pragma unroll
        for (int t = CS; t < RB; ++t) lj[t] = cb[tx + 16 * t];
#pragma unroll
        for (int r = CS; r < RB; ++r)
#pragma unroll
            for (int t = CS; t <= r; ++t) {
                const int i = ty + 16 * r, j = tx + 16 * t;
                if (j > c && i >= j) a[r][t] = fma(-li[r], lj[t], a[r][t]);
            }
        if (tx == cl) {  // column c is final: scale it
#pragma unroll
            for (int r = CS; r < RB; ++r) {
                const int i = ty + 16 * r;
                if (i == c) a[r][CS] = sd;
                else if (i > c) a[r][CS] *= isd;
            }
        }
        // the owner of (c+1, c+1) prepares the next pivot (its entry got its last update above)
        const int c1 = c + 1;
        if (c1 < PB && tx == (c1 & 15) && ty == (c1 & 15)) {
            const double d1 = (cl == 15) ? (CS + 1 < RB ? a[CS + 1 < RB ? CS + 1 : CS][CS + 1 < RB ? CS + 1 : CS] : 0.0)
                                         : a[CS][CS];
            const double sd1 = sqrt(d1);
            double* q1 = pv + (c1 & 1) * 4;
            q1[0] = d1;
            q1[1] = sd1;
            q1[2] = 1.0 / sd1;
            q1[3] = 1.0 / d1;
        }
    }
    if constexpr (CS + 1 < RB) reg_cholesky_cols<CS + 1>(a, colbuf, pv, jb, col0, info);
}

// Cholesky (lower, right-looking): a <- L.  The pivot quartet of column c (d, sqrt d, 1/sqrt d, 1/d)
// is computed by the owner of (c, c) right after its last update (end of step c-1).
__device__ __forceinline__ void reg_cholesky(double (&a)[RB][RB], double* colbuf, double* pv, int jb, int col0,
                                             int* info) {
    if (threadIdx.x == 0) {
        const double d = a[0][0], sd = sqrt(d);
        pv[0] = d;
        pv[1] = sd;
        pv[2] = 1.0 / sd;
        pv[3] = 1.0 / d;
    }
    reg_cholesky_cols<0>(a, colbuf, pv, jb, col0, info);
}

// W = L^-1 (lower) in registers from L in shared memory (S, ld PLD) and invd[i] = 1 / L_ii:
// Gauss-Jordan by rows — row p of W is final after scaling by 1/L_pp, then every row i > p
// subtracts L_ip times it.
template <int PS>
__device__ __forceinline__ void reg_trtri_rows(double (&w)[RB][RB], const double* S, const double* invd, double* rowbuf) {
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
#pragma unroll 1
    for (int pl = 0; pl < 16; ++pl) {
        const int p = PS * 16 + pl;
        double* rb = rowbuf + (p & 1) * PB;
        if (ty == pl) {  // owners of row p: scale and publish it
            const double ip = invd[p];
#pragma unroll
            for (int t = 0; t <= PS; ++t)
                if (tx + 16 * t <= p) {
                    w[PS][t] *= ip;
                    rb[tx + 16 * t] = w[PS][t];
                }
        }
        double lc[RB];
#pragma unroll
        for (int r = PS; r < RB; ++r) lc[r] = S[(ty + 16 * r) * PLD + p];
        __syncthreads();
        double rp[RB];
#pragma unroll
        for (int t = 0; t <= PS; ++t) rp[t] = rb[tx + 16 * t];
#pragma unroll
        for (int r = PS; r < RB; ++r)
#pragma unroll
            for (int t = 0; t <= PS; ++t) {
                const int i = ty + 16 * r, j = tx + 16 * t;
                if (i > p && j <= p) w[r][t] = fma(-lc[r], rp[t], w[r][t]);
            }
    }
    if constexpr (PS + 1 < RB) reg_trtri_rows<PS + 1>(w, S, invd, rowbuf);
}

__device__ __forceinline__ void reg_trtri(double (&w)[RB][RB], const double* S, const double* invd, double* rowbuf) {
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
#pragma unroll
    for (int r = 0; r < RB; ++r)
#pragma unroll
        for (int t = 0; t < RB; ++t) w[r][t] = (ty + 16 * r == tx + 16 * t) ? 1.0 : 0.0;
    reg_trtri_rows<0>(w, S, invd, rowbuf);
}

constexpr int RP_SMEM = (PB * PLD + 2 * PB + 2 * PB + PB + 8) * 8;

__global__ void __launch_bounds__(PT, 1)
    potrf_diag_block_kernel(double* A, int lda, int jb, double* W, int col0, int* info) {
    extern __shared__ double S[];
    double* colbuf = S + PB * PLD;  // 2 x PB (also the row buffer of the inverse)
    double* invd = colbuf + 2 * PB;
    double* pv = invd + PB;         // 2 x 4
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
    double a[RB][RB];
#pragma unroll
    for (int r = 0; r < RB; ++r)
#pragma unroll
        for (int t = 0; t < RB; ++t) {
            const int i = ty + 16 * r, j = tx + 16 * t;
            a[r][t] = (i < jb && j < jb) ? (j <= i ? A[(size_t)i * lda + j] : 0.0) : (i == j ? 1.0 : 0.0);
        }
    reg_cholesky(a, colbuf, pv, jb, col0, info);
    // L -> shared memory (inverse operand) and global memory (zeros above the diagonal)
#pragma unroll
    for (int r = 0; r < RB; ++r)
#pragma unroll
        for (int t = 0; t < RB; ++t) {
            const int i = ty + 16 * r, j = tx + 16 * t;
            const double v = j <= i ? a[r][t] : 0.0;
            S[i * PLD + j] = v;
            if (i < jb && j < jb) A[(size_t)i * lda + j] = v;
            if (i == j) invd[i] = 1.0 / v;
        }
    __syncthreads();
    reg_trtri(a, S, invd, colbuf);
#pragma unroll
    for (int r = 0; r < RB; ++r)
#pragma unroll
        for (int t = 0; t < RB; ++t) {
            const int i = ty + 16 * r, j = tx + 16 * t;
            if (i < jb && j < jb) W[i * PB + j] = j <= i ? a[r][t] : 0.0;
        }
}

// W_b = L_bb^-1 for the 128-blocks of a diagonal tile (register-blocked inverse, one CTA per block)
__device__ __forceinline__ void trtri_block(const double* Lb, int ld, int jb, double* Wb) {
    extern __shared__ double S[];
    double* rowbuf = S + PB * PLD;
    double* invd = rowbuf + 2 * PB;
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
#pragma unroll
    for (int r = 0; r < RB; ++r)
#pragma unroll
        for (int t = 0; t < RB; ++t) {
            const int i = ty + 16 * r, j = tx + 16 * t;
            const double v = (i < jb && j < jb) ? (j <= i ? Lb[(size_t)i * ld + j] : 0.0) : (i == j ? 1.0 : 0.0);
            S[i * PLD + j] = v;
            if (i == j) invd[i] = 1.0 / v;
        }
    __syncthreads();
    double w[RB][RB];
    reg_trtri(w, S, invd, rowbuf);
#pragma unroll
    for (int r = 0; r < RB; ++r)
#pragma unroll
        for (int t = 0; t < RB; ++t) {
            const int i = ty + 16 * r, j = tx + 16 * t;
            if (i < jb && j < jb) Wb[i * PB + j] = j <= i ? w[r][t] : 0.0;
        }
}

__global__ void __launch_bounds__(PT, 1) trtri_blocks_kernel(const double* L, int nb, double* W) {
    const int b = blockIdx.x;
    const int j0 = b * PB;
    trtri_block(L + (size_t)j0 * nb + j0, nb, min(PB, nb - j0), W + (size_t)b * PB * PB);
}

// Batched: blockIdx.y selects the diagonal tile; W layout [tile][block][128][128].
__global__ void __launch_bounds__(PT, 1) trtri_batch_kernel(const double* const* Ls, int nb, double* W) {
    const int b = blockIdx.x, t = blockIdx.y;
    const int nblk = (nb + PB - 1) / PB;
    const int j0 = b * PB;
    trtri_block(Ls[t] + (size_t)j0 * nb + j0, nb, min(PB, nb - j0), W + ((size_t)t * nblk + b) * PB * PB);
}

static cudaError_t set_smem(const void* f, int bytes) {
    return cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
}

cudaError_t potrf_diag_block_launch(double* A, int lda, int jb, double* W, int col0, int* info,
                                    cudaStream_t s) {
    static bool init = false;
    if (!init) {
        cudaError_t e = set_smem((const void*)potrf_diag_block_kernel, RP_SMEM);
        if (e != cudaSuccess) return e;
        init = true;
    }
    potrf_diag_block_kernel<<<1, PT, RP_SMEM, s>>>(A, lda, jb, W, col0, info);
    return cudaGetLastError();
}

cudaError_t trtri_batch_launch(const double* const* Ls, int ntiles, int nb, double* W, cudaStream_t s) {
    static bool init = false;
    if (!init) {
        cudaError_t e = set_smem((const void*)trtri_batch_kernel, RP_SMEM);
        if (e != cudaSuccess) return e;
        init = true;
    }
    if (ntiles <= 0) return cudaSuccess;
    trtri_batch_kernel<<<dim3((nb + PB - 1) / PB, ntiles), PT, RP_SMEM, s>>>(Ls, nb, W);
    return cudaGetLastError();
}

cudaError_t trtri_blocks_launch(const double* L, int nb, double* W, cudaStream_t s) {
    static bool init = false;
    if (!init) {
        cudaError_t e = set_smem((const void*)trtri_blocks_kernel, RP_SMEM);
        if (e != cudaSuccess) return e;
        init = true;
    }
    trtri_blocks_kernel<<<(nb + PB - 1) / PB, PT, RP_SMEM, s>>>(L, nb, W);
    return cudaGetLastError();
}

}  // namespace mpgeo
