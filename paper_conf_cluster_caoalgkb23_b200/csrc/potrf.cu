// K3 helpers — FP64 Cholesky and triangular inverse of one <= 128 x 128 diagonal block held in
// shared memory.  The tile DPOTRF of Algorithm 1 ("D" = FP64 on diagonal tiles)
// and the panel TRSM are blocked right-looking loops whose bulk work is the DMMA GEMM
// (dgemm_dmma.cu); only these small sequential pieces live here.  The inverse W = L_bb^{-1} turns
// each block's triangular solve into a 128-wide GEMM (X_b = A_b W^T).
//
// One 128 x 129 FP64 smem array holds the block: L in the lower triangle, W^T in the strictly
// upper triangle, diag(W) in a side array, so L and W (264 KB together) fit in 132 KB.
//   Cholesky: right-looking, ONE barrier per column — the update of step c uses the unscaled
//     column c and 1/pivot; the column is scaled by 1/sqrt(pivot) during step c+1, when nobody
//     reads it any more.
//   Inverse:  Gauss-Jordan on [L | I]: for p, row p of W is final after dividing by L_pp and every
//     row i > p subtracts L_ip times it (n^3/6 FMAs spread over all threads, 2 barriers per p).
#include <math.h>

#include "common.cuh"
#include "kernels.h"

namespace mpgeo {

constexpr int PB = POTRF_IB;  // 128
constexpr int PLD = PB + 1;   // padded smem leading dimension
constexpr int PT = 256;       // threads
constexpr int P_SMEM = PB * PLD * 8 + 3 * PB * 8;

// Cholesky of S[0:n, 0:n] (lower) in place; pivots checked against `info`.
__device__ void smem_cholesky(double* S, double* piv, int n, int col0, int* info) {
    const int tid = threadIdx.x;
    const int tx = tid & 15, ty = tid >> 4;
    for (int c = 0; c < n; ++c) {
        const double d = S[c * PLD + c];
        if (tid == 0) {
            if (!(d > 0.0)) atomicMin(info, col0 + c + 1);
            piv[c] = sqrt(d);
        }
        if (c > 0) {  // finalise column c-1 (no longer read by anyone)
            const double inv = 1.0 / piv[c - 1];
            for (int i = c + tid; i < n; i += PT) S[i * PLD + c - 1] *= inv;
        }
        const double ip = 1.0 / d;
        for (int i = c + 1 + ty; i < n; i += 16) {
            const double lic = S[i * PLD + c] * ip;
            for (int j = c + 1 + tx; j <= i; j += 16) S[i * PLD + j] = fma(-lic, S[j * PLD + c], S[i * PLD + j]);
        }
        __syncthreads();
    }
    for (int c = tid; c < n; c += PT) S[c * PLD + c] = piv[c];
    __syncthreads();
}

// W = L^{-1} by Gauss-Jordan; W[i][c] (c < i) stored at S[c][i], W[i][i] in wd[i].
__device__ void smem_trtri_gj(double* S, double* wd, double* rowp, int n) {
    const int tid = threadIdx.x;
    for (int idx = tid; idx < n * n; idx += PT) {
        const int r = idx / n, c = idx - r * n;
        if (c > r) S[r * PLD + c] = 0.0;  // W starts as I (strict part)
    }
    for (int i = tid; i < n; i += PT) wd[i] = 1.0;
    __syncthreads();
    for (int p = 0; p < n; ++p) {
        // row p of W: entries c < p at S[c][p], diagonal wd[p]; scale by 1/L_pp into rowp
        const double ip = 1.0 / S[p * PLD + p];
        for (int c = tid; c <= p; c += PT) rowp[c] = (c < p ? S[c * PLD + p] : wd[p]) * ip;
        __syncthreads();
        for (int c = tid; c <= p; c += PT) {
            if (c < p) S[c * PLD + p] = rowp[c];
            else wd[p] = rowp[p];
        }
        // rows i > p: W[i][c] -= L_ip * W[p][c], c <= p; lanes run over i (conflict-free S[c][i]),
        // warps over c, L_ip kept in a register
        const int lane = tid & 31, wq = tid >> 5;
        for (int i = p + 1 + lane; i < n; i += 32) {
            const double l = S[i * PLD + p];
            for (int c = wq; c <= p; c += PT / 32) S[c * PLD + i] = fma(-l, rowp[c], S[c * PLD + i]);
        }
        __syncthreads();
    }
}

__device__ void write_block(const double* S, const double* wd, int n, double* A, int lda, double* W) {
    const int tid = threadIdx.x;
    for (int idx = tid; idx < n * n; idx += PT) {
        const int r = idx / n, c = idx - r * n;
        if (A) A[(size_t)r * lda + c] = (c <= r) ? S[r * PLD + c] : 0.0;
        if (W) W[r * PB + c] = (c < r) ? S[c * PLD + r] : (c == r ? wd[r] : 0.0);
    }
}

__global__ void __launch_bounds__(PT, 1)
    potrf_diag_block_kernel(double* A, int lda, int jb, double* W, int col0, int* info) {
    extern __shared__ double S[];
    double* piv = S + PB * PLD;
    double* wd = piv + PB;
    double* rowp = wd + PB;
    const int tid = threadIdx.x;
    for (int idx = tid; idx < jb * jb; idx += PT) {
        const int r = idx / jb, c = idx - r * jb;
        if (c <= r) S[r * PLD + c] = A[(size_t)r * lda + c];
    }
    __syncthreads();
    smem_cholesky(S, piv, jb, col0, info);
    smem_trtri_gj(S, wd, rowp, jb);
    write_block(S, wd, jb, A, lda, W);
}

__global__ void __launch_bounds__(PT, 1) trtri_blocks_kernel(const double* L, int nb, double* W) {
    extern __shared__ double S[];
    double* wd = S + PB * PLD + PB;
    double* rowp = wd + PB;
    const int b = blockIdx.x;
    const int j0 = b * PB;
    const int jb = min(PB, nb - j0);
    const double* Lb = L + (size_t)j0 * nb + j0;
    const int tid = threadIdx.x;
    for (int idx = tid; idx < jb * jb; idx += PT) {
        const int r = idx / jb, c = idx - r * jb;
        if (c <= r) S[r * PLD + c] = Lb[(size_t)r * nb + c];
    }
    __syncthreads();
    smem_trtri_gj(S, wd, rowp, jb);
    write_block(S, wd, jb, nullptr, 0, W + (size_t)b * PB * PB);
}

// Batched: blockIdx.y selects the diagonal tile; W layout [tile][block][128][128].
__global__ void __launch_bounds__(PT, 1) trtri_batch_kernel(const double* const* Ls, int nb, double* W) {
    extern __shared__ double S[];
    double* wd = S + PB * PLD + PB;
    double* rowp = wd + PB;
    const int b = blockIdx.x, t = blockIdx.y;
    const int nblk = (nb + PB - 1) / PB;
    const int j0 = b * PB;
    const int jb = min(PB, nb - j0);
    const double* Lb = Ls[t] + (size_t)j0 * nb + j0;
    const int tid = threadIdx.x;
    for (int idx = tid; idx < jb * jb; idx += PT) {
        const int r = idx / jb, c = idx - r * jb;
        if (c <= r) S[r * PLD + c] = Lb[(size_t)r * nb + c];
    }
    __syncthreads();
    smem_trtri_gj(S, wd, rowp, jb);
    write_block(S, wd, jb, nullptr, 0, W + ((size_t)t * nblk + b) * PB * PB);
}

static cudaError_t set_smem(const void* f, int bytes) {
    return cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
}

cudaError_t potrf_diag_block_launch(double* A, int lda, int jb, double* W, int col0, int* info,
                                    cudaStream_t s) {
    static bool init = false;
    if (!init) {
        cudaError_t e = set_smem((const void*)potrf_diag_block_kernel, P_SMEM);
        if (e != cudaSuccess) return e;
        init = true;
    }
    potrf_diag_block_kernel<<<1, PT, P_SMEM, s>>>(A, lda, jb, W, col0, info);
    return cudaGetLastError();
}

cudaError_t trtri_batch_launch(const double* const* Ls, int ntiles, int nb, double* W, cudaStream_t s) {
    static bool init = false;
    if (!init) {
        cudaError_t e = set_smem((const void*)trtri_batch_kernel, P_SMEM);
        if (e != cudaSuccess) return e;
        init = true;
    }
    if (ntiles <= 0) return cudaSuccess;
    trtri_batch_kernel<<<dim3((nb + PB - 1) / PB, ntiles), PT, P_SMEM, s>>>(Ls, nb, W);
    return cudaGetLastError();
}

cudaError_t trtri_blocks_launch(const double* L, int nb, double* W, cudaStream_t s) {
    static bool init = false;
    if (!init) {
        cudaError_t e = set_smem((const void*)trtri_blocks_kernel, P_SMEM);
        if (e != cudaSuccess) return e;
        init = true;
    }
    trtri_blocks_kernel<<<(nb + PB - 1) / PB, PT, P_SMEM, s>>>(L, nb, W);
    return cudaGetLastError();
}

}  // namespace mpgeo
