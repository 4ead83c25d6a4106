// K3 helpers — FP64 Cholesky and triangular inverse of one <=128 x 128 diagonal block in
// shared memory.  The tile DPOTRF of Algorithm 1 ("D" = FP64 on diagonal tiles,
// P:146) and the panel TRSM are blocked right-looking loops over 128-column
// blocks whose bulk work is the DMMA GEMM (dgemm_dmma.cu); only these small sequential
// pieces live here.  The inverse W = L_bb^{-1} turns each block's triangular solve into a
// 128-wide GEMM (X_b = A_b W^T), the usual GPU treatment of small diagonal blocks.
#include <math.h>

#include "common.cuh"
#include "kernels.h"

namespace mpgeo {

constexpr int PB = POTRF_IB;     // 128
constexpr int PLD = PB + 1;      // padded smem leading dimension
constexpr int PT = 256;          // threads
constexpr int P_SMEM = PB * PLD * 8;

// In-place inverse of the jb x jb lower-triangular S (ld PLD) by columns, last to first:
// L = [[l, 0], [x, L2]]  ->  L^{-1} = [[1/l, 0], [-(L2^{-1} x)/l, L2^{-1}]].
__device__ void smem_trtri_lower(double* S, int jb, double* tmp) {
    const int tid = threadIdx.x;
    for (int j = jb - 1; j >= 0; --j) {
        // tmp[i] = sum_{p=j+1..i} Winv[i][p] * x[p], x = S[j+1:, j] (old values)
        for (int i = j + 1 + tid; i < jb; i += PT) {
            double s = 0.0;
            for (int p = j + 1; p <= i; ++p) s = fma(S[i * PLD + p], S[p * PLD + j], s);
            tmp[i] = s;
        }
        __syncthreads();
        const double inv = 1.0 / S[j * PLD + j];
        for (int i = j + 1 + tid; i < jb; i += PT) S[i * PLD + j] = -inv * tmp[i];
        __syncthreads();
        if (tid == 0) S[j * PLD + j] = inv;
        __syncthreads();
    }
}

__global__ void __launch_bounds__(PT, 1)
    potrf_diag_block_kernel(double* A, int lda, int jb, double* W, int col0, int* info) {
    extern __shared__ double S[];
    double* tmp = S + PB * PLD;
    const int tid = threadIdx.x;
    for (int idx = tid; idx < jb * jb; idx += PT) {
        const int r = idx / jb, c = idx - r * jb;
        S[r * PLD + c] = (c <= r) ? A[(size_t)r * lda + c] : 0.0;
    }
    __syncthreads();
    const int tx = tid & 15, ty = tid >> 4;
    for (int c = 0; c < jb; ++c) {
        if (tid == 0) {
            const double d = S[c * PLD + c];
            if (!(d > 0.0)) atomicMin(info, col0 + c + 1);
            S[c * PLD + c] = sqrt(d);
        }
        __syncthreads();
        const double inv = 1.0 / S[c * PLD + c];
        for (int i = c + 1 + tid; i < jb; i += PT) S[i * PLD + c] *= inv;
        __syncthreads();
        for (int i = c + 1 + ty; i < jb; i += 16) {
            const double lic = S[i * PLD + c];
            for (int j = c + 1 + tx; j <= i; j += 16) S[i * PLD + j] = fma(-lic, S[j * PLD + c], S[i * PLD + j]);
        }
        __syncthreads();
    }
    // L back to the tile (upper part of the block zeroed)
    for (int idx = tid; idx < jb * jb; idx += PT) {
        const int r = idx / jb, c = idx - r * jb;
        A[(size_t)r * lda + c] = (c <= r) ? S[r * PLD + c] : 0.0;
    }
    __syncthreads();
    smem_trtri_lower(S, jb, tmp);
    for (int idx = tid; idx < jb * jb; idx += PT) {
        const int r = idx / jb, c = idx - r * jb;
        W[r * PB + c] = (c <= r) ? S[r * PLD + c] : 0.0;
    }
}

__global__ void __launch_bounds__(PT, 1) trtri_blocks_kernel(const double* L, int nb, double* W) {
    extern __shared__ double S[];
    double* tmp = S + PB * PLD;
    const int b = blockIdx.x;
    const int j0 = b * PB;
    const int jb = min(PB, nb - j0);
    const double* Lb = L + (size_t)j0 * nb + j0;
    double* Wb = W + (size_t)b * PB * PB;
    const int tid = threadIdx.x;
    for (int idx = tid; idx < jb * jb; idx += PT) {
        const int r = idx / jb, c = idx - r * jb;
        S[r * PLD + c] = (c <= r) ? Lb[(size_t)r * nb + c] : 0.0;
    }
    __syncthreads();
    smem_trtri_lower(S, jb, tmp);
    for (int idx = tid; idx < jb * jb; idx += PT) {
        const int r = idx / jb, c = idx - r * jb;
        Wb[r * PB + c] = (c <= r) ? S[r * PLD + c] : 0.0;
    }
}

static cudaError_t set_smem(const void* f, int bytes) {
    return cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
}

cudaError_t potrf_diag_block_launch(double* A, int lda, int jb, double* W, int col0, int* info,
                                    cudaStream_t s) {
    static bool init = false;
    const int smem = P_SMEM + PB * 8;
    if (!init) {
        cudaError_t e = set_smem((const void*)potrf_diag_block_kernel, smem);
        if (e != cudaSuccess) return e;
        init = true;
    }
    potrf_diag_block_kernel<<<1, PT, smem, s>>>(A, lda, jb, W, col0, info);
    return cudaGetLastError();
}

cudaError_t trtri_blocks_launch(const double* L, int nb, double* W, cudaStream_t s) {
    static bool init = false;
    const int smem = P_SMEM + PB * 8;
    if (!init) {
        cudaError_t e = set_smem((const void*)trtri_blocks_kernel, smem);
        if (e != cudaSuccess) return e;
        init = true;
    }
    trtri_blocks_kernel<<<(nb + PB - 1) / PB, PT, smem, s>>>(L, nb, W);
    return cudaGetLastError();
}

}  // namespace mpgeo
