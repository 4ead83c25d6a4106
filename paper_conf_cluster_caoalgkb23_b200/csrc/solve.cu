// K8 — the two reductions of Eq. (1): log|Sigma| = 2 sum log L_ii and
// Z^T Sigma^{-1} Z = y^T y with y = L^{-1} Z by tile forward substitution.  L is read in its
// storage precision, all arithmetic is FP64 (reading C15).  Every reduction has a fixed order
// (per-tile / per-chunk partials summed on the host in index order), so results are
// bit-reproducible run to run.
#include <math.h>

#include <algorithm>

#include "common.cuh"
#include "kernels.h"

namespace mpgeo {

constexpr int TS_T = 1024;  // trsv threads (32 warps)

// One FP64 lower tile: y = L^{-1} r, blocked by 32 rows.  Warp 0 solves each 32 x 32 diagonal
// block with shuffles; all warps then apply the block column to the rows below (warp per row,
// coalesced 256-byte row segments).  Padding rows are identity rows with r = 0.
__global__ void __launch_bounds__(TS_T, 1) trsv_tile_kernel(const double* L, int nb, const double* r, double* y) {
    extern __shared__ double sm[];
    double* rr = sm;  // nb
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (int i = tid; i < nb; i += TS_T) rr[i] = r[i];
    __syncthreads();
    for (int b = 0; b < nb; b += 32) {
        const int bw = min(32, nb - b);
        if (warp == 0) {
            double row[32];
            const int i = b + lane;
#pragma unroll
            for (int c = 0; c < 32; ++c) row[c] = (lane < bw && c < bw) ? L[(size_t)i * nb + b + c] : 0.0;
            double v = (lane < bw) ? rr[i] : 0.0;
#pragma unroll
            for (int c = 0; c < 32; ++c) {
                if (c < bw) {
                    double yc = (lane == c) ? v / row[c] : 0.0;
                    yc = __shfl_sync(0xffffffffu, yc, c);
                    if (lane == c) v = yc;
                    else if (lane > c) v = fma(-row[c], yc, v);
                }
            }
            if (lane < bw) rr[i] = v;  // rr now holds y for this block
        }
        __syncthreads();
        const double yl = (lane < bw) ? rr[b + lane] : 0.0;
        for (int i = b + bw + warp; i < nb; i += TS_T / 32) {
            double p = (lane < bw) ? L[(size_t)i * nb + b + lane] * yl : 0.0;
            p = warp_sum(p);
            if (lane == 0) rr[i] -= p;
        }
        __syncthreads();
    }
    for (int i = tid; i < nb; i += TS_T) y[i] = rr[i];
}

constexpr int GV_T = 256, GV_ROWS = 32;  // rows per CTA (8 warps x 4 rows)

__global__ void __launch_bounds__(GV_T) gemv_sub_kernel(const GemvTile* tiles, const double* y, int nb) {
    extern __shared__ double ys[];
    const GemvTile t = tiles[blockIdx.y];
    for (int i = threadIdx.x; i < nb; i += GV_T) ys[i] = y[i];
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int r0 = blockIdx.x * GV_ROWS;
    for (int rr = warp; rr < GV_ROWS; rr += GV_T / 32) {
        const int i = r0 + rr;
        if (i >= nb) break;
        double s = 0.0;
        if (t.prec == P64) {
            const double* row = (const double*)t.L + (size_t)i * nb;
            for (int c = 2 * lane; c < nb; c += 64) {
                const double2 v = *(const double2*)(row + c);
                s = fma(v.x, ys[c], s);
                s = fma(v.y, ys[c + 1], s);
            }
        } else if (t.prec == P16) {
            const __half* row = (const __half*)t.L + (size_t)i * nb;
            for (int c = 2 * lane; c < nb; c += 64) {
                const __half2 v = *(const __half2*)(row + c);
                s = fma(load16(__low2half(v), t.scale), ys[c], s);
                s = fma(load16(__high2half(v), t.scale), ys[c + 1], s);
            }
        } else {
            const float* row = (const float*)t.L + (size_t)i * nb;
            for (int c = 2 * lane; c < nb; c += 64) {
                const float2 v = *(const float2*)(row + c);
                s = fma((double)v.x, ys[c], s);
                s = fma((double)v.y, ys[c + 1], s);
            }
        }
        s = warp_sum(s);
        if (lane == 0) t.r[i] -= s;
    }
}

__global__ void logdiag_kernel(const double* const* diag, const int* nreal, int nb, double* out) {
    const double* L = diag[blockIdx.x];
    const int nr = nreal[blockIdx.x];
    double s = 0.0;
    for (int i = threadIdx.x; i < nr; i += blockDim.x) s += log(L[(size_t)i * nb + i]);
    __shared__ double red[32];
    s = warp_sum(s);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += red[w];
        out[blockIdx.x] = t;
    }
}

__global__ void sumsq_chunks_kernel(const double* v, int64_t n, int chunk, double* out) {
    const int64_t b0 = (int64_t)blockIdx.x * chunk;
    const int64_t b1 = min(n, b0 + chunk);
    double s = 0.0;
    for (int64_t i = b0 + threadIdx.x; i < b1; i += blockDim.x) s = fma(v[i], v[i], s);
    __shared__ double red[32];
    s = warp_sum(s);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += red[w];
        out[blockIdx.x] = t;
    }
}

// ---- blocked TRSV on one diagonal tile with the 128-block inverses W_j = L_jj^{-1}:
//   y_j = W_j r_j  (one CTA),  then  r_i -= L_ij y_j  for the rows below (many CTAs)
constexpr int TB = 128;

__global__ void __launch_bounds__(128) blk_matvec_kernel(const double* W, const double* r, double* y, int jb) {
    // warp per row, lanes over columns: y[i] = sum_c W[i][c] r[c]
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int i = warp; i < jb; i += 4) {
        double s = 0.0;
        for (int c = lane; c < jb; c += 32) s = fma(W[i * TB + c], r[c], s);
        s = warp_sum(s);
        if (lane == 0) y[i] = s;
    }
}

__global__ void __launch_bounds__(256) blk_update_kernel(const double* L, int nb, int j0, int jb, const double* y,
                                                         double* r, int row0) {
    // rows i = row0 + blockIdx.x*8 + warp: r[i] -= sum_c L[i][j0 + c] y[c]
    __shared__ double ys[TB];
    for (int c = threadIdx.x; c < jb; c += 256) ys[c] = y[c];
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int i = row0 + blockIdx.x * 8 + warp;
    if (i >= nb) return;
    const double* row = L + (size_t)i * nb + j0;
    double s = 0.0;
    for (int c = lane; c < jb; c += 32) s = fma(row[c], ys[c], s);
    s = warp_sum(s);
    if (lane == 0) r[i] -= s;
}

cudaError_t trsv_blocked_launch(const double* L, int nb, const double* Wk, double* r, double* y, cudaStream_t s) {
    for (int j0 = 0; j0 < nb; j0 += TB) {
        const int jb = nb - j0 < TB ? nb - j0 : TB;
        blk_matvec_kernel<<<1, 128, 0, s>>>(Wk + (size_t)(j0 / TB) * TB * TB, r + j0, y + j0, jb);
        const int rows = nb - (j0 + jb);
        if (rows > 0) blk_update_kernel<<<(rows + 7) / 8, 256, 0, s>>>(L, nb, j0, jb, y + j0, r, j0 + jb);
    }
    return cudaGetLastError();
}

cudaError_t trsv_tile_launch(const double* L, int nb, const double* r, double* y, cudaStream_t s) {
    const int smem = nb * 8;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(trsv_tile_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
    }
    trsv_tile_kernel<<<1, TS_T, smem, s>>>(L, nb, r, y);
    return cudaGetLastError();
}

cudaError_t gemv_sub_launch(const GemvTile* t, int ntiles, const double* y, int nb, cudaStream_t s) {
    if (ntiles <= 0) return cudaSuccess;
    const int smem = nb * 8;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(gemv_sub_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
    }
    dim3 grid((nb + GV_ROWS - 1) / GV_ROWS, ntiles);
    gemv_sub_kernel<<<grid, GV_T, smem, s>>>(t, y, nb);
    return cudaGetLastError();
}

cudaError_t logdiag_launch(const double* const* diag_tiles, const int* nreal, int ntiles, int nb, double* out,
                           cudaStream_t s) {
    if (ntiles <= 0) return cudaSuccess;
    logdiag_kernel<<<ntiles, 256, 0, s>>>(diag_tiles, nreal, nb, out);
    return cudaGetLastError();
}

__global__ void scale_vec_kernel(double* dst, const double* src, int64_t n, double a) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) dst[i] = a * src[i];
}

cudaError_t scale_vec_launch(double* dst, const double* src, int64_t n, double a, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    scale_vec_kernel<<<(unsigned)std::min<int64_t>((n + 255) / 256, 1184), 256, 0, s>>>(dst, src, n, a);
    return cudaGetLastError();
}

cudaError_t sumsq_chunks_launch(const double* v, int64_t n, int chunk, double* out, cudaStream_t s) {
    const int64_t nchunks = (n + chunk - 1) / chunk;
    if (nchunks <= 0) return cudaSuccess;
    sumsq_chunks_kernel<<<(unsigned)nchunks, 256, 0, s>>>(v, n, chunk, out);
    return cudaGetLastError();
}

}  // namespace mpgeo
