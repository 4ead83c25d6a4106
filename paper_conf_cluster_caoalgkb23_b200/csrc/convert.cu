// K2 — precision conversion of panel tiles.
//
// After TRSM(m, k) the tile L_mk exists once, in FP64, in the GPU's panel buffer.  panel_out
//   * writes it back to the tile pool in its storage precision (the factor the solve reads),
//   * rounds the panel copy to the communication precision comm(m, k) — what the successors
//     receive (STC when comm < storage, TTC otherwise; Algorithm 2).
// Once per panel and GPU, after the previous trailing update has released the (single-buffered)
// operand caches, the format kernels derive from the panel copy the operands its consuming GEMMs
// need: the row-scaled FP16 hi/lo split (FP16 class: hi; FP32 class as 3xFP16: hi + lo), the TF32
// hi/lo pair (FP32 class as 3xTF32) and, in crt.cu, the CRT residue planes (FP64 class).
// Consumers therefore convert on the GPU they run on (target-side conversion), but at most
// once per tile instead of once per GEMM.  All kernels are elementwise and HBM-bound.
#include "common.cuh"
#include "kernels.h"

namespace mpgeo {

constexpr int CV_T = 256;

__device__ __forceinline__ float tf32_rna(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return __uint_as_float(r);
}

__global__ void __launch_bounds__(CV_T) panel_in_kernel(const PanelTile* tiles, int64_t elems) {
    const PanelTile t = tiles[blockIdx.y];
    const int64_t stride = (int64_t)gridDim.x * CV_T * 2;
    for (int64_t i = ((int64_t)blockIdx.x * CV_T + threadIdx.x) * 2; i < elems; i += stride) {
        double2 v;
        if (t.store_prec == P64) {
            v = *(const double2*)((const double*)t.store + i);
        } else if (t.store_prec == P16) {
            const __half2 h = *(const __half2*)((const __half*)t.store + i);
            v = make_double2(load16(__low2half(h), t.scale), load16(__high2half(h), t.scale));
        } else {
            const float2 f = *(const float2*)((const float*)t.store + i);
            v = make_double2((double)f.x, (double)f.y);
        }
        *(double2*)(t.p64 + i) = v;
    }
}

__global__ void __launch_bounds__(CV_T) panel_out_kernel(const PanelTile* tiles, int64_t elems) {
    const PanelTile t = tiles[blockIdx.y];
    const int64_t stride = (int64_t)gridDim.x * CV_T * 2;
    for (int64_t i = ((int64_t)blockIdx.x * CV_T + threadIdx.x) * 2; i < elems; i += stride) {
        const double2 v = *(const double2*)(t.p64 + i);
        if (t.store_prec == P64) {
            *(double2*)((double*)t.store + i) = v;
        } else if (t.store_prec == P16) {  // FP16 storage class: the successors receive the stored values
            const __half h0 = store16(v.x, t.scale), h1 = store16(v.y, t.scale);
            *(__half2*)((__half*)t.store + i) = __halves2half2(h0, h1);
            *(double2*)(t.p64 + i) = make_double2(load16(h0, t.scale), load16(h1, t.scale));
            continue;
        } else {
            *(float2*)((float*)t.store + i) = make_float2(__double2float_rn(v.x), __double2float_rn(v.y));
        }
        if (t.comm_prec != P64) *(double2*)(t.p64 + i) = make_double2(round_to(v.x, t.comm_prec), round_to(v.y, t.comm_prec));
    }
}

// 3xTF32 operands of the FP32 class (reading C13): hi = rna_tf32(fp32(x)), lo = rna_tf32(fp32(x) - hi)
__global__ void __launch_bounds__(CV_T) tf32_split_kernel(const Tf32Item* items, int64_t elems) {
    const Tf32Item t = items[blockIdx.y];
    const int64_t stride = (int64_t)gridDim.x * CV_T * 2;
    for (int64_t i = ((int64_t)blockIdx.x * CV_T + threadIdx.x) * 2; i < elems; i += stride) {
        const double2 v = *(const double2*)(t.src + i);
        const float f0 = __double2float_rn(v.x), f1 = __double2float_rn(v.y);
        const float h0 = tf32_rna(f0), h1 = tf32_rna(f1);
        *(float2*)(t.hi + i) = make_float2(h0, h1);
        *(float2*)(t.lo + i) = make_float2(tf32_rna(f0 - h0), tf32_rna(f1 - h1));
    }
}

__global__ void round_copy_kernel(const double* src, double* dst, int64_t elems, int prec) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < elems; i += stride)
        dst[i] = round_to(src[i], prec);
}

__global__ void zero_upper_kernel(double* A, int nb) {
    const int r = blockIdx.x;
    for (int c = r + 1 + threadIdx.x; c < nb; c += blockDim.x) A[(size_t)r * nb + c] = 0.0;
}

// A = I (nb x nb): the right-hand side whose TRSM gives L~_kk^-T, the inverse factor of the
// low-precision-class TRSMs (engine.cu step 4b)
__global__ void identity_kernel(double* A, int nb) {
    const int r = blockIdx.x;
    for (int c = threadIdx.x; c < nb; c += blockDim.x) A[(size_t)r * nb + c] = c == r ? 1.0 : 0.0;
}

// dst = src^T (nb x nb FP64), 32 x 32 shared-memory tiles (coalesced reads and writes)
__global__ void __launch_bounds__(256) transpose_kernel(const double* __restrict__ src, double* __restrict__ dst, int nb) {
    __shared__ double t[32][33];
    const int bx = blockIdx.x * 32, by = blockIdx.y * 32;
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    for (int r = ty; r < 32; r += 8) t[r][tx] = src[(size_t)(by + r) * nb + bx + tx];
    __syncthreads();
    for (int r = ty; r < 32; r += 8) dst[(size_t)(bx + r) * nb + by + tx] = t[tx][r];
}

// Row-scaled FP16 operands (reading C13c): row i of the FP64 panel tile, rounded to FP32
// (the FP32-class operand), is scaled by 2^s_i with max_j |x_ij| 2^s_i < 2^15 and split into FP16
// hi = rn(x 2^s), lo = rn(x 2^s - hi) (x 2^s - hi is exact in FP32), i.e. the 11 + 11-bit split of
// 3xTF32, now within FP16 range; e_i = -s_i is stored for the GEMM epilogue.  hi + lo are the
// 3xFP16 FP32-class operands; hi alone is the FP16-class operand (FP16 = 11 significant bits, with
// the power-of-two row scale keeping small entries out of the FP16 subnormal range).  lo may be
// null (FP16 class only).  hs (optional, four-level maps' pure FP16 class) = rn(x 2^(s - 13)): the same
// row scale with the row max in [2, 4), so K = nb products of two such rows sum to <= K 2^4 < 65504 in an
// FP16 accumulator (tc_gemm KIND 3 multiplies by 2^(e_i + e_j + 26)).  One warp per row.
__global__ void __launch_bounds__(256) split16_kernel(const Split16Item* items, int nb) {
    const Split16Item it = items[blockIdx.y];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int row = blockIdx.x * 8 + warp;
    if (row >= nb) return;
    const double* x = it.src + (size_t)row * nb;
    float mx = 0.f;
    for (int j = lane * 2; j < nb; j += 64) {
        const double2 v = *(const double2*)(x + j);
        mx = fmaxf(mx, fmaxf(fabsf(__double2float_rn(v.x)), fabsf(__double2float_rn(v.y))));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    int e = 0;
    if (mx > 0.f) frexpf(mx, &e);  // mx < 2^e
    const int sc = min(max(15 - e, -100), 115);  // 2^sc and 2^-sc are normal FP32 numbers
    if (lane == 0) it.exps[row] = -sc;
    const float f = ldexpf(1.f, sc);
    __half* hi = it.hi ? it.hi + (size_t)row * nb : nullptr;
    __half* lo = it.lo ? it.lo + (size_t)row * nb : nullptr;
    __half* hs = it.hs ? it.hs + (size_t)row * nb : nullptr;
    for (int j = lane * 2; j < nb; j += 64) {
        const double2 v = *(const double2*)(x + j);
        const float a0 = __double2float_rn(v.x) * f, a1 = __double2float_rn(v.y) * f;
        const __half h0 = __float2half_rn(a0), h1 = __float2half_rn(a1);
        if (hi) *(__half2*)(hi + j) = __halves2half2(h0, h1);
        if (lo) *(__half2*)(lo + j) = __halves2half2(__float2half_rn(a0 - __half2float(h0)), __float2half_rn(a1 - __half2float(h1)));
        // pure-FP16 class operand: the row at max in [2, 4) (|sums| <= K 2^4 in an FP16 accumulator)
        if (hs) *(__half2*)(hs + j) = __halves2half2(__float2half_rn(a0 * 0x1p-13f), __float2half_rn(a1 * 0x1p-13f));
    }
}

cudaError_t split16_launch(const Split16Item* items, int n, int nb, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    if (nb % 64) return cudaErrorInvalidValue;
    split16_kernel<<<dim3((nb + 7) / 8, n), 256, 0, s>>>(items, nb);
    return cudaGetLastError();
}

cudaError_t identity_launch(double* A, int nb, cudaStream_t s) {
    identity_kernel<<<nb, 256, 0, s>>>(A, nb);
    return cudaGetLastError();
}

cudaError_t transpose_launch(const double* src, double* dst, int nb, cudaStream_t s) {
    if (nb % 32) return cudaErrorInvalidValue;
    transpose_kernel<<<dim3(nb / 32, nb / 32), 256, 0, s>>>(src, dst, nb);
    return cudaGetLastError();
}

static unsigned chunks_for(int64_t elems, int ntiles) {
    // about 4 waves of 148 SMs in total, at least one chunk per tile
    int64_t per = (4LL * 148 * 8 + ntiles - 1) / ntiles;
    const int64_t maxc = (elems / 2 + CV_T - 1) / CV_T;
    if (per > maxc) per = maxc;
    if (per < 1) per = 1;
    return (unsigned)per;
}

cudaError_t panel_in_launch(const PanelTile* t, int ntiles, int64_t elems, cudaStream_t s) {
    if (ntiles <= 0) return cudaSuccess;
    dim3 grid(chunks_for(elems, ntiles), ntiles);
    panel_in_kernel<<<grid, CV_T, 0, s>>>(t, elems);
    return cudaGetLastError();
}

cudaError_t panel_out_launch(const PanelTile* t, int ntiles, int64_t elems, cudaStream_t s) {
    if (ntiles <= 0) return cudaSuccess;
    dim3 grid(chunks_for(elems, ntiles), ntiles);
    panel_out_kernel<<<grid, CV_T, 0, s>>>(t, elems);
    return cudaGetLastError();
}

cudaError_t tf32_split_launch(const Tf32Item* t, int ntiles, int64_t elems, cudaStream_t s) {
    if (ntiles <= 0) return cudaSuccess;
    dim3 grid(chunks_for(elems, ntiles), ntiles);
    tf32_split_kernel<<<grid, CV_T, 0, s>>>(t, elems);
    return cudaGetLastError();
}

cudaError_t round_copy_launch(const double* src, double* dst, int64_t elems, int prec, cudaStream_t s) {
    round_copy_kernel<<<592, 256, 0, s>>>(src, dst, elems, prec);
    return cudaGetLastError();
}

cudaError_t zero_upper_launch(double* A, int nb, cudaStream_t s) {
    zero_upper_kernel<<<nb, 256, 0, s>>>(A, nb);
    return cudaGetLastError();
}

}  // namespace mpgeo
