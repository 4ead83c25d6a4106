// K5b — FP64-class tile GEMM emulated on INT8 tcgen05 tensor cores (Ozaki scheme, splitting
// variant).  SURVEY §8(f) item 4 ("FP64-class acceleration beyond the paper ... must keep the
// <= 1e-13 residual"); the FP64 class of Algorithm 1 (GEMM/SYRK at FP64).
//
// Split (once per panel tile and GPU, like the K2 conversions): for every row i of a tile with
// max_j |x_ij| < 2^{e_i},  x_ij 2^{-e_i} = sum_{s=1..S} d^{(s)}_ij 2^{-7 s} + r_ij,  |r_ij| < 2^{-7S},
// with int8 digits d^{(s)} in [-127, 127] obtained exactly by S rounds of "multiply by 128,
// take the integer part (toward zero), subtract" in FP64.
// Product: (A B^T)_ij = 2^{e_i + f_j} sum_{g=2}^{S+1} 2^{-7g} G_g,ij + (dropped terms),
//   G_g = sum_{s+t=g} D^{(s)}_A D^{(t)T}_B,
// every G_g exact in INT32 (|G_g| <= (g-1) * K * 127^2 < 2^31 for K <= 2048, S <= 8) and
// accumulated by tcgen05.mma kind::i8 directly in TMEM — one accumulator per g, 36 products for
// S = 8.  The dropped terms (s + t > S + 1) and residuals are below 2^{e_i + f_j - 7(S+1)} K,
// i.e. ~2^-52 of the row-max x column-max product scale for S = 8, K = 2048.
// Epilogue: G_g -> FP64 (exact), scaled by 2^{-7g} (exact), summed smallest first, multiplied by
// 2^{e_i + f_j} (exact), C -= result in FP64.
//
// CTA tile 128 x 64: 8 TMEM accumulators x 64 columns = all 512 TMEM columns; per k-step 12 MMAs of
// N = 64..256 (A slice s against the concatenated B slices 1..S+1-s) instead of 36 of N = 64, which
// cuts the shared-memory operand reads per MMA cycle by ~45%.  K-major int8
// operands, 64-byte rows with the 64-byte TMA/UMMA swizzle; one 3D TMA box brings all S slices of
// a 128 x 64 (A) or 64 x 64 (B) block; 2 stages of 96 KB.
#include <cudaTypedefs.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "common.cuh"
#include "ozaki.h"

namespace mpgeo {

// ------------------------------------------------------------------ split
// One warp per row; lanes cover 4 consecutive elements (char4 stores per slice plane).
__global__ void __launch_bounds__(256) ozaki_split_kernel(const OzSplitItem* items, int nb, int S) {
    const OzSplitItem it = items[blockIdx.y];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int row = blockIdx.x * 8 + warp;
    if (row >= nb) return;
    const double* x = it.src + (size_t)row * nb;
    double mx = 0.0;
    for (int j = lane; j < nb; j += 32) mx = fmax(mx, fabs(x[j]));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    int e = 0;
    if (mx > 0.0) frexp(mx, &e);  // mx = f 2^e, f in [0.5, 1)  =>  |x| < 2^e
    if (lane == 0) it.exps[row] = e;
    const size_t plane = (size_t)it.plane_stride;
    for (int j0 = lane * 4; j0 < nb; j0 += 128) {
        double y[4];
#pragma unroll
        for (int v = 0; v < 4; ++v) y[v] = (j0 + v < nb) ? ldexp(x[j0 + v], -e) : 0.0;
        for (int s = 0; s < S; ++s) {
            char4 d;
            int dv[4];
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                y[v] *= 128.0;
                dv[v] = (int)y[v];  // trunc toward zero, |y| < 128
                y[v] -= (double)dv[v];
            }
            d.x = (signed char)dv[0];
            d.y = (signed char)dv[1];
            d.z = (signed char)dv[2];
            d.w = (signed char)dv[3];
            *(char4*)(it.dst + s * plane + (size_t)row * nb + j0) = d;
        }
    }
}

cudaError_t ozaki_split_launch(const OzSplitItem* items, int n, int nb, int S, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    dim3 grid((nb + 7) / 8, n);
    ozaki_split_kernel<<<grid, 256, 0, s>>>(items, nb, S);
    return cudaGetLastError();
}

// ------------------------------------------------------------------ GEMM
constexpr int OZ_BM = 128, OZ_BK = 64, OZ_THREADS = 256;

struct __align__(64) OzParams {
    CUtensorMap a, b;  // 3D [S][rows][nb] int8, boxes {64, 128, S / CL} and {64, 64, S}
    const OzJob* jobs;
    const int* exps;   // row exponents of the slice cache rows [nt*nb]
    int nb, S, tiles_n, tiles_per_job, lower;
};

// S slices -> S TMEM accumulators of BN columns (S * BN = 512): S = 8 (FP64 class) uses 128 x 64
// tiles, S = 4 (FP32 class: the first 4 planes of the same split, 28 bits) uses 128 x 128 tiles.
template <int S>
struct OzCfg {
    static constexpr int BN = 512 / S;
    static constexpr int PER_MMA = 256 / BN;  // B slices concatenated per MMA (N <= 256)
    static constexpr int STAGES = S == 8 ? 2 : 3;  // 96 KB / 64 KB per stage
};

__device__ __forceinline__ uint32_t oz_smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void oz_mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void oz_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void oz_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "W_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra W_%=;\n\t}" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void oz_tma3d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1, int c2) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(dst),
        "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
        : "memory");
}
__device__ __forceinline__ void oz_tma3d_mc(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1, int c2,
                                            uint16_t mask) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1, {%3, %4, %5}], [%2], %6;" ::"r"(dst),
        "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "r"(c2), "h"(mask)
        : "memory");
}
__device__ __forceinline__ void oz_commit_mc(uint32_t bar, uint16_t mask) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(bar),
                 "h"(mask)
                 : "memory");
}
__device__ __forceinline__ void oz_cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t oz_cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void oz_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void oz_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void oz_commit(uint32_t bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
// K-major, 64-byte swizzle: 8-row x 64-byte atoms every 512 bytes (SBO), layout SWIZZLE_64B (4).
__device__ __forceinline__ uint64_t oz_desc(uint32_t saddr) {
    uint64_t d = (uint64_t)((saddr & 0x3FFFFu) >> 4);
    d |= (uint64_t)1 << 16;
    d |= (uint64_t)(512 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)4 << 61;
    return d;
}
// instruction descriptor: D = S32 (2), A = B = signed int8 (1), K-major, M = 128, N = n (16..256)
__device__ __forceinline__ uint32_t oz_idesc(int n) {
    return (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(OZ_BM >> 4) << 24);
}
__device__ __forceinline__ void oz_mma(uint32_t tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t accum) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
        "l"(a), "l"(b), "r"(idesc), "r"(accum));
}
__device__ __forceinline__ void oz_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// CL = CTAs per cluster along N (1 or 2).  With CL = 2 the two CTAs compute neighbouring 64-column
// blocks of the same 128 rows: each loads half of the A slice planes and multicasts them to both,
// and every MMA commit releases the stage in both CTAs (a stage is refilled only when both consumed it).
template <int S, int CL, bool CF32>
__global__ void __launch_bounds__(OZ_THREADS, 1) ozaki_gemm_kernel(const __grid_constant__ OzParams p) {
    constexpr int OZ_BN = OzCfg<S>::BN;
    constexpr int A_SL = OZ_BM * OZ_BK;     // bytes of one A slice block (8 KB)
    constexpr int B_SL = OZ_BN * OZ_BK;     // 4 KB (BN = 64) or 8 KB (BN = 128)
    constexpr int STAGE = S * (A_SL + B_SL);
    constexpr int OZ_STAGES = OzCfg<S>::STAGES;
    extern __shared__ uint8_t oz_smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)oz_smem_raw + 1023) & ~(uintptr_t)1023);
    __shared__ __align__(8) uint64_t full_bar[OZ_STAGES], empty_bar[OZ_STAGES], done_bar;
    __shared__ uint32_t tmem_slot;
    __shared__ double colscale[128];

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int job = blockIdx.x / p.tiles_per_job;
    const int t = blockIdx.x - job * p.tiles_per_job;
    const int bi = t / p.tiles_n, bj = t - bi * p.tiles_n;
    // strictly upper block of a SYRK (with CL = 2 both CTAs of a cluster exit together: BM = 2 BN)
    if (p.lower && (bj / CL) * CL * OZ_BN > bi * OZ_BM + OZ_BM - 1) return;
    const uint32_t crank = CL > 1 ? oz_cluster_rank() : 0;
    const OzJob jb = p.jobs[job];
    const int rowA = jb.m * p.nb + bi * OZ_BM;
    const int rowB = jb.n * p.nb + bj * OZ_BN;
    const int KB = p.nb / OZ_BK;

    if (threadIdx.x == 0) {
        for (int s = 0; s < OZ_STAGES; ++s) {
            oz_mbar_init(oz_smem_u32(&full_bar[s]), 1);
            oz_mbar_init(oz_smem_u32(&empty_bar[s]), CL);  // one MMA commit from every CTA of the cluster
        }
        oz_mbar_init(oz_smem_u32(&done_bar), 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(oz_smem_u32(&tmem_slot)),
                     "r"(512)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    if (threadIdx.x >= 64 && threadIdx.x < 64 + OZ_BN) {
        const int j = threadIdx.x - 64;
        colscale[j] = ldexp(1.0, p.exps[rowB + j]);
    }
    oz_fence_before();
    __syncthreads();
    if (CL > 1) oz_cluster_sync();  // peers' barriers are initialised before any multicast arrives
    oz_fence_after();
    const uint32_t tmem = tmem_slot;

    if (warp == 0 && lane == 0) {
        for (int kb = 0; kb < KB; ++kb) {
            const int s = kb % OZ_STAGES;
            const uint32_t ph = (uint32_t)(kb / OZ_STAGES) & 1u;
            oz_wait(oz_smem_u32(&empty_bar[s]), ph ^ 1u);
            const uint32_t st = oz_smem_u32(smem + s * STAGE);
            const uint32_t fb = oz_smem_u32(&full_bar[s]);
            oz_expect_tx(fb, STAGE);
            if (CL > 1) {
                constexpr int PL = S / CL;  // A planes loaded (and multicast) by this CTA
                oz_tma3d_mc(st + crank * PL * A_SL, &p.a, fb, kb * OZ_BK, rowA, (int)crank * PL, (uint16_t)((1u << CL) - 1));
            } else {
                oz_tma3d(st, &p.a, fb, kb * OZ_BK, rowA, 0);
            }
            oz_tma3d(st + S * A_SL, &p.b, fb, kb * OZ_BK, rowB, 0);
        }
    } else if (warp == 1 && lane == 0) {
        for (int kb = 0; kb < KB; ++kb) {
            const int s = kb % OZ_STAGES;
            const uint32_t ph = (uint32_t)(kb / OZ_STAGES) & 1u;
            oz_wait(oz_smem_u32(&full_bar[s]), ph);
            oz_fence_after();
            const uint32_t base = oz_smem_u32(smem + s * STAGE);
#pragma unroll
            for (int k = 0; k < OZ_BK / 32; ++k) {
                const uint32_t koff = k * 32;
                // For A slice s, the B slices t = 1 .. S+1-s are contiguous in shared memory: ONE MMA
                // with N = 64 (S+1-s) (split at N = 256) writes product (s, t) into TMEM columns
                // (s-1+t-1)*64 = (g-2)*64, exactly group g = s+t's accumulator.  The s = 1 MMAs
                // cover all 8 groups and initialise them (accumulate = 0) on the first k-step.
#pragma unroll
                for (int sa = 1; sa <= S; ++sa) {
                    const int nt_total = S + 1 - sa;  // number of B slices paired with sa
                    const uint64_t da = oz_desc(base + (sa - 1) * A_SL + koff);
#pragma unroll
                    for (int t0 = 0; t0 < nt_total; t0 += OzCfg<S>::PER_MMA) {  // N <= 256 per MMA
                        const int cnt = nt_total - t0 < OzCfg<S>::PER_MMA ? nt_total - t0 : OzCfg<S>::PER_MMA;
                        const uint64_t db = oz_desc(base + S * A_SL + t0 * B_SL + koff);
                        const uint32_t col = (uint32_t)(sa - 1 + t0) * OZ_BN;
                        const uint32_t acc = (kb | k) != 0 || sa != 1;
                        oz_mma(tmem + col, da, db, oz_idesc(cnt * OZ_BN), acc);
                    }
                }
            }
            if (CL > 1) oz_commit_mc(oz_smem_u32(&empty_bar[s]), (uint16_t)((1u << CL) - 1));
            else oz_commit(oz_smem_u32(&empty_bar[s]));
        }
        oz_commit(oz_smem_u32(&done_bar));
    } else if (warp >= 4) {
        oz_wait(oz_smem_u32(&done_bar), 0);
        oz_fence_after();
        const int q = warp - 4;
        const int row = bi * OZ_BM + q * 32 + lane;
        const uint32_t tl = (uint32_t)(q * 32) << 16;
        const double rs = ldexp(1.0, p.exps[rowA + q * 32 + lane]);
#pragma unroll 1
        for (int c0 = 0; c0 < OZ_BN; c0 += 32) {  // 32-column chunks: all groups, then C update
            double acc[32];
#pragma unroll
            for (int j = 0; j < 32; ++j) acc[j] = 0.0;
#pragma unroll 1
            for (int g = S + 1; g >= 2; --g) {  // smallest terms first
                const double sc = ldexp(1.0, -7 * g);
                uint32_t r[32];
                oz_ld32(tmem + tl + (uint32_t)((g - 2) * OZ_BN + c0), r);
#pragma unroll
                for (int v = 0; v < 32; ++v) acc[v] = fma((double)(int)r[v], sc, acc[v]);
            }
            if (CF32) {
                float* crow = (float*)jb.C + (size_t)row * p.nb + bj * OZ_BN + c0;
#pragma unroll
                for (int j = 0; j < 32; j += 4) {
                    float4 c = *(float4*)(crow + j);
                    c.x = (float)((double)c.x - acc[j] * rs * colscale[c0 + j]);
                    c.y = (float)((double)c.y - acc[j + 1] * rs * colscale[c0 + j + 1]);
                    c.z = (float)((double)c.z - acc[j + 2] * rs * colscale[c0 + j + 2]);
                    c.w = (float)((double)c.w - acc[j + 3] * rs * colscale[c0 + j + 3]);
                    *(float4*)(crow + j) = c;
                }
            } else {
                double* crow = (double*)jb.C + (size_t)row * p.nb + bj * OZ_BN + c0;
#pragma unroll
                for (int j = 0; j < 32; j += 2) {
                    double2 c = *(double2*)(crow + j);
                    c.x -= acc[j] * rs * colscale[c0 + j];
                    c.y -= acc[j + 1] * rs * colscale[c0 + j + 1];
                    *(double2*)(crow + j) = c;
                }
            }
        }
    }
    oz_fence_before();
    __syncthreads();
    if (CL > 1) oz_cluster_sync();  // no CTA leaves while its peer may still signal or fill it
    if (warp == 2) {
        oz_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
    }
}

static PFN_cuTensorMapEncodeTiled_v12000 oz_encode() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    if (!fn) {
        cudaDriverEntryPointQueryResult q;
        void* f = nullptr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (PFN_cuTensorMapEncodeTiled_v12000)f;
    }
    return fn;
}

static bool oz_map(CUtensorMap* m, const int8_t* base, uint64_t planes, uint64_t rows, uint64_t cols,
                   uint64_t plane_stride, uint32_t box_rows, uint32_t box_planes) {
    auto fn = oz_encode();
    if (!fn) return false;
    cuuint64_t dims[3] = {cols, rows, planes};
    cuuint64_t strides[2] = {cols, plane_stride};
    cuuint32_t box[3] = {(cuuint32_t)OZ_BK, box_rows, box_planes};
    cuuint32_t es[3] = {1, 1, 1};
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, const_cast<int8_t*>(base), dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <int S, int CL, bool CF32>
static cudaError_t oz_launch_s(const OzArgs& a, int njobs, cudaStream_t s) {
    constexpr int OZ_BN = OzCfg<S>::BN;
    constexpr int SMEM = OzCfg<S>::STAGES * S * (OZ_BM + OZ_BN) * OZ_BK + 1024;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(ozaki_gemm_kernel<S, CL, CF32>, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    OzParams p;
    memset(&p, 0, sizeof p);
    const uint64_t rows = (uint64_t)a.nt * a.nb;
    // the slice cache always holds 8 planes; an S-slice GEMM reads the first S (prefix-consistent split)
    if (!oz_map(&p.a, a.slices, 8, rows, a.nb, a.plane_stride, OZ_BM, S / CL) ||
        !oz_map(&p.b, a.slices, 8, rows, a.nb, a.plane_stride, OZ_BN, S))
        return cudaErrorInvalidValue;
    p.jobs = a.jobs;
    p.exps = a.exps;
    p.nb = a.nb;
    p.S = S;
    p.tiles_n = a.nb / OZ_BN;
    p.tiles_per_job = (a.nb / OZ_BM) * p.tiles_n;
    p.lower = a.lower;
    const long long grid = (long long)njobs * p.tiles_per_job;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(OZ_THREADS);
    cfg.dynamicSmemBytes = SMEM;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, ozaki_gemm_kernel<S, CL, CF32>, p);
}

cudaError_t ozaki_gemm_launch(const OzArgs& a, int njobs, cudaStream_t s) {
    if (njobs <= 0) return cudaSuccess;
    if (a.nb % OZ_BM || a.nb > 2048 * 4) return cudaErrorInvalidValue;
    static const int cl = [] {
        const char* e = getenv("MPGEO_OZAKI_CLUSTER");
        return e ? atoi(e) : 2;
    }();
    if (a.S == 8 && !a.c_f32) return cl == 2 ? oz_launch_s<8, 2, false>(a, njobs, s) : oz_launch_s<8, 1, false>(a, njobs, s);
    // S = 4: the 2-CTA multicast variant measured 2.6x slower than single-CTA (profiles/r01): no cluster
    if (a.S == 4 && a.c_f32) return oz_launch_s<4, 1, true>(a, njobs, s);
    return cudaErrorInvalidValue;  // S = 8 is the only validated split (FP64-level accuracy)
}

bool ozaki_available() { return oz_encode() != nullptr; }

}  // namespace mpgeo
