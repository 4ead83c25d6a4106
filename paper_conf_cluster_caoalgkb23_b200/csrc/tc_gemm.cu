// K6 / K7 — tcgen05 (5th-generation tensor core) tile GEMMs, sm_100a.
//
//   C_mn (FP32, nb x nb, row-major)  -=  P_m P_n^T        P = panel operand cache [nt*nb][nb]
//
// One CTA computes a 128 x BN block of C over the full K = nb:
//   warp 0 (1 lane)  TMA producer: 128-byte-swizzled K-major boxes into a STAGES-deep ring
//                    guarded by full/empty mbarriers;
//   warp 1 (1 lane)  MMA issuer: tcgen05.mma.cta_group::1 (M = 128, N = BN), accumulator in TMEM,
//                    tcgen05.commit releases each stage back to the producer;
//   warp 2           TMEM allocator (BN FP32 columns);
//   warps 4-7        epilogue: tcgen05.ld 32x32b (warp w reads TMEM lanes 32(w%4)..+31 = its rows),
//                    C -= acc with 16-byte loads/stores of the row.
// KIND 0 (FP16 class, "FP16_32"): kind::f16, BN = 256, BK = 64, 4 stages (48 KB each).
// KIND 1 (FP32 class, 3xTF32, reading C13): kind::tf32, BN = 256, BK = 32, 2 stages of
//   {A_hi, A_lo, B_hi, B_lo} (96 KB), 8 epilogue warps; per k-step three MMAs lo.hi + hi.lo + hi.hi; K is split in
//   chunks of 64 accumulated in two ping-pong TMEM accumulators and summed by the epilogue in FP32.
#include <cudaTypedefs.h>
#include <stdint.h>
#include <string.h>

#include "tc_gemm.h"

namespace mpgeo {

constexpr int TC_BM = 128;
template <int KIND>
struct TcThreads {
    static constexpr int EPI_WARPS = KIND == 0 ? 4 : 8;  // 3xTF32: two warpgroups, one per 128-column half
    static constexpr int N = (4 + EPI_WARPS) * 32;
};

struct __align__(64) TcParams {
    CUtensorMap a, b, a_lo, b_lo;
    const TcJob* jobs;
    int nb, tiles_n, tiles_per_job;
};

template <int KIND>
struct TcCfg {
    static constexpr int BN = 256;
    static constexpr int ESZ = KIND == 0 ? 2 : 4;
    static constexpr int BK = 128 / ESZ;          // elements per 128-byte row
    static constexpr int UK = KIND == 0 ? 16 : 8;  // K per tcgen05.mma (32 bytes)
    static constexpr int A_BYTES = TC_BM * 128;
    static constexpr int B_BYTES = BN * 128;
    static constexpr int STAGE_BYTES = KIND == 0 ? A_BYTES + B_BYTES : 2 * (A_BYTES + B_BYTES);
    static constexpr int STAGES = KIND == 0 ? 4 : 2;
    static constexpr int SMEM = STAGES * STAGE_BYTES + 1024;
    // KIND 1: accumulate CHUNK_KB k-blocks (64 of K) per TMEM accumulator, two accumulators
    // ping-pong; the epilogue sums the chunks in FP32 registers (round-to-nearest), which keeps
    // the tensor core's non-RN FP32 accumulation error from growing with K (reading C13).
    static constexpr int CHUNK_KB = KIND == 0 ? 1 << 20 : 2;
    static constexpr uint32_t TMEM_COLS = KIND == 0 ? BN : 2 * BN;  // power of two >= 32
    // instruction descriptor: D = F32 (bit 4), A/B format (bits 7-9 / 10-12), K-major both,
    // N >> 3 (bits 17-22), M >> 4 (bits 24-28)
    static constexpr uint32_t IDESC = (1u << 4) | ((KIND == 0 ? 0u : 2u) << 7) | ((KIND == 0 ? 0u : 2u) << 10) |
                                      ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(TC_BM >> 4) << 24);
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
        "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1)
        : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(uint32_t bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}

// K-major operand, 128-byte swizzle: 8-row x 128-byte atoms stacked every 1024 bytes (SBO),
// descriptor version 1 (bits 46-47), layout SWIZZLE_128B (bits 61-63 = 2).
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
    uint64_t d = (uint64_t)((saddr & 0x3FFFFu) >> 4);
    d |= (uint64_t)1 << 16;
    d |= (uint64_t)(1024 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}

template <int KIND>
__device__ __forceinline__ void tc_mma(uint32_t tmem, uint64_t a, uint64_t b, uint32_t accum) {
    if (KIND == 0) {
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(a), "l"(b), "r"(TcCfg<KIND>::IDESC), "r"(accum));
    } else {
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(a), "l"(b), "r"(TcCfg<KIND>::IDESC), "r"(accum));
    }
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
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

template <int KIND>
__global__ void __launch_bounds__(TcThreads<KIND>::N, 1) tc_gemm_kernel(const __grid_constant__ TcParams p) {
    using Cfg = TcCfg<KIND>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    __shared__ __align__(8) uint64_t full_bar[Cfg::STAGES], empty_bar[Cfg::STAGES], done_bar;
    __shared__ __align__(8) uint64_t acc_full[2], acc_empty[2];
    __shared__ uint32_t tmem_slot;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int job = blockIdx.x / p.tiles_per_job;
    const int t = blockIdx.x - job * p.tiles_per_job;
    const int bi = t / p.tiles_n, bj = t - bi * p.tiles_n;
    const TcJob jb = p.jobs[job];
    const int rowA = jb.m * p.nb + bi * TC_BM;
    const int rowB = jb.n * p.nb + bj * Cfg::BN;
    const int KB = p.nb / Cfg::BK;

    if (threadIdx.x == 0) {
        for (int s = 0; s < Cfg::STAGES; ++s) {
            mbar_init(smem_u32(&full_bar[s]), 1);
            mbar_init(smem_u32(&empty_bar[s]), 1);
        }
        mbar_init(smem_u32(&done_bar), 1);
        for (int i = 0; i < 2; ++i) {
            mbar_init(smem_u32(&acc_full[i]), 1);
            mbar_init(smem_u32(&acc_empty[i]), TcThreads<KIND>::EPI_WARPS);  // one arrive per epilogue warp
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&p.a) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&p.b) : "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_slot)),
                     "r"(Cfg::TMEM_COLS)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tmem_slot;

    if (warp == 0 && lane == 0) {
        // ---------------- TMA producer
        for (int kb = 0; kb < KB; ++kb) {
            const int s = kb % Cfg::STAGES;
            const uint32_t ph = (uint32_t)(kb / Cfg::STAGES) & 1u;
            mbar_wait(smem_u32(&empty_bar[s]), ph ^ 1u);
            const uint32_t st = smem_u32(smem + s * Cfg::STAGE_BYTES);
            const uint32_t fb = smem_u32(&full_bar[s]);
            mbar_expect_tx(fb, Cfg::STAGE_BYTES);
            const int kc = kb * Cfg::BK;
            if (KIND == 0) {
                tma_load_2d(st, &p.a, fb, kc, rowA);
                tma_load_2d(st + Cfg::A_BYTES, &p.b, fb, kc, rowB);
            } else {
                tma_load_2d(st, &p.a, fb, kc, rowA);
                tma_load_2d(st + Cfg::A_BYTES, &p.a_lo, fb, kc, rowA);
                tma_load_2d(st + 2 * Cfg::A_BYTES, &p.b, fb, kc, rowB);
                tma_load_2d(st + 2 * Cfg::A_BYTES + Cfg::B_BYTES, &p.b_lo, fb, kc, rowB);
            }
        }
    } else if (warp == 1 && lane == 0) {
        // ---------------- MMA issuer
        for (int kb = 0; kb < KB; ++kb) {
            const int s = kb % Cfg::STAGES;
            const uint32_t ph = (uint32_t)(kb / Cfg::STAGES) & 1u;
            const int chunk = kb / Cfg::CHUNK_KB, kin = kb % Cfg::CHUNK_KB;
            const uint32_t abuf = (uint32_t)(chunk & 1);
            const uint32_t dacc = KIND == 0 ? tmem : tmem + abuf * Cfg::BN;
            if (KIND == 1 && kin == 0) {  // wait until the epilogue drained this accumulator
                mbar_wait(smem_u32(&acc_empty[abuf]), ((uint32_t)(chunk >> 1) & 1u) ^ 1u);
                tc_fence_after();
            }
            mbar_wait(smem_u32(&full_bar[s]), ph);
            tc_fence_after();
            const uint32_t base = smem_u32(smem + s * Cfg::STAGE_BYTES);
#pragma unroll
            for (int k = 0; k < Cfg::BK / Cfg::UK; ++k) {
                const uint32_t koff = k * 32;  // bytes along K inside the 128-byte swizzle atom
                const uint32_t acc = (kin | k) != 0;
                if (KIND == 0) {
                    tc_mma<0>(dacc, desc_sw128(base + koff), desc_sw128(base + Cfg::A_BYTES + koff), acc);
                } else {
                    const uint64_t ahi = desc_sw128(base + koff);
                    const uint64_t alo = desc_sw128(base + Cfg::A_BYTES + koff);
                    const uint64_t bhi = desc_sw128(base + 2 * Cfg::A_BYTES + koff);
                    const uint64_t blo = desc_sw128(base + 2 * Cfg::A_BYTES + Cfg::B_BYTES + koff);
                    tc_mma<1>(dacc, alo, bhi, acc);  // small terms first
                    tc_mma<1>(dacc, ahi, blo, 1u);
                    tc_mma<1>(dacc, ahi, bhi, 1u);
                }
            }
            tc_commit(smem_u32(&empty_bar[s]));
            if (KIND == 1 && (kin == Cfg::CHUNK_KB - 1 || kb == KB - 1)) tc_commit(smem_u32(&acc_full[abuf]));
        }
        if (KIND == 0) tc_commit(smem_u32(&done_bar));
    } else if (warp >= 4) {
        // ---------------- epilogue: C -= acc.  Warp w reads TMEM lanes 32 (w % 4) .. +31 (its rows);
        // with 8 epilogue warps the two warpgroups split the columns in halves.
        constexpr int COLS = Cfg::BN / (TcThreads<KIND>::EPI_WARPS / 4);
        const int q = (warp - 4) & 3;
        const int half = (warp - 4) >> 2;
        const int row = bi * TC_BM + q * 32 + lane;
        float* crow = jb.C + (size_t)row * p.nb + bj * Cfg::BN + half * COLS;
        const uint32_t tl = ((uint32_t)(q * 32) << 16) + (uint32_t)(half * COLS);
        if (KIND == 0) {
            mbar_wait(smem_u32(&done_bar), 0);
            tc_fence_after();
#pragma unroll 1
            for (int c0 = 0; c0 < COLS; c0 += 32) {
                uint32_t r[32];
                tmem_ld32(tmem + tl + (uint32_t)c0, r);
                float4* cp = (float4*)(crow + c0);
#pragma unroll
                for (int v = 0; v < 8; ++v) {
                    float4 c = cp[v];
                    c.x -= __uint_as_float(r[4 * v + 0]);
                    c.y -= __uint_as_float(r[4 * v + 1]);
                    c.z -= __uint_as_float(r[4 * v + 2]);
                    c.w -= __uint_as_float(r[4 * v + 3]);
                    cp[v] = c;
                }
            }
        } else {
            float sum[COLS];
#pragma unroll
            for (int i = 0; i < COLS; ++i) sum[i] = 0.f;
            const int nchunks = (KB + Cfg::CHUNK_KB - 1) / Cfg::CHUNK_KB;
#pragma unroll 1
            for (int c = 0; c < nchunks; ++c) {
                const uint32_t abuf = (uint32_t)(c & 1);
                mbar_wait(smem_u32(&acc_full[abuf]), (uint32_t)(c >> 1) & 1u);
                tc_fence_after();
#pragma unroll
                for (int c0 = 0; c0 < COLS; c0 += 32) {
                    uint32_t r[32];
                    tmem_ld32(tmem + tl + abuf * Cfg::BN + (uint32_t)c0, r);
#pragma unroll
                    for (int v = 0; v < 32; ++v) sum[c0 + v] += __uint_as_float(r[v]);
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&acc_empty[abuf])) : "memory");
            }
#pragma unroll
            for (int c0 = 0; c0 < COLS; c0 += 4) {
                float4* cp = (float4*)(crow + c0);
                float4 cv = *cp;
                cv.x -= sum[c0];
                cv.y -= sum[c0 + 1];
                cv.z -= sum[c0 + 2];
                cv.w -= sum[c0 + 3];
                *cp = cv;
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS)
                     : "memory");
    }
}

// ------------------------------------------------------------------ host side
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
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

static bool make_map(CUtensorMap* m, const void* base, CUtensorMapDataType dt, int esz, uint64_t rows, uint64_t cols,
                     uint32_t box_cols, uint32_t box_rows) {
    auto fn = encode_fn();
    if (!fn) return false;
    cuuint64_t dims[2] = {cols, rows};
    cuuint64_t strides[1] = {cols * (cuuint64_t)esz};
    cuuint32_t box[2] = {box_cols, box_rows};
    cuuint32_t es[2] = {1, 1};
    return fn(m, dt, 2, const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool tc_gemm_available() { return encode_fn() != nullptr; }

template <int KIND>
static cudaError_t launch(const TcArgs& a, int njobs, cudaStream_t s) {
    using Cfg = TcCfg<KIND>;
    if (njobs <= 0) return cudaSuccess;
    if (a.nb % Cfg::BN || a.nb % TC_BM) return cudaErrorInvalidValue;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(tc_gemm_kernel<KIND>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    TcParams p;
    memset(&p, 0, sizeof p);
    const uint64_t rows = (uint64_t)a.nt * a.nb;
    bool ok;
    if (KIND == 0) {
        ok = make_map(&p.a, a.p16, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, rows, a.nb, Cfg::BK, TC_BM) &&
             make_map(&p.b, a.p16, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, rows, a.nb, Cfg::BK, Cfg::BN);
    } else {
        ok = make_map(&p.a, a.hi, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, rows, a.nb, Cfg::BK, TC_BM) &&
             make_map(&p.a_lo, a.lo, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, rows, a.nb, Cfg::BK, TC_BM) &&
             make_map(&p.b, a.hi, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, rows, a.nb, Cfg::BK, Cfg::BN) &&
             make_map(&p.b_lo, a.lo, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, rows, a.nb, Cfg::BK, Cfg::BN);
    }
    if (!ok) return cudaErrorInvalidValue;
    p.jobs = a.jobs;
    p.nb = a.nb;
    p.tiles_n = a.nb / Cfg::BN;
    p.tiles_per_job = (a.nb / TC_BM) * p.tiles_n;
    const long long grid = (long long)njobs * p.tiles_per_job;
    if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    tc_gemm_kernel<KIND><<<(unsigned)grid, TcThreads<KIND>::N, Cfg::SMEM, s>>>(p);
    return cudaGetLastError();
}

cudaError_t tc_gemm_f16_launch(const TcArgs& a, int njobs, cudaStream_t s) { return launch<0>(a, njobs, s); }
cudaError_t tc_gemm_tf32x3_launch(const TcArgs& a, int njobs, cudaStream_t s) { return launch<1>(a, njobs, s); }

}  // namespace mpgeo
