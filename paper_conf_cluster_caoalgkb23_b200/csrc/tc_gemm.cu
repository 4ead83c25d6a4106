// K6 / K7 — tcgen05 (5th-generation tensor core) tile GEMMs, sm_100a.
//
//   C_mn (FP32, nb x nb, row-major)  -=  P_m P_n^T        P = panel operand cache [nt*nb][nb]
//
// A CTA pair (cluster of 2 on one TPC, tcgen05.mma.cta_group::2, M = 256) computes a 256 x 256
// block of C over the full K = nb (CL = 1: one CTA, M = 128, 128 x 256):
//   warp 0 (1 lane)  TMA producer: 128-byte-swizzled K-major boxes into a multi-stage ring guarded
//                    by full/empty mbarriers; each CTA loads its 128 rows of A and its half of B,
//                    the bytes of both CTAs complete on the leader's full barrier;
//   warp 1 (1 lane)  MMA issuer (leader CTA only): accumulator in TMEM, tcgen05.commit (multicast
//                    to both CTAs) releases each stage and publishes finished accumulators;
//   warp 2           TMEM allocator;
//   warps 4-..       epilogue: tcgen05.ld 32x32b (warp w reads TMEM lanes 32(w%4)..+31 = its rows),
//                    -acc staged in shared memory (128-byte swizzle) and reduced into C with
//                    cp.reduce.async.bulk.tensor .add (one add per element: RN(C - acc)).
// KIND 0 (FP16 class, "FP16_32"): kind::f16, BK = 64, 96 KB of stages so two CTAs share an SM;
//   the operands are the row-scaled FP16 hi planes of the 3xFP16 split and the epilogue multiplies
//   by 2^(eA_i + eB_j) (exact), so tiny FP16-class entries keep 11 bits relative to their row.
// KIND 1 (FP32 class, 3xTF32, reading C13): kind::tf32, BK = 32, stages of {A_hi, A_lo, B_hi, B_lo},
//   8 epilogue warps; per k-step three MMAs lo.hi + hi.lo + hi.hi; K is split in chunks of 64
//   accumulated in two ping-pong TMEM accumulators and summed by the epilogue in FP32.
// KIND 2 (FP32 class, 3xFP16, reading C13c): the same three products with an 11-bit hi/lo split in
//   FP16 (kind::f16, twice the TF32 rate): each panel row is scaled by a power of two so its max is
//   below 2^15 (split16_kernel, convert.cu); the epilogue multiplies by 2^(eA_i + eB_j).
// KIND 3 (the paper's pure FP16 class, "A, B, C, and operation are all in FP16"; four-level
//   maps): KIND 0 with an F16 accumulator (idesc dtype F16) over the whole K; the
//   operands are the hs planes of split16_kernel (row max in [2, 4), so |sum| <= K 2^4 stays inside
//   FP16's range), the epilogue widens the FP16 result to FP32 and multiplies by 2^(eA_i + eB_j + 26).
#include <cudaTypedefs.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "tc_gemm.h"

namespace mpgeo {

constexpr int TC_BM = 128;  // output rows per CTA (TMEM lanes)
#ifndef TC16X3_EPI_WARPS
#define TC16X3_EPI_WARPS 8
#endif
#ifndef TC16X3_CHUNK_KB
#define TC16X3_CHUNK_KB 2  // KIND 2: k-blocks of 64 per TMEM accumulator chunk (K = 128; measured 187 vs 181 Tflop/s at K = 64)
#endif
// TMEM layout of an F16 accumulator (tools/dbg/tmem_f16acc.cu): 0 = one FP16 per 32-bit column (low
// half), 1 = two per column
#ifndef TC_F16ACC_PACKED
#define TC_F16ACC_PACKED 0
#endif
template <int KIND>
struct TcThreads {
    // 3xTF32: two warpgroups, one per 128-column half; 3xFP16: TC16X3_EPI_WARPS / 4 column groups
    static constexpr int EPI_WARPS = (KIND == 0 || KIND == 3) ? 4 : KIND == 1 ? 8 : TC16X3_EPI_WARPS;
    static constexpr int N = (4 + EPI_WARPS) * 32;
};

struct __align__(64) TcParams {
    CUtensorMap a, b, a_lo, b_lo, c;
    const TcJob* jobs;
    const char* cbase;
    const int* exps;  // per panel-cache row, 2^exps undoes the operand's power-of-two row scale
    int nb, tiles_n, tiles_per_job;
    int total;        // persistent kernel: pair tiles of the launch
    int c16;          // KIND 0: FP16 C tiles (FP16 storage class)
};

// CL = CTAs per MMA: 1 (tcgen05.mma.cta_group::1, M = 128) or 2 (a CTA pair on one TPC,
// cta_group::2, M = 256).  In a pair each CTA loads its own 128 rows of A and half (BN / 2 rows) of
// B; the MMA reads B from both CTAs' shared memory, so every byte fetched from L2 feeds twice the
// flops (the single-CTA kernel is bound by L2 -> SM bandwidth, profiles/r01).
template <int KIND, int CL>
struct TcCfg {
    static constexpr int BN = 256;                 // MMA N = output columns per CTA
    static constexpr int BM = TC_BM * CL;          // MMA M = output rows per cluster
    static constexpr int ESZ = KIND == 1 ? 4 : 2;
    static constexpr int BK = 128 / ESZ;           // elements per 128-byte row
    static constexpr int UK = KIND == 1 ? 8 : 16;  // K per tcgen05.mma (32 bytes)
    static constexpr int A_BYTES = TC_BM * 128;
    static constexpr int B_BYTES = (BN / CL) * 128;
    static constexpr bool ONE = KIND == 0 || KIND == 3;  // one operand plane each (FP16 class, pure FP16)
    static constexpr int STAGE_BYTES = ONE ? A_BYTES + B_BYTES : 2 * (A_BYTES + B_BYTES);
    // KIND 0: 96 KB of stages so two CTAs share an SM (one's epilogue overlaps the other's main
    // loop; 2 x 256 TMEM columns); KIND 1: 192 KB, one CTA per SM (512 TMEM columns)
    static constexpr int STAGES = (ONE ? 96 * 1024 : 192 * 1024) / STAGE_BYTES;
    static constexpr int MIN_BLOCKS = ONE ? 2 : 1;
    static constexpr int SMEM = STAGES * STAGE_BYTES + 1024;
    // KIND 1: accumulate CHUNK_KB k-blocks (64 of K) per TMEM accumulator, two accumulators
    // ping-pong; the epilogue sums the chunks in FP32 registers (round-to-nearest), which keeps
    // the tensor core's non-RN FP32 accumulation error from growing with K (reading C13).
    static constexpr int CHUNK_KB = ONE ? 1 << 20 : KIND == 1 ? 2 : TC16X3_CHUNK_KB;
    static constexpr uint32_t TMEM_COLS = ONE ? BN : 2 * BN;  // power of two >= 32
    // instruction descriptor: D = F32 (bit 4), A/B format (bits 7-9 / 10-12), K-major both,
    // N >> 3 (bits 17-22), M >> 4 (bits 24-28)
    static constexpr uint32_t IDESC = ((KIND == 3 ? 0u : 1u) << 4) | ((KIND == 1 ? 2u : 0u) << 7) | ((KIND == 1 ? 2u : 0u) << 10) |
                                      ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
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
// shared::cluster address of the same shared variable in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t cluster_addr(uint32_t saddr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
    return r;
}
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cbar) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cbar) : "memory");
}
// relaxed arrive: the epilogue only signals that its tcgen05.ld of the accumulator completed
// (wait::ld), which orders nothing else, so no release (a release adds a MEMBAR per chunk: 21% of
// the 3xFP16 kernel's stalls, profiles/r01/s4_ncu_f16x3_summary.txt)
__device__ __forceinline__ void mbar_arrive_cluster_relaxed(uint32_t cbar) {
    asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(cbar) : "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// TMA 2D load into this CTA's shared memory; with CL = 2 the completion is signalled on the
// leader CTA's mbarrier (cta_group::2 form), which the leader's MMA issuer waits on.
template <int CL>
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1) {
    if (CL == 1)
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
            "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1)
            : "memory");
    else
        asm volatile(
            "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
            "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1)
            : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
// MMA-completion arrive: CL = 1 on this CTA's barrier; CL = 2 on the barrier at the same offset in
// both CTAs of the pair
template <int CL>
__device__ __forceinline__ void tc_commit(uint32_t bar) {
    if (CL == 1)
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
    else
        asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(bar),
                     "h"((uint16_t)3)
                     : "memory");
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

template <int KIND, int CL>
__device__ __forceinline__ void tc_mma(uint32_t tmem, uint64_t a, uint64_t b, uint32_t accum) {
    constexpr uint32_t ID = TcCfg<KIND, CL>::IDESC;
    if (KIND != 1 && CL == 1)
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(a), "l"(b), "r"(ID), "r"(accum));
    else if (KIND != 1)
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(a), "l"(b), "r"(ID), "r"(accum));
    else if (CL == 1)
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(a), "l"(b), "r"(ID), "r"(accum));
    else
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(a), "l"(b), "r"(ID), "r"(accum));
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

// 16 consecutive 32-bit TMEM columns of the warp's 32 lanes (KIND 3 with packed FP16 accumulators)
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// C -= acc through the TMA unit: the warp stages -acc for a 32 x 32 box in shared memory
// (128-byte swizzle: 16-byte chunk j of row r at chunk j ^ (r & 7), conflict-free for the
// row-per-lane writes) and one lane issues a bulk tensor reduce-add into global C.  Each element
// of C receives exactly one add, so the result is RN(C - acc), as with a load / subtract / store.
__device__ __forceinline__ void stage_box_neg(uint32_t buf, int lane, const float* v) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        const uint32_t a = buf + (uint32_t)lane * 128u + ((uint32_t)(j ^ (lane & 7)) << 4);
        asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(a), "f"(-v[4 * j]), "f"(-v[4 * j + 1]),
                     "f"(-v[4 * j + 2]), "f"(-v[4 * j + 3])
                     : "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
}
// 3xFP16: v_j *= 2^(e_row) 2^(e_col j) for one 32-column group (exponents in [-115, 100], so each
// power of two is built from its bits)
__device__ __forceinline__ void scale_group(float* v, float ra, const int4* eb) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        const int4 e4 = __ldg(eb + i);
        v[4 * i] = (v[4 * i] * ra) * __int_as_float((e4.x + 127) << 23);
        v[4 * i + 1] = (v[4 * i + 1] * ra) * __int_as_float((e4.y + 127) << 23);
        v[4 * i + 2] = (v[4 * i + 2] * ra) * __int_as_float((e4.z + 127) << 23);
        v[4 * i + 3] = (v[4 * i + 3] * ra) * __int_as_float((e4.w + 127) << 23);
    }
}
// FP16 C (FP16 storage class): -v 2^cscale as FP16 into a 32 x 32 box with 64-byte rows (64-byte swizzle:
// 16-byte chunk j of row r at chunk j ^ ((r >> 1) & 3)); v already carries the operands' row scales
__device__ __forceinline__ void stage_box_neg16(uint32_t buf, int lane, const float* v, float cs) {
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        uint32_t w[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const __half2 h = __floats2half2_rn(-v[8 * j + 2 * i] * cs, -v[8 * j + 2 * i + 1] * cs);
            w[i] = *(const uint32_t*)&h;
        }
        const uint32_t a = buf + (uint32_t)lane * 64u + ((uint32_t)(j ^ ((lane >> 1) & 3)) << 4);
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3])
                     : "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
}
__device__ __forceinline__ void tma_reduce_add(const CUtensorMap* map, uint32_t buf, int c0, int c1) {
    asm volatile("cp.reduce.async.bulk.tensor.2d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                     (uint64_t)map),
                 "r"(buf), "r"(c0), "r"(c1)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read_1() { asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

template <int CL>
__device__ __forceinline__ void tmem_alloc(uint32_t slot, uint32_t cols) {
    if (CL == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(slot), "r"(cols) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    } else {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(slot), "r"(cols) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
}
template <int CL>
__device__ __forceinline__ void tmem_dealloc(uint32_t tmem, uint32_t cols) {
    if (CL == 1)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(cols) : "memory");
    else
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(cols) : "memory");
}

template <int KIND, int CL>
__global__ void __launch_bounds__(TcThreads<KIND>::N, TcCfg<KIND, CL>::MIN_BLOCKS) tc_gemm_kernel(const __grid_constant__ TcParams p) {
    using Cfg = TcCfg<KIND, CL>;
    constexpr int EPI_WARPS = TcThreads<KIND>::EPI_WARPS;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    __shared__ __align__(8) uint64_t full_bar[Cfg::STAGES], empty_bar[Cfg::STAGES], done_bar;
    __shared__ __align__(8) uint64_t acc_full[2], acc_empty[2];
    __shared__ uint32_t tmem_slot;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t crank = CL > 1 ? cluster_rank() : 0;
    const int cta = blockIdx.x / CL;  // output block (one per CTA pair when CL = 2)
    const int job = cta / p.tiles_per_job;
    const int t = cta - job * p.tiles_per_job;
    const int bi = t / p.tiles_n, bj = t - bi * p.tiles_n;
    const TcJob jb = p.jobs[job];
    const int rowA = jb.m * p.nb + bi * Cfg::BM + (int)crank * TC_BM;
    const int rowB = jb.n * p.nb + bj * Cfg::BN + (int)crank * (Cfg::BN / CL);
    const int KB = p.nb / Cfg::BK;

    if (threadIdx.x == 0) {
        for (int s = 0; s < Cfg::STAGES; ++s) {
            mbar_init(smem_u32(&full_bar[s]), 1);   // leader: its producer's arrive + both CTAs' bytes
            mbar_init(smem_u32(&empty_bar[s]), 1);  // the leader's MMA commit
        }
        mbar_init(smem_u32(&done_bar), 1);
        for (int i = 0; i < 2; ++i) {
            mbar_init(smem_u32(&acc_full[i]), 1);
            mbar_init(smem_u32(&acc_empty[i]), CL * EPI_WARPS);  // one arrive per epilogue warp of the pair
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&p.a) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&p.b) : "memory");
    }
    if (warp == 2) tmem_alloc<CL>(smem_u32(&tmem_slot), Cfg::TMEM_COLS);
    tc_fence_before();
    if (CL > 1) cluster_sync();  // the peer's barriers exist before any remote arrive / multicast
    else __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tmem_slot;

    if (warp == 0 && lane == 0) {
        // ---------------- TMA producer (every CTA loads its own A rows and its share of B)
        for (int kb = 0; kb < KB; ++kb) {
            const int s = kb % Cfg::STAGES;
            const uint32_t ph = (uint32_t)(kb / Cfg::STAGES) & 1u;
            mbar_wait(smem_u32(&empty_bar[s]), ph ^ 1u);
            const uint32_t st = smem_u32(smem + s * Cfg::STAGE_BYTES);
            const uint32_t lb = smem_u32(&full_bar[s]);
            const uint32_t fb = CL > 1 ? cluster_addr(lb, 0) : lb;
            if (crank == 0) mbar_expect_tx(lb, CL * Cfg::STAGE_BYTES);
            const int kc = kb * Cfg::BK;
            if (Cfg::ONE) {
                tma_load_2d<CL>(st, &p.a, fb, kc, rowA);
                tma_load_2d<CL>(st + Cfg::A_BYTES, &p.b, fb, kc, rowB);
            } else {
                tma_load_2d<CL>(st, &p.a, fb, kc, rowA);
                tma_load_2d<CL>(st + Cfg::A_BYTES, &p.a_lo, fb, kc, rowA);
                tma_load_2d<CL>(st + 2 * Cfg::A_BYTES, &p.b, fb, kc, rowB);
                tma_load_2d<CL>(st + 2 * Cfg::A_BYTES + Cfg::B_BYTES, &p.b_lo, fb, kc, rowB);
            }
        }
    } else if (warp == 1 && lane == 0 && crank == 0) {
        // ---------------- MMA issuer (the leader CTA issues for the pair)
        for (int kb = 0; kb < KB; ++kb) {
            const int s = kb % Cfg::STAGES;
            const uint32_t ph = (uint32_t)(kb / Cfg::STAGES) & 1u;
            const int chunk = kb / Cfg::CHUNK_KB, kin = kb % Cfg::CHUNK_KB;
            const uint32_t abuf = (uint32_t)(chunk & 1);
            const uint32_t dacc = Cfg::ONE ? tmem : tmem + abuf * Cfg::BN;
            if (!Cfg::ONE && kin == 0) {  // wait until the epilogues drained this accumulator
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
                if (Cfg::ONE) {
                    tc_mma<KIND, CL>(dacc, desc_sw128(base + koff), desc_sw128(base + Cfg::A_BYTES + koff), acc);
                } else {
                    const uint64_t ahi = desc_sw128(base + koff);
                    const uint64_t alo = desc_sw128(base + Cfg::A_BYTES + koff);
                    const uint64_t bhi = desc_sw128(base + 2 * Cfg::A_BYTES + koff);
                    const uint64_t blo = desc_sw128(base + 2 * Cfg::A_BYTES + Cfg::B_BYTES + koff);
                    tc_mma<KIND, CL>(dacc, alo, bhi, acc);  // small terms first
                    tc_mma<KIND, CL>(dacc, ahi, blo, 1u);
                    tc_mma<KIND, CL>(dacc, ahi, bhi, 1u);
                }
            }
            tc_commit<CL>(smem_u32(&empty_bar[s]));
            if (!Cfg::ONE && (kin == Cfg::CHUNK_KB - 1 || kb == KB - 1)) tc_commit<CL>(smem_u32(&acc_full[abuf]));
        }
        if (Cfg::ONE) tc_commit<CL>(smem_u32(&done_bar));
    } else if (warp >= 4) {
        // ---------------- epilogue: C -= acc.  Warp w reads TMEM lanes 32 (w % 4) .. +31 (its rows);
        // with 8 epilogue warps the two warpgroups split the columns in halves.  The stage ring is
        // idle once the last accumulator is complete, so it doubles as the staging buffer.
        constexpr int COLS = Cfg::BN / (EPI_WARPS / 4);
        const int q = (warp - 4) & 3;
        const int half = (warp - 4) >> 2;
        const int crow0 = (int)(((const char*)jb.C - p.cbase) / ((size_t)p.nb * (p.c16 ? 2 : 4))) + bi * Cfg::BM +
                          (int)crank * TC_BM + q * 32;
        const int ccol0 = bj * Cfg::BN + half * COLS;
        const uint32_t tl = ((uint32_t)(q * 32) << 16) + (uint32_t)(half * COLS);
        const uint32_t stg = smem_u32(smem) + (uint32_t)(warp - 4) * 8192u;  // two 4 KB boxes per warp
        if (Cfg::ONE) {
            // KIND 3: the hs planes carry an extra 2^-13 per operand (split16_kernel)
            const float ra = __int_as_float((p.exps[rowA + q * 32 + lane] + (KIND == 3 ? 26 : 0) + 127) << 23);
            const int4* eb = (const int4*)(p.exps + jb.n * p.nb + ccol0);
            mbar_wait(smem_u32(&done_bar), 0);
            tc_fence_after();
#pragma unroll 1
            for (int g = 0; g < COLS / 32; ++g) {
                uint32_t r[32];
                float v[32];
                if (KIND == 3 && TC_F16ACC_PACKED) {  // two FP16 accumulators per 32-bit TMEM column
                    tmem_ld16(tmem + tl + (uint32_t)(g * 16), r);
#pragma unroll
                    for (int i = 0; i < 16; ++i) {
                        const float2 f = __half22float2(*(const __half2*)&r[i]);
                        v[2 * i] = f.x;
                        v[2 * i + 1] = f.y;
                    }
                } else {
                    tmem_ld32(tmem + tl + (uint32_t)(g * 32), r);
#pragma unroll
                    for (int i = 0; i < 32; ++i)
                        v[i] = KIND == 3 ? __half2float(__ushort_as_half((unsigned short)(r[i] & 0xffffu))) : __uint_as_float(r[i]);
                }
                const uint32_t buf = stg + (uint32_t)(g & 1) * 4096u;
                if (g >= 2) {
                    if (lane == 0) bulk_wait_read_1();
                    __syncwarp();
                }
                scale_group(v, ra, eb + g * 8);  // undo the operands' power-of-two row scales
                if (p.c16) stage_box_neg16(buf, lane, v, __int_as_float((jb.cscale + 127) << 23));
                else stage_box_neg(buf, lane, v);
                if (lane == 0) tma_reduce_add(&p.c, buf, ccol0 + g * 32, crow0);
            }
        } else {
            float sum[COLS];
#pragma unroll
            for (int i = 0; i < COLS; ++i) sum[i] = 0.f;
            const int nchunks = (KB + Cfg::CHUNK_KB - 1) / Cfg::CHUNK_KB;
            const uint32_t ae0 = CL > 1 ? cluster_addr(smem_u32(&acc_empty[0]), 0) : smem_u32(&acc_empty[0]);
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
                if (lane == 0) {
                    if (CL > 1) mbar_arrive_cluster_relaxed(ae0 + abuf * 8u);
                    else asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(ae0 + abuf * 8u) : "memory");
                }
            }
            if (KIND == 2) {  // undo the operands' power-of-two row scales: 2^(eA_i) 2^(eB_j), exact
                // exponents lie in [-115, 100] (split16_kernel), so 2^e is built from its bits
                const float ra = __int_as_float((p.exps[rowA + q * 32 + lane] + 127) << 23);
                const int4* eb = (const int4*)(p.exps + jb.n * p.nb + ccol0);
#pragma unroll
                for (int gi = 0; gi < COLS / 32; ++gi) scale_group(sum + gi * 32, ra, eb + gi * 8);
            }
            // the last acc_full also means every MMA (and so every shared-memory read of the ring,
            // in both CTAs of a pair) has completed
#pragma unroll
            for (int g = 0; g < COLS / 32; ++g) {
                const uint32_t buf = stg + (uint32_t)(g & 1) * 4096u;
                if (g >= 2) {
                    if (lane == 0) bulk_wait_read_1();
                    __syncwarp();
                }
                stage_box_neg(buf, lane, sum + g * 32);
                if (lane == 0) tma_reduce_add(&p.c, buf, ccol0 + g * 32, crow0);
            }
        }
        if (lane == 0) bulk_wait_all();
    }
    tc_fence_before();
    if (CL > 1) cluster_sync();  // neither CTA frees TMEM / exits while its peer may still signal it
    else __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc<CL>(tmem, Cfg::TMEM_COLS);
    }
}

// Persistent 3xFP16 (KIND 2) kernel: CTA pairs loop over the pair tiles of the launch (static
// round robin), so the MMAs of the next tile run while the epilogue scales the finished FP32 sums
// (registers) and reduces them into C — the accumulators are free once the last chunk is drained.
// The staging boxes get their own shared memory (the stage ring stays busy across tiles).
constexpr int P16_STAGES = 3;
constexpr int P16_EPI = 8;
constexpr int P16_STG = 4096;  // one 32 x 32 FP32 box per epilogue warp
constexpr int P16_SMEM = P16_STAGES * TcCfg<2, 2>::STAGE_BYTES + P16_EPI * P16_STG + 1024;

__global__ void __launch_bounds__((4 + P16_EPI) * 32, 1) tc_f16x3_persistent_kernel(const __grid_constant__ TcParams p) {
    using Cfg = TcCfg<2, 2>;
    constexpr int CL = 2;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    __shared__ __align__(8) uint64_t full_bar[P16_STAGES], empty_bar[P16_STAGES];
    __shared__ __align__(8) uint64_t acc_full[2], acc_empty[2];
    __shared__ uint32_t tmem_slot;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t crank = cluster_rank();
    const int pair = blockIdx.x / CL, npairs = gridDim.x / CL;
    const int KB = p.nb / Cfg::BK;
    const int nchunks = (KB + Cfg::CHUNK_KB - 1) / Cfg::CHUNK_KB;

    if (threadIdx.x == 0) {
        for (int s = 0; s < P16_STAGES; ++s) {
            mbar_init(smem_u32(&full_bar[s]), 1);
            mbar_init(smem_u32(&empty_bar[s]), 1);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(smem_u32(&acc_full[i]), 1);
            mbar_init(smem_u32(&acc_empty[i]), CL * P16_EPI);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&p.a) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&p.b) : "memory");
    }
    if (warp == 2) tmem_alloc<CL>(smem_u32(&tmem_slot), Cfg::TMEM_COLS);
    tc_fence_before();
    cluster_sync();
    tc_fence_after();
    const uint32_t tmem = tmem_slot;

    auto coords = [&](int t, int& job, int& bi, int& bj) {
        job = t / p.tiles_per_job;
        const int u = t - job * p.tiles_per_job;
        bi = u / p.tiles_n;
        bj = u - bi * p.tiles_n;
    };

    if (warp == 0 && lane == 0) {
        uint32_t it = 0;
        for (int t = pair; t < p.total; t += npairs) {
            int job, bi, bj;
            coords(t, job, bi, bj);
            const TcJob jb = p.jobs[job];
            const int rowA = jb.m * p.nb + bi * Cfg::BM + (int)crank * TC_BM;
            const int rowB = jb.n * p.nb + bj * Cfg::BN + (int)crank * (Cfg::BN / CL);
            for (int kb = 0; kb < KB; ++kb, ++it) {
                const uint32_t s = it % P16_STAGES;
                const uint32_t ph = (it / P16_STAGES) & 1u;
                mbar_wait(smem_u32(&empty_bar[s]), ph ^ 1u);
                const uint32_t st = smem_u32(smem + s * Cfg::STAGE_BYTES);
                const uint32_t lb = smem_u32(&full_bar[s]);
                const uint32_t fb = cluster_addr(lb, 0);
                if (crank == 0) mbar_expect_tx(lb, CL * Cfg::STAGE_BYTES);
                const int kc = kb * Cfg::BK;
                tma_load_2d<CL>(st, &p.a, fb, kc, rowA);
                tma_load_2d<CL>(st + Cfg::A_BYTES, &p.a_lo, fb, kc, rowA);
                tma_load_2d<CL>(st + 2 * Cfg::A_BYTES, &p.b, fb, kc, rowB);
                tma_load_2d<CL>(st + 2 * Cfg::A_BYTES + Cfg::B_BYTES, &p.b_lo, fb, kc, rowB);
            }
        }
    } else if (warp == 1 && lane == 0 && crank == 0) {
        uint32_t it = 0, g = 0;
        for (int t = pair; t < p.total; t += npairs) {
            for (int kb = 0; kb < KB; ++kb, ++it) {
                const uint32_t s = it % P16_STAGES;
                const uint32_t ph = (it / P16_STAGES) & 1u;
                const int kin = kb % Cfg::CHUNK_KB;
                const uint32_t abuf = g & 1u;
                const uint32_t dacc = tmem + abuf * Cfg::BN;
                if (kin == 0) {
                    mbar_wait(smem_u32(&acc_empty[abuf]), ((g >> 1) & 1u) ^ 1u);
                    tc_fence_after();
                }
                mbar_wait(smem_u32(&full_bar[s]), ph);
                tc_fence_after();
                const uint32_t base = smem_u32(smem + s * Cfg::STAGE_BYTES);
#pragma unroll
                for (int k = 0; k < Cfg::BK / Cfg::UK; ++k) {
                    const uint32_t koff = k * 32;
                    const uint32_t acc = (kin | k) != 0;
                    const uint64_t ahi = desc_sw128(base + koff);
                    const uint64_t alo = desc_sw128(base + Cfg::A_BYTES + koff);
                    const uint64_t bhi = desc_sw128(base + 2 * Cfg::A_BYTES + koff);
                    const uint64_t blo = desc_sw128(base + 2 * Cfg::A_BYTES + Cfg::B_BYTES + koff);
                    tc_mma<2, CL>(dacc, alo, bhi, acc);
                    tc_mma<2, CL>(dacc, ahi, blo, 1u);
                    tc_mma<2, CL>(dacc, ahi, bhi, 1u);
                }
                tc_commit<CL>(smem_u32(&empty_bar[s]));
                if (kin == Cfg::CHUNK_KB - 1 || kb == KB - 1) {
                    tc_commit<CL>(smem_u32(&acc_full[abuf]));
                    ++g;
                }
            }
        }
    } else if (warp >= 4) {
        constexpr int COLS = Cfg::BN / (P16_EPI / 4);
        const int q = (warp - 4) & 3;
        const int half = (warp - 4) >> 2;
        const uint32_t tl = ((uint32_t)(q * 32) << 16) + (uint32_t)(half * COLS);
        const uint32_t stg = smem_u32(smem + P16_STAGES * Cfg::STAGE_BYTES) + (uint32_t)(warp - 4) * P16_STG;
        const uint32_t ae0 = cluster_addr(smem_u32(&acc_empty[0]), 0);
        uint32_t g = 0;
        for (int t = pair; t < p.total; t += npairs) {
            int job, bi, bj;
            coords(t, job, bi, bj);
            const TcJob jb = p.jobs[job];
            const int rowA = jb.m * p.nb + bi * Cfg::BM + (int)crank * TC_BM;
            const int crow0 = (int)(((const char*)jb.C - p.cbase) / ((size_t)p.nb * 4)) + bi * Cfg::BM + (int)crank * TC_BM + q * 32;
            const int ccol0 = bj * Cfg::BN + half * COLS;
            float sum[COLS];
#pragma unroll
            for (int i = 0; i < COLS; ++i) sum[i] = 0.f;
#pragma unroll 1
            for (int c = 0; c < nchunks; ++c, ++g) {
                const uint32_t abuf = g & 1u;
                mbar_wait(smem_u32(&acc_full[abuf]), (g >> 1) & 1u);
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
                if (lane == 0) mbar_arrive_cluster_relaxed(ae0 + abuf * 8u);
            }
            // the accumulators are released: the next tile's MMAs overlap the scaling and C update
            const float ra = __int_as_float((p.exps[rowA + q * 32 + lane] + 127) << 23);
            const int4* eb = (const int4*)(p.exps + jb.n * p.nb + ccol0);
#pragma unroll
            for (int gi = 0; gi < COLS / 32; ++gi) {
                scale_group(sum + gi * 32, ra, eb + gi * 8);
                if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // box free again
                __syncwarp();
                stage_box_neg(stg, lane, sum + gi * 32);
                if (lane == 0) tma_reduce_add(&p.c, stg, ccol0 + gi * 32, crow0);
            }
        }
        if (lane == 0) bulk_wait_all();
    }
    tc_fence_before();
    cluster_sync();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc<CL>(tmem, Cfg::TMEM_COLS);
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
                     uint32_t box_cols, uint32_t box_rows, CUtensorMapSwizzle sw = CU_TENSOR_MAP_SWIZZLE_128B) {
    auto fn = encode_fn();
    if (!fn) return false;
    cuuint64_t dims[2] = {cols, rows};
    cuuint64_t strides[1] = {cols * (cuuint64_t)esz};
    cuuint32_t box[2] = {box_cols, box_rows};
    cuuint32_t es[2] = {1, 1};
    return fn(m, dt, 2, const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
              sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool tc_gemm_available() { return encode_fn() != nullptr; }

static int tc_sm_count() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}
// The persistent 3xFP16 kernel (opt-in, mp_config::f16x3_persistent).  Measured at C3 (profiles/r01,
// s4_persist_*.json): the FP32-class update drops from 1.88 to 1.27-1.35 s, but the evaluation does
// not gain (183.6-186.5 vs 187.1 Tflop/s): the GPU runs at its power cap, so the denser kernel
// lowers the clock for the CRT and FP16 launches, and with reserved pairs the panel stream gets
// fewer SMs.  Default: one CTA pair per output tile.
template <int KIND, int CL>
static cudaError_t launch(const TcArgs& a, int njobs, cudaStream_t s) {
    using Cfg = TcCfg<KIND, CL>;
    if (njobs <= 0) return cudaSuccess;
    if (a.nb % Cfg::BN || a.nb % Cfg::BM) return cudaErrorInvalidValue;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(tc_gemm_kernel<KIND, CL>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    TcParams p;
    memset(&p, 0, sizeof p);
    const uint64_t rows = (uint64_t)a.nt * a.nb;
    constexpr uint32_t BROWS = Cfg::BN / CL;
    bool ok;
    if (KIND == 0 || KIND == 3) {
        ok = a.h16hi && a.e16 &&
             make_map(&p.a, a.h16hi, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, rows, a.nb, Cfg::BK, TC_BM) &&
             make_map(&p.b, a.h16hi, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, rows, a.nb, Cfg::BK, BROWS);
        p.exps = a.e16;
    } else if (KIND == 2) {
        ok = a.h16hi && a.h16lo && a.e16 &&
             make_map(&p.a, a.h16hi, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, rows, a.nb, Cfg::BK, TC_BM) &&
             make_map(&p.a_lo, a.h16lo, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, rows, a.nb, Cfg::BK, TC_BM) &&
             make_map(&p.b, a.h16hi, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, rows, a.nb, Cfg::BK, BROWS) &&
             make_map(&p.b_lo, a.h16lo, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, rows, a.nb, Cfg::BK, BROWS);
        p.exps = a.e16;
    } else {
        ok = make_map(&p.a, a.hi, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, rows, a.nb, Cfg::BK, TC_BM) &&
             make_map(&p.a_lo, a.lo, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, rows, a.nb, Cfg::BK, TC_BM) &&
             make_map(&p.b, a.hi, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, rows, a.nb, Cfg::BK, BROWS) &&
             make_map(&p.b_lo, a.lo, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, rows, a.nb, Cfg::BK, BROWS);
    }
    // C: FP32 rows of nb over [cbase, cbase + crows * nb), 32 x 32 boxes, 128-byte swizzle; FP16 C (KIND 0
    // with c16): 32 x 32 boxes of 64-byte rows, 64-byte swizzle
    if (a.c16 && KIND != 0) return cudaErrorInvalidValue;
    if (a.c16)
        ok = ok && a.cbase && make_map(&p.c, a.cbase, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, a.crows, a.nb, 32, 32,
                                       CU_TENSOR_MAP_SWIZZLE_64B);
    else
        ok = ok && a.cbase && make_map(&p.c, a.cbase, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, a.crows, a.nb, 32, 32);
    if (!ok) return cudaErrorInvalidValue;
    p.jobs = a.jobs;
    p.cbase = (const char*)a.cbase;
    p.c16 = a.c16;
    p.nb = a.nb;
    p.tiles_n = a.nb / Cfg::BN;
    p.tiles_per_job = (a.nb / Cfg::BM) * p.tiles_n;
    long long grid = (long long)njobs * p.tiles_per_job * CL;
    if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    void (*kern)(TcParams) = tc_gemm_kernel<KIND, CL>;
    int smem_bytes = Cfg::SMEM;
    if (KIND == 2 && CL == 2 && a.persistent) {
        static bool pattr = false;
        if (!pattr) {
            cudaError_t e = cudaFuncSetAttribute(tc_f16x3_persistent_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, P16_SMEM);
            if (e != cudaSuccess) return e;
            pattr = true;
        }
        p.total = (int)(grid / CL);
        int pairs = a.pairs > 0 ? a.pairs : tc_sm_count() / 2;
        if (pairs > p.total) pairs = p.total;
        grid = (long long)pairs * CL;
        kern = tc_f16x3_persistent_kernel;
        smem_bytes = P16_SMEM;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(kern == tc_f16x3_persistent_kernel ? (4 + P16_EPI) * 32 : TcThreads<KIND>::N);
    cfg.dynamicSmemBytes = smem_bytes;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, p);
}

// CTA pairs (cta_group::2) for every kind: faster than single CTAs for both (profiles/r01/README.md)
cudaError_t tc_gemm_f16_launch(const TcArgs& a, int njobs, cudaStream_t s) { return launch<0, 2>(a, njobs, s); }
cudaError_t tc_gemm_f16h_launch(const TcArgs& a, int njobs, cudaStream_t s) {
    return a.c16 ? cudaErrorInvalidValue : launch<3, 2>(a, njobs, s);
}
cudaError_t tc_gemm_f16x3_launch(const TcArgs& a, int njobs, cudaStream_t s) { return launch<2, 2>(a, njobs, s); }
cudaError_t tc_gemm_tf32x3_launch(const TcArgs& a, int njobs, cudaStream_t s) { return launch<1, 2>(a, njobs, s); }

}  // namespace mpgeo
