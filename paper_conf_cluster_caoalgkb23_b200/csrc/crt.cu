// K5c — FP64-class tile GEMM on INT8 tcgen05 tensor cores, modular integer emulation
// ("Ozaki scheme II"; SURVEY §8(f) item 4, FP64 class of Algorithm 1: GEMM/SYRK at FP64, P:132,
// P:136).  C_mn (FP64) -= P_m P_n^T over K = nb.
//
// Operands (crt_split_kernel, once per panel tile and GPU, like the K2 conversions): row i of a
// tile with max_j |x_ij| < 2^{e_i} becomes the integer row x'_ij = rint(x_ij 2^{b - e_i}), |x'| <=
// 2^b (exact in FP64: x has 53 significant bits), stored as N int8 residue planes x'_ij mod p_t
// (symmetric representative in [-128, 127]) for N pairwise coprime moduli p_t <= 256.
// Product: X_ij = sum_k x'_ik y'_jk is an integer with |X| <= K 2^{2b} <= 0.3 M, M = prod p_t, so it
// is fixed by its residues.  Per modulus one INT8 GEMM (kind::i8, exact INT32 accumulation in TMEM:
// |acc| <= K 128^2 = 2^25) gives acc_t == X (mod p_t).  The epilogue reduces the first modulus a of
// each pair to r_a (exact Barrett), combines it with the second modulus b by Shoup's modular
// multiplication into the pair residue R_j = r_a + a ((acc_b - r_a) a^-1 mod b) in [0, ab), and, once
// all pairs are known, reconstructs
//     X = sum_j R_j w_j  -  q M,   w_j = (M/m_j) ((M/m_j)^-1 mod m_j)
// with integer + FP32 arithmetic only (crt_recon_bits, crt.h: FP32 quotient estimate, 96-bit limb
// sums, the FP64 bit pattern of X 2^{e_i + f_j - 2b} assembled by count-leading-zeros) — the FP64
// pipe runs ~25x slower while the tensor core is busy.  C_ij -= that value by TMA
// reduce-add.  Accuracy: the operand rounding is 2^-(b+1) of the row max (b = 56 for N = 16,
// K = 2048), i.e. the product error is <= K 2^-(b+1) (max_k|a_ik| max_k|b_jk|) — FP64-GEMM level
// (K 2^-53 sum|a||b|); the reconstruction adds < 2^51.6 absolute on X (2^-15 of that bound) and one
// rounding to 53 bits.  N = 16 GEMMs per tile product (an 8-slice Ozaki split needs 36).
//
// Kernel: persistent CTA pairs (cluster of 2 on a TPC, tcgen05.mma.cta_group::2, M = 256, N = 256,
// K = 32 per MMA), 128-byte-swizzled K-major TMA boxes of 128 x 128 int8 per CTA and operand, five
// 32 KB stages.  Accumulators: two 256-column TMEM buffers, one per modulus in flight, so the
// epilogue reduces modulus t while the tensor core computes modulus t+1.
//   warp 0: TMA producer; warp 1: MMA issuer (leader CTA); warp 2: TMEM allocator;
//   warps 4-11 (CRT_EPI = 8; 16 also builds): epilogue — warp w owns TMEM lanes 32 (w % 4).. (its rows)
//   and one column part; per moduli pair it stores the uint16 pair residues into a per-CTA scratch of
//   recycled 2 KB blocks and reconstructs the previous tile group by group in between (see the epilogue).
#include <cudaTypedefs.h>
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <cstdio>

#include "common.cuh"
#include "crt.h"

namespace mpgeo {

// ------------------------------------------------------------------ host constants
static const int kModuli[CRT_NMAX] = {256, 255, 253, 251, 247, 241, 239, 233,
                                      229, 227, 223, 217, 211, 199, 197, 193};

static int u128_bits(unsigned __int128 v) {
    int b = 0;
    while (v) {
        ++b;
        v >>= 1;
    }
    return b;
}
static double u128_to_double(unsigned __int128 v) {  // correctly rounded enough (only used for L, Ml < 2^85)
    const uint64_t hi = (uint64_t)(v >> 64), lo = (uint64_t)v;
    return ldexp((double)hi, 64) + (double)lo;
}

bool crt_constants(int nmod, int K, CrtConst* c) {
    if (nmod < 2 || nmod > CRT_NMAX || (nmod & 1) || K < 1 || K > 8192) return false;
    memset(c, 0, sizeof *c);
    c->nmod = nmod;
    unsigned __int128 M = 1;
    for (int t = 0; t < nmod; ++t) M *= (unsigned)kModuli[t];
    // largest b with K 2^{2b} <= 0.3 M (crt.h: uniqueness, and the margin of the FP32 quotient estimate)
    {
        const unsigned __int128 lim = M / 10 * 3;
        int b = 0;
        while (2 * (b + 1) + 13 < 128 && ((unsigned __int128)K << (2 * (b + 1))) <= lim) ++b;  // K <= 2^13
        c->bits = b;
    }
    if (c->bits < 8) return false;
    for (int t = 0; t < nmod; ++t) {
        const unsigned p = (unsigned)kModuli[t];
        c->p[t] = (int)p;
        c->invp[t] = 1.0 / (double)p;
        c->bm[t] = (unsigned)(((1ull << 38) + p - 1) / p);
    }
    // paired moduli m_j = p_2j p_2j+1 (< 2^16): the epilogue combines the two residues exactly,
    // R = r_a + a ((r_b - r_a) a^-1 mod b), and reconstructs from nmod/2 residues R_j in [0, m_j).
    // Split unit: H_j multiples of 2^sh with < 2^33 multiples, so sum_j R_j H_j is exact in FP64
    // (R < 2^16, 8 terms: < 2^52 units).
    const int npair = nmod / 2;
    const int sh = u128_bits(M) > 33 ? u128_bits(M) - 33 : 0;
    const unsigned __int128 mask = (((unsigned __int128)1) << sh) - 1;
    for (int j = 0; j < npair; ++j) {
        const unsigned a = (unsigned)kModuli[2 * j], b = (unsigned)kModuli[2 * j + 1];
        unsigned ia = 0;
        for (unsigned v = 1; v < b; ++v)
            if ((a % b) * v % b == 1) {
                ia = v;
                break;
            }
        if (!ia) return false;  // moduli not coprime
        const unsigned m = a * b;
        const unsigned __int128 Mj = M / m;
        const unsigned mj = (unsigned)(Mj % m);
        unsigned y = 0;
        for (unsigned v = 1; v < m; ++v)
            if ((unsigned long long)mj * v % m == 1) {
                y = v;
                break;
            }
        if (!y) return false;
        const unsigned __int128 w = Mj * y;  // < M
        c->ia[j] = (int)ia;
        c->shoup[j] = (unsigned)(((unsigned long long)ia << 32) / b);  // floor(ia 2^32 / b)
        c->mpair[j] = (int)m;
        c->H[j] = ldexp((double)(uint64_t)(w >> sh), sh);  // exact (< 2^33 units)
        c->L[j] = u128_to_double(w & mask);
    }
    c->Mh = ldexp((double)(uint64_t)(M >> sh), sh);
    c->Ml = u128_to_double(M & mask);
    c->invM = 1.0 / u128_to_double(M);
    // integer + FP32 reconstruction constants (crt_recon_bits, crt.h)
    c->ld = u128_bits(M) > 64 ? 1 : 0;
    const int lsh = 32 * c->ld;
    for (int t = 0; t < 3; ++t) c->Mw[t] = (uint32_t)((M >> lsh) >> (32 * t));
    const double Md = u128_to_double(M);
    unsigned __int128 Dr = 0;  // sum_j h_j w_j = Dq M + Dr, exact (shift-and-add modulo M; M < 2^126)
    long long Dq = 0;
    for (int j = 0; j < npair; ++j) {
        const unsigned a = (unsigned)kModuli[2 * j], b = (unsigned)kModuli[2 * j + 1], m = a * b;
        const unsigned __int128 Mj = M / m;
        const unsigned mj = (unsigned)(Mj % m);
        unsigned y = 0;
        for (unsigned v = 1; v < m; ++v)
            if ((unsigned long long)mj * v % m == 1) {
                y = v;
                break;
            }
        const unsigned __int128 w = Mj * y;
        for (int t = 0; t < 3; ++t) c->W[j][t] = (uint32_t)((w >> lsh) >> (32 * t));
        c->cw[j] = (float)(u128_to_double(w) / Md);
        const unsigned h = m / 2;
        c->hoff[j] = 8388608.0f + (float)h;
        unsigned __int128 r = 0;
        long long qq = 0;
        for (int bit = 15; bit >= 0; --bit) {
            r <<= 1;
            qq <<= 1;
            if (r >= M) r -= M, ++qq;
            if ((h >> bit) & 1u) {
                r += w;
                if (r >= M) r -= M, ++qq;
            }
        }
        Dr += r;
        if (Dr >= M) Dr -= M, ++qq;
        Dq += qq;
    }
    c->Dq = (int)Dq;
    c->fD = (float)(u128_to_double(Dr) / Md);
    return true;
}

// ------------------------------------------------------------------ operand residues
// One warp per row; lanes cover 4 consecutive elements (char4 stores per plane).
__global__ void __launch_bounds__(256) crt_split_kernel(const CrtSplitItem* items, int nb, const __grid_constant__ CrtConst c) {
    const CrtSplitItem it = items[blockIdx.y];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int row = blockIdx.x * 8 + warp;
    if (row >= nb) return;
    const double* x = it.src + (size_t)row * nb;
    double mx = 0.0;
    for (int j = lane; j < nb; j += 32) mx = fmax(mx, fabs(x[j]));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    int e = 0;
    if (mx > 0.0) frexp(mx, &e);  // |x| < 2^e
    if (lane == 0) it.exps[row] = e;
    const size_t plane = (size_t)it.plane_stride;
    const double magic = 6755399441055744.0;  // 1.5 * 2^52: adding it leaves a small integer in the low word
    for (int j0 = lane * 4; j0 < nb; j0 += 128) {
        double xi[4];
#pragma unroll
        for (int v = 0; v < 4; ++v) xi[v] = (j0 + v < nb) ? rint(ldexp(x[j0 + v], c.bits - e)) : 0.0;
#pragma unroll 4
        for (int t = 0; t < c.nmod; ++t) {
            const double p = (double)c.p[t];
            int r[4];
#pragma unroll
            for (int v = 0; v < 4; ++v) {
                const double q = rint(xi[v] * c.invp[t]);
                const double rd = fma(-q, p, xi[v]);  // exact: the true value is a small integer
                int ri = (int)__double2loint(rd + magic);
                ri -= ri > 127 ? c.p[t] : 0;
                ri += ri < -128 ? c.p[t] : 0;
                r[v] = ri;
            }
            char4 d;
            d.x = (signed char)r[0];
            d.y = (signed char)r[1];
            d.z = (signed char)r[2];
            d.w = (signed char)r[3];
            *(char4*)(it.dst + t * plane + (size_t)row * nb + j0) = d;
        }
    }
}

cudaError_t crt_split_launch(const CrtSplitItem* items, int n, int nb, const CrtConst& c, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    if (nb % 4) return cudaErrorInvalidValue;
    dim3 grid((nb + 7) / 8, n);
    crt_split_kernel<<<grid, 256, 0, s>>>(items, nb, c);
    return cudaGetLastError();
}

// ------------------------------------------------------------------ GEMM
namespace {

constexpr int BM = 128;             // rows per CTA (TMEM lanes); the pair covers 256
constexpr int BN = 256;             // MMA N = output columns per pair tile
constexpr int BK = 128;             // int8 elements per 128-byte swizzled row
constexpr int A_BYTES = BM * BK;    // 16 KB
constexpr int B_BYTES = (BN / 2) * BK;  // 16 KB: each CTA loads half of B
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int STAGES = 5;  // 5 x 32 KB: with the C staging (32 KB) and the scratch-block tables the CTA fits in 227 KB
constexpr int RING = 4;  // tile-index ring depth (dynamic scheduler)
// C update staging: per epilogue warp two 32 x 8 FP64 boxes (2 KB, 64-byte swizzle) reduced into C
// by the TMA unit (cp.reduce.async.bulk.tensor .add on the FP64 C map)
// epilogue warps: 8 (two per TMEM lane quarter, 128 columns each) or 16 (four per quarter, 64 columns)
#ifndef CRT_EPI
#define CRT_EPI 8
#endif
constexpr int EPI_WARPS = CRT_EPI;
constexpr int PARTS = EPI_WARPS / 4;     // column parts of the 256-column accumulator
constexpr int PCOLS = BN / PARTS;        // columns per epilogue warp
constexpr int CHUNKS = PCOLS / 32;       // 32-column TMEM loads per accumulator and warp
constexpr int GROUPS = PCOLS / 8;        // 8-column reconstruction groups per warp and tile
constexpr int STG_BOX = 32 * 8 * 8;
constexpr int NSTG = EPI_WARPS == 8 ? 2 : 1;  // staging boxes per warp (shared-memory budget)
constexpr int STG_WARP = NSTG * STG_BOX;
constexpr int SMEM = STAGES * STAGE_BYTES + EPI_WARPS * STG_WARP + 1024;
constexpr int THREADS = (4 + EPI_WARPS) * 32;
constexpr int SCR_BLOCKS_P = CRT_NMAX / 2 * GROUPS + GROUPS;  // blocks per column part (a tile + one step's spare)
static_assert(PARTS * SCR_BLOCKS_P * CRT_SCR_BLOCK <= (int)CRT_SLOT_BYTES, "scratch slot too small");
constexpr uint32_t TMEM_COLS = 512;  // two 256-column accumulators
// L2 eviction priority of the operand loads (residue planes): 0 normal, 1 evict_last for A (the row
// operand consecutive jobs share), 2 evict_last for A and B
#ifndef CRT_L2HINT
#define CRT_L2HINT 0
#endif
// 1: the first scratch group of each pair step's reconstruction is loaded before the residue steps;
// 2: between the two residue steps
#ifndef CRT_EARLY
#define CRT_EARLY 0
#endif
// 1: reconstructed residue-scratch lines are discarded from L2 (discard.global.L2) instead of being
// evicted dirty to HBM
#ifndef CRT_DISCARD
#define CRT_DISCARD 0
#endif
// 1: residue-scratch stores carry an L2 evict_last policy
#ifndef CRT_SCRHINT
#define CRT_SCRHINT 0
#endif
// instruction descriptor: D = S32 (2 << 4), A = B = signed int8 (1 << 7, 1 << 10), K-major,
// N >> 3 at bit 17, M >> 4 at bit 24 (M = 256 for the pair)
constexpr uint32_t IDESC = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);

struct __align__(64) CrtParams {
    CUtensorMap a, b;  // 3D [N][rows][nb] int8, box {128, 128, 1}
    CUtensorMap cmap;  // C rows [crows][nb] from cbase, box {8, 32}: FP64 (64-byte swizzle) or FP32 (no swizzle)
    const void* cbase;
    const CrtJob* jobs;
    const int* exps;
    uint8_t* scratch;
    int* slot_flags;
    int nslots, nb, tiles_n, tiles_per_job, lower, total;
    int store;  // 1: C = P_m P_n^T (TMA store), 0: C -= P_m P_n^T (TMA reduce-add)
    int* tile_counter;  // [0]: dynamic tile scheduler, [1]: current modulus-pair phase (zero before the launch)
    int phase_lock;     // 1: start each tile at the current modulus-pair phase (CrtArgs::phase_lock)
    CrtConst c;
};

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
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
__device__ __forceinline__ uint32_t cluster_addr(uint32_t saddr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
    return r;
}
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cbar) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cbar) : "memory");
}
// relaxed arrive: the epilogue only signals that its tcgen05.ld of the accumulator completed
// (wait::ld), so no memory ordering of its global stores is needed (a release would add a MEMBAR)
__device__ __forceinline__ void mbar_arrive_cluster_relaxed(uint32_t cbar) {
    asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(cbar) : "memory");
}
// wait with cluster-scope acquire: the awaited data (the tile ring) may be written by the peer CTA
__device__ __forceinline__ void mbar_wait_cl(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void st_cluster_u32(uint32_t addr, int v) {
    asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_id() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t num_clusters() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// 3D TMA load; the completion is signalled on the leader CTA's barrier (cta_group::2 form)
__device__ __forceinline__ void tma3d_pair(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1, int c2) {
    asm volatile(
        "cp.async.bulk.tensor.3d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(dst),
        "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
        : "memory");
}
// the same with an L2 cache-policy hint (createpolicy)
__device__ __forceinline__ void tma3d_pair_hint(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1, int c2,
                                                uint64_t pol) {
    asm volatile(
        "cp.async.bulk.tensor.3d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%3, %4, %5}], [%2], %6;" ::"r"(dst),
        "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "r"(c2), "l"(pol)
        : "memory");
}
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void commit_pair(uint32_t bar) {
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(bar),
                 "h"((uint16_t)3)
                 : "memory");
}
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
    uint64_t d = (uint64_t)((saddr & 0x3FFFFu) >> 4);
    d |= (uint64_t)1 << 16;
    d |= (uint64_t)(1024 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}
__device__ __forceinline__ void mma_i8_pair(uint32_t tmem, uint64_t a, uint64_t b, uint32_t accum) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
        "l"(a), "l"(b), "r"(IDESC), "r"(accum));
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

#ifdef CRT_PROF
#define PROF_T0() long long _t0 = clock64()
#define PROF_ADD(v) v += clock64() - _t0
#else
#define PROF_T0()
#define PROF_ADD(v)
#endif

// pair tile index -> (job, bi, bj) over 256 x 256 blocks; lower: only bj <= bi (SYRK)
__device__ __forceinline__ void tile_coords(const CrtParams& p, int t, int& job, int& bi, int& bj) {
    job = t / p.tiles_per_job;
    const int u = t - job * p.tiles_per_job;
    if (p.lower) {
        int i = (int)((sqrtf(8.0f * (float)u + 1.0f) - 1.0f) * 0.5f);
        while ((i + 1) * (i + 2) / 2 <= u) ++i;
        while (i * (i + 1) / 2 > u) --i;
        bi = i;
        bj = u - i * (i + 1) / 2;
    } else {
        bi = u / p.tiles_n;
        bj = u - bi * p.tiles_n;
    }
}

// scratch byte offset of the 16-byte run (block b of column half h, CTA row r) holding 8 combined
// residues R (uint16) of one moduli pair and one 8-column group: a warp's 32 rows of one block are
// 512 contiguous bytes (coalesced stores and loads)
__device__ __forceinline__ uint32_t scr_off(int b, int h, int r) {
    return ((uint32_t)(h * SCR_BLOCKS_P + b) * 128u + (uint32_t)r) * 16u;
}

__device__ __forceinline__ void tmem_ld32_nowait(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}
// wait for every outstanding tcgen05.ld of this thread; the register "touch" keeps the compiler
// from hoisting uses of r above the wait
__device__ __forceinline__ void tmem_wait(uint32_t (&r)[32]) {
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 32; ++i) asm volatile("" : "+r"(r[i]));
}
// canonical residue of a modulo p in [0, p), |a| <= 2^27 (the INT32 accumulator bound K 2^14 for
// K <= 8192; |(r_b - r_a) ia| < 2^16): exact Barrett reduction.  a' = a + p 2^20 is a multiple-of-p
// shift of a in [0, 2^29); with m = ceil(2^38/p), floor(a' m / 2^38) = floor(a'/p) because the excess
// a' (m - 2^38/p) / 2^38 < 2^-9 < 1/p.  One IMAD.HI + shift + IMAD, no correction step
// (tools/dbg/epi_rate.cu measures it against the previous rounded-quotient form).
__device__ __forceinline__ int mod_canon(int a, int p, unsigned bm) {
    const unsigned ap = (unsigned)(a + (p << 20));
    const unsigned q = __umulhi(ap, bm) >> 6;
    return (int)(ap - q * (unsigned)p);
}

}  // namespace

// NMOD moduli (16: FP64 class, b = 56 at K = 2048; 8: the FP32-class TRSM product, b = 25); C is FP64
template <int NMOD>
__global__ void __launch_bounds__(THREADS, 1) crt_gemm_kernel(const __grid_constant__ CrtParams p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    __shared__ __align__(8) uint64_t full_bar[STAGES], empty_bar[STAGES];
    __shared__ __align__(8) uint64_t acc_full[2], acc_empty[2];
    __shared__ uint32_t tmem_slot;
    __shared__ int slot_sh;
    // dynamic tile scheduler: the leader's producer claims pair tiles from a global counter and
    // publishes them in a ring in both CTAs (late-starting pairs simply claim fewer tiles)
    __shared__ int tile_ring[RING];
    __shared__ __align__(8) uint64_t ring_full[RING], ring_empty[RING];
    // per epilogue warp: scratch block of (moduli pair j, group gi) for the two tiles in flight, and
    // the 16 blocks the last reconstruction step freed (the next residue step's destinations)
    __shared__ uint8_t scr_tab[EPI_WARPS][2][CRT_NMAX / 2 * GROUPS];
    __shared__ uint8_t scr_free[EPI_WARPS][GROUPS];

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t crank = cluster_rank();
    constexpr int N = NMOD;
    const int KB = p.nb / BK;

    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(su32(&full_bar[s]), 1);   // leader: its producer's arrive + both CTAs' bytes
            mbar_init(su32(&empty_bar[s]), 1);  // the leader's MMA commit (multicast)
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(su32(&acc_full[i]), 1);
            mbar_init(su32(&acc_empty[i]), 2 * EPI_WARPS);  // every epilogue warp of the pair
        }
        for (int i = 0; i < RING; ++i) {
            mbar_init(su32(&ring_full[i]), 1);  // the leader producer's publish
            // readers: leader MMA + CTA-1 producer + every epilogue warp of the pair (leader's barrier)
            mbar_init(su32(&ring_empty[i]), 2 + 2 * EPI_WARPS);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&p.a) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&p.b) : "memory");
        // scratch slot: at most one CTA of this kernel per SM is resident, and 2 x SMs slots exist
        int s = (int)(blockIdx.x % (unsigned)p.nslots);
        while (atomicCAS(&p.slot_flags[s], 0, 1) != 0) s = s + 1 == p.nslots ? 0 : s + 1;
        __threadfence();
        slot_sh = s;
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(&tmem_slot)),
                     "r"(TMEM_COLS)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    fence_before();
    cluster_sync();
    fence_after();
    const uint32_t tmem = tmem_slot;
#ifdef CRT_PROF
    long long pw_accempty = 0, pw_full = 0, pw_accfull = 0, pw_resid = 0, pw_recon = 0, pw_stgwait = 0, pw_ld = 0;
#endif

    // ring slot i % RING: wait for the published tile index, then release the slot to the leader
    auto ring_take = [&](int i, bool release) {
        const int s = i % RING;
        mbar_wait_cl(su32(&ring_full[s]), (uint32_t)(i / RING) & 1u);
        const int t = tile_ring[s];
        if (release) mbar_arrive_cluster(cluster_addr(su32(&ring_empty[s]), 0));
        return t;
    };

    if (warp == 0 && lane == 0) {
        // ---------------- TMA producer: per tile, per modulus, K in 128-byte blocks
        uint32_t it = 0;
        uint64_t pol_last = 0;
        if (CRT_L2HINT) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_last));
        for (int i = 0;; ++i) {
            int tile;
            if (crank == 0) {  // claim the next pair tile and publish it to both CTAs
                const int s = i % RING;
                mbar_wait(su32(&ring_empty[s]), ((uint32_t)(i / RING) & 1u) ^ 1u);
                tile = atomicAdd(p.tile_counter, 1);
                // modulus-pair phase: start where the other pairs currently are (p.tile_counter[1],
                // written by every MMA issuer), so concurrent tiles read the same residue planes
                // and the operands of one phase stay L2-resident; any order gives the same result
                if (tile >= p.total) tile = -1;
                else if (p.phase_lock) tile |= (*(volatile int*)(p.tile_counter + 1) & (NMOD / 2 - 1)) << 28;
                tile_ring[s] = tile;
                st_cluster_u32(cluster_addr(su32(&tile_ring[s]), 1), tile);
                mbar_arrive_cluster(su32(&ring_full[s]));
                mbar_arrive_cluster(cluster_addr(su32(&ring_full[s]), 1));
            } else {
                tile = ring_take(i, true);
            }
            if (tile < 0) break;
            const int j0 = tile >> 28;
            tile &= (1 << 28) - 1;
            int job, bi, bj;
            tile_coords(p, tile, job, bi, bj);
            const CrtJob jb = p.jobs[job];
            const int rowA = jb.m * p.nb + bi * 256 + (int)crank * BM;
            const int rowB = jb.n * p.nb + bj * BN + (int)crank * (BN / 2);
            for (int tt = 0; tt < N; ++tt) {
                const int t = (2 * j0 + tt) & (N - 1);
                for (int kb = 0; kb < KB; ++kb, ++it) {
                    const uint32_t s = it % STAGES;
                    const uint32_t ph = (it / STAGES) & 1u;
                    mbar_wait(su32(&empty_bar[s]), ph ^ 1u);
                    const uint32_t st = su32(smem + s * STAGE_BYTES);
                    const uint32_t lb = su32(&full_bar[s]);
                    const uint32_t fb = cluster_addr(lb, 0);
                    if (crank == 0) mbar_expect_tx(lb, 2 * STAGE_BYTES);
                    if (CRT_L2HINT >= 1) tma3d_pair_hint(st, &p.a, fb, kb * BK, rowA, t, pol_last);
                    else tma3d_pair(st, &p.a, fb, kb * BK, rowA, t);
                    if (CRT_L2HINT >= 2) tma3d_pair_hint(st + A_BYTES, &p.b, fb, kb * BK, rowB, t, pol_last);
                    else tma3d_pair(st + A_BYTES, &p.b, fb, kb * BK, rowB, t);
                }
            }
        }
    } else if (warp == 1 && lane == 0 && crank == 0) {
        // ---------------- MMA issuer (leader CTA): one accumulator per modulus, two in flight
        uint32_t it = 0, g = 0;
        for (int i = 0;; ++i) {
            const int tv = ring_take(i, true);
            if (tv < 0) break;
            const int j0 = tv >> 28;
            for (int tt = 0; tt < N; ++tt, ++g) {
                if (p.phase_lock && !(tt & 1)) *(volatile int*)(p.tile_counter + 1) = ((j0 + (tt >> 1)) & (N / 2 - 1));
                const uint32_t buf = g & 1u;
                { PROF_T0();
                mbar_wait(su32(&acc_empty[buf]), ((g >> 1) & 1u) ^ 1u);
                PROF_ADD(pw_accempty); }
                fence_after();
                const uint32_t dacc = tmem + buf * (uint32_t)BN;
                for (int kb = 0; kb < KB; ++kb, ++it) {
                    const uint32_t s = it % STAGES;
                    const uint32_t ph = (it / STAGES) & 1u;
                    { PROF_T0();
                    mbar_wait(su32(&full_bar[s]), ph);
                    PROF_ADD(pw_full); }
                    fence_after();
                    const uint32_t base = su32(smem + s * STAGE_BYTES);
#pragma unroll
                    for (int k = 0; k < BK / 32; ++k) {
                        const uint32_t koff = (uint32_t)k * 32u;
                        mma_i8_pair(dacc, desc_sw128(base + koff), desc_sw128(base + A_BYTES + koff), (kb | k) != 0);
                    }
                    commit_pair(su32(&empty_bar[s]));
                }
                commit_pair(su32(&acc_full[buf]));
            }
        }
    } else if (warp >= 4) {
        // ---------------- epilogue.  Per tile T: for each moduli pair j, reduce modulus a (residues
        // kept as bytes), reduce modulus b and store the combined residues R_j of T into 16 scratch
        // blocks (one per 8-column group), then reconstruct 16/NP of the 16 eight-column groups of
        // tile T-1 and reduce-add them into C — so the reconstruction fills the epilogue's slack while
        // the tensor core works on T.  The 16 blocks each reconstruction step frees are the next
        // residue step's destinations (scr_tab / scr_free): one tile of scratch + 16 spare blocks per
        // CTA (576 KB) instead of two tiles, so the scratch in flight stays within L2.
        const int q = (warp - 4) & 3, h = (warp - 4) >> 2;
        const int r = q * 32 + lane;  // CTA row = TMEM lane
        uint8_t* const scr0 = p.scratch + (size_t)slot_sh * CRT_SLOT_BYTES;
        uint64_t scr_pol = 0;
        if (CRT_SCRHINT) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(scr_pol));
        const uint32_t tl = ((uint32_t)(q * 32) << 16) + (uint32_t)(h * PCOLS);
        const uint32_t ae0 = cluster_addr(su32(&acc_empty[0]), 0);
        const uint32_t stg_s = su32(smem + STAGES * STAGE_BYTES + (warp - 4) * STG_WARP);
        constexpr int NP = N / 2;
        uint32_t g = 0;       // accumulator-buffer counter (one per modulus)
        uint32_t nred = 0;    // C reduce-adds issued by this warp (staging-buffer parity)
        // the previous tile, whose reconstruction is pending
        bool pv = false;
        int pv_crow0 = 0, pv_ccol0 = 0, pv_tab = 0;
        int pv_e0 = 0;  // row exponent e_i - 2b of the pending tile (C += X 2^(e_i + f_j - 2b))
        const int* pv_ecol = nullptr;
        const int ew = warp - 4;
        if (lane < GROUPS) scr_free[ew][lane] = (uint8_t)(NP * GROUPS + lane);  // the spare blocks
        __syncwarp();

        // reconstruct groups gi (8 columns each) of the pending tile: X = sum_j R_j w_j - q M, scaled
        auto load_group = [&](int gi, uint4 (&w)[NP]) {
#pragma unroll
            for (int jj = 0; jj < NP; ++jj)  // last use of each block
                w[jj] = __ldcs((const uint4*)(scr0 + scr_off(scr_tab[ew][pv_tab][jj * GROUPS + gi], h, r)));
        };
        // after reconstructing groups [g0, g0 + 16/NP) of the pending tile their 16 blocks are free
        auto free_groups = [&](int g0) {
            __syncwarp();
            if (CRT_DISCARD) {
                // the residues are dead once read: drop this warp's 4 lines (32 rows x 16 B) of every freed
                // block from L2 without writing them back (otherwise each is evicted dirty to HBM later)
                for (int i = lane; i < GROUPS * 4; i += 32) {
                    const int blk = scr_tab[ew][pv_tab][((i >> 2) % NP) * GROUPS + g0 + (i >> 2) / NP];
                    asm volatile("discard.global.L2 [%0], 128;" ::"l"(scr0 + scr_off(blk, h, q * 32 + (i & 3) * 8)) : "memory");
                }
                asm volatile("fence.acq_rel.cta;" ::: "memory");
                __syncwarp();
            }
            if (lane < GROUPS) scr_free[ew][lane] = scr_tab[ew][pv_tab][(lane % NP) * GROUPS + g0 + lane / NP];
            __syncwarp();
        };
        // L2 prefetch of groups [g0, g1) of the pending tile (all 128 rows of this column half: one
        // 2 KB bulk prefetch per moduli pair and group, issued by one warp of the half)
        auto prefetch_groups = [&](int g0, int g1) {
            if (q == 0 && lane == 0)
                for (int gi = g0; gi < g1; ++gi)
                    for (int jj = 0; jj < NP; ++jj) {
                        const uint8_t* src = scr0 + scr_off(scr_tab[ew][pv_tab][jj * GROUPS + gi], h, 0);
                        asm volatile("cp.async.bulk.prefetch.L2.global [%0], 2048;" ::"l"(src) : "memory");
                    }
        };
        auto recon = [&](int gi, const uint4 (&w)[NP]) {
            const int col0 = (gi >> 2) * 32 + (gi & 3) * 8;
#ifdef CRT_PROF
            {  // time until the scratch loads of this group have landed
                PROF_T0();
                uint32_t t = 0;
#pragma unroll
                for (int jj = 0; jj < NP; ++jj) t ^= w[jj].x ^ w[jj].w;
                asm volatile("" ::"r"(t));
                PROF_ADD(pw_ld);
            }
#endif
            // stage -out in the warp's 32 x 8 box (64-byte swizzle: 16-byte chunk k of row l at
            // k ^ ((l >> 1) & 3)); one lane reduces the box into C through the TMA unit.  The box is
            // free once the TMA unit has read the reduce-add issued NSTG groups ago.
            const uint32_t sb = stg_s + (nred % NSTG) * (uint32_t)STG_BOX;
            if (nred >= NSTG) {
                PROF_T0();
                if (lane == 0) {
                    if (NSTG == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
                    else asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
                }
                PROF_ADD(pw_stgwait);
                __syncwarp();
            }
            // integer + FP32 reconstruction (crt_recon_bits, crt.h): no FP64 instruction while the
            // tensor core runs; two elements at a time, stored as they are done
#pragma unroll
            for (int v = 0; v < 8; v += 2) {
                uint64_t o[2];
#pragma unroll
                for (int u = 0; u < 2; ++u) {
                    uint32_t R[NP];
                    const int vv = v + u;
#pragma unroll
                    for (int jj = 0; jj < NP; ++jj) {
                        const uint32_t wv = (vv >> 1) == 0 ? w[jj].x : (vv >> 1) == 1 ? w[jj].y : (vv >> 1) == 2 ? w[jj].z : w[jj].w;
                        R[jj] = (vv & 1) ? (wv >> 16) : (wv & 0xffffu);
                    }
                    o[u] = crt_recon_bits<NP>(R, p.c, pv_e0 + __ldg(pv_ecol + col0 + vv), p.store ? 0u : 1u);
                }
                const uint32_t a = sb + (uint32_t)lane * 64u + ((uint32_t)((v >> 1) ^ ((lane >> 1) & 3)) << 4);
                asm volatile("st.shared.v2.b64 [%0], {%1, %2};" ::"r"(a), "l"(o[0]), "l"(o[1]) : "memory");
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (lane == 0) {
                if (p.store)
                    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                                     (uint64_t)&p.cmap),
                                 "r"(sb), "r"(pv_ccol0 + col0), "r"(pv_crow0)
                                 : "memory");
                else
                    asm volatile("cp.reduce.async.bulk.tensor.2d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                                     (uint64_t)&p.cmap),
                                 "r"(sb), "r"(pv_ccol0 + col0), "r"(pv_crow0)
                                 : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
            ++nred;
        };

        // Walk the warp's CHUNKS 32-column TMEM chunks of accumulator buffer `buf`: double-buffered loads
        // with 8 epilogue warps, single-buffered with 16 (register budget); the accumulator is released to
        // the MMA as soon as its last chunk is in registers.
        auto tmem_chunks = [&](uint32_t buf, auto&& f) {
            const uint32_t base = tmem + tl + buf * (uint32_t)BN;
            auto release = [&]() {
                fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive_cluster_relaxed(ae0 + buf * 8u);
            };
            if constexpr (EPI_WARPS == 8) {
                uint32_t v0[32], v1[32];
                tmem_ld32_nowait(base, v0);
                tmem_wait(v0);
#pragma unroll
                for (int c = 0; c < CHUNKS; ++c) {
                    uint32_t (&vc)[32] = (c & 1) ? v1 : v0;
                    uint32_t (&vn)[32] = (c & 1) ? v0 : v1;
                    if (c < CHUNKS - 1) tmem_ld32_nowait(base + (uint32_t)((c + 1) * 32), vn);
                    if (c == CHUNKS - 1) release();
                    f(vc, c);
                    if (c < CHUNKS - 1) tmem_wait(vn);
                }
            } else {
#pragma unroll
                for (int c = 0; c < CHUNKS; ++c) {
                    uint32_t v0[32];
                    tmem_ld32_nowait(base + (uint32_t)(c * 32), v0);
                    tmem_wait(v0);
                    if (c == CHUNKS - 1) release();
                    f(v0, c);
                }
            }
        };

        int it_tile = 0;
        for (;; ++it_tile) {
            int tile = 0;
            if (lane == 0) tile = ring_take(it_tile, false);
            tile = __shfl_sync(0xffffffffu, tile, 0);
            if (lane == 0) mbar_arrive_cluster(cluster_addr(su32(&ring_empty[it_tile % RING]), 0));
            if (tile < 0) break;
            const int j0 = tile >> 28;
            tile &= (1 << 28) - 1;
            int job, bi, bj;
            tile_coords(p, tile, job, bi, bj);
            const int ct = it_tile & 1;  // this tile's block table
            for (int jj = 0; jj < NP; ++jj) {
                const int j = (j0 + jj) & (NP - 1);  // moduli pair (phase-rotated order)
                // pending tile: L2 prefetch one pair step ahead, and the first group of this step's
                // reconstruction loaded into registers now (its latency hides behind the residue steps)
                uint4 wa[NP];
                if (pv) {
                    if (CRT_EARLY == 1) {
                        if (jj == 0) prefetch_groups(0, GROUPS / NP);
                        if (jj + 1 < NP) prefetch_groups(((jj + 1) * GROUPS) / NP, ((jj + 2) * GROUPS) / NP);
                        load_group((jj * GROUPS) / NP, wa);
                    } else {
                        prefetch_groups((jj * GROUPS) / NP, ((jj + 1) * GROUPS) / NP);
                    }
                }
                // this pair's 16 destination blocks: those the last reconstruction step freed (the
                // first tile of the CTA takes the blocks in order)
                if (lane < GROUPS) scr_tab[ew][ct][j * GROUPS + lane] = pv ? scr_free[ew][lane] : (uint8_t)(j * GROUPS + lane);
                __syncwarp();
                // ---- first modulus a of pair j: canonical residues r_a kept as bytes (32 registers)
                uint32_t ra[CHUNKS][8];
                {
                    const uint32_t buf = g & 1u;
                    { PROF_T0();
                    mbar_wait(su32(&acc_full[buf]), (g >> 1) & 1u);
                    PROF_ADD(pw_accfull); }
                    PROF_T0();
                    fence_after();
                    const int pa = p.c.p[2 * j];
                    const unsigned mqa = p.c.bm[2 * j];
                    auto resid_a = [&](const uint32_t (&vc)[32], int c) {
#pragma unroll
                        for (int k = 0; k < 8; ++k) {
                            const uint32_t b0 = (uint32_t)mod_canon((int)vc[4 * k], pa, mqa);
                            const uint32_t b1 = (uint32_t)mod_canon((int)vc[4 * k + 1], pa, mqa);
                            const uint32_t b2 = (uint32_t)mod_canon((int)vc[4 * k + 2], pa, mqa);
                            const uint32_t b3 = (uint32_t)mod_canon((int)vc[4 * k + 3], pa, mqa);
                            ra[c][k] = __byte_perm(__byte_perm(b0, b1, 0x0040), __byte_perm(b2, b3, 0x0040), 0x5410);
                        }
                    };
                    tmem_chunks(buf, resid_a);
                    ++g;
                    PROF_ADD(pw_resid);
                }
                if (CRT_EARLY == 2 && pv) load_group((jj * GROUPS) / NP, wa);  // in flight during modulus b
                // ---- second modulus b: R = r_a + a ((r_b - r_a) a^-1 mod b) in [0, ab), stored as uint16
                {
                    const uint32_t buf = g & 1u;
                    { PROF_T0();
                    mbar_wait(su32(&acc_full[buf]), (g >> 1) & 1u);
                    PROF_ADD(pw_accfull); }
                    PROF_T0();
                    fence_after();
                    const unsigned pa = (unsigned)p.c.p[2 * j], pb = (unsigned)p.c.p[2 * j + 1], ia = (unsigned)p.c.ia[j];
                    const unsigned shb = p.c.shoup[j], offb = pb << 21;
                    auto resid_b = [&](const uint32_t (&vc)[32], int c) {
#pragma unroll
                        for (int e4 = 0; e4 < 4; ++e4) {  // 8 columns -> one 16-byte store per block
                            uint32_t pk[4];
#pragma unroll
                            for (int k = 0; k < 4; ++k) {
                                uint32_t R2[2];
#pragma unroll
                                for (int u = 0; u < 2; ++u) {
                                    const int e = 8 * e4 + 2 * k + u;
                                    // t = ((acc_b - r_a) a^-1) mod b by Shoup's multiplication: x = acc_b - r_a +
                                    // b 2^21 in [0, 2^32); q = floor(x shoup / 2^32); x ia - q b in [0, 2b)
                                    const uint32_t rav = (ra[c][e >> 2] >> (8 * (e & 3))) & 0xffu;
                                    const uint32_t x = vc[e] - rav + offb;
                                    const uint32_t r2 = x * ia - __umulhi(x, shb) * pb;
                                    const uint32_t tt = min(r2, r2 - pb);
                                    R2[u] = rav + pa * tt;
                                }
                                pk[k] = R2[0] | (R2[1] << 16);
                            }
                            uint8_t* const dst = scr0 + scr_off(scr_tab[ew][ct][j * GROUPS + c * 4 + e4], h, r);
                            if (CRT_SCRHINT)  // keep the residues in L2 until the reconstruction reads them
                                asm volatile("st.global.L2::cache_hint.v4.b32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(dst), "r"(pk[0]),
                                             "r"(pk[1]), "r"(pk[2]), "r"(pk[3]), "l"(scr_pol)
                                             : "memory");
                            else
                                *(uint4*)dst = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                        }
                    };
                    tmem_chunks(buf, resid_b);
                    ++g;
                    PROF_ADD(pw_resid);
                }
                // ---- two groups of the pending tile's reconstruction (16 groups over the NP pairs)
                if (pv) {
                    PROF_T0();
                    const int g0 = (jj * GROUPS) / NP, g1 = ((jj + 1) * GROUPS) / NP;
                    if (CRT_EARLY == 0) load_group(g0, wa);
                    if constexpr (EPI_WARPS == 8) {  // two groups in flight
                        uint4 wb[NP];
                        for (int gi = g0; gi < g1; gi += 2) {
                            if (gi + 1 < g1) load_group(gi + 1, wb);
                            recon(gi, wa);
                            if (gi + 1 < g1) recon(gi + 1, wb);
                            if (gi + 2 < g1) load_group(gi + 2, wa);
                        }
                    } else {  // one (register budget of 20 warps)
                        for (int gi = g0; gi < g1; ++gi) {
                            if (gi > g0) load_group(gi, wa);
                            recon(gi, wa);
                        }
                    }
                    free_groups(g0);
                    PROF_ADD(pw_recon);
                }
            }
            // this tile becomes the pending one
            const CrtJob jb = p.jobs[job];
            const int grow = bi * 256 + (int)crank * BM + r;  // row inside the tile
            pv = true;
            pv_tab = ct;
            pv_e0 = p.exps[jb.m * p.nb + grow] - 2 * p.c.bits;
            pv_ecol = p.exps + (size_t)jb.n * p.nb + bj * BN + h * PCOLS;
            pv_crow0 = (int)(((const char*)jb.C - (const char*)p.cbase) / ((size_t)p.nb * 8)) + bi * 256 +
                       (int)crank * BM + q * 32;
            pv_ccol0 = bj * BN + h * PCOLS;
        }
        if (pv) {  // drain: the last tile's reconstruction
            PROF_T0();
            prefetch_groups(0, GROUPS);
            uint4 wa[NP];
            if constexpr (EPI_WARPS == 8) {
                uint4 wb[NP];
                load_group(0, wa);
                for (int gi = 0; gi < GROUPS; gi += 2) {
                    load_group(gi + 1, wb);
                    recon(gi, wa);
                    if (gi + 2 < GROUPS) load_group(gi + 2, wa);
                    recon(gi + 1, wb);
                }
            } else {
                for (int gi = 0; gi < GROUPS; ++gi) {
                    load_group(gi, wa);
                    recon(gi, wa);
                }
            }
            PROF_ADD(pw_recon);
        }
        if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
#ifdef CRT_PROF
    if (blockIdx.x < 4 && (threadIdx.x == 32 || threadIdx.x == 128 || threadIdx.x == 288))
        printf("cta %d thr %d: accempty %lld full %lld | accfull %lld resid %lld recon %lld (cycles)\n", blockIdx.x,
               threadIdx.x, pw_accempty, pw_full, pw_accfull, pw_resid, pw_recon);
    if (blockIdx.x < 2 && threadIdx.x == 128)
        printf("cta %d thr %d: recon detail: staging-buffer waits %lld, first-use of the scratch loads %lld (cycles)\n",
               blockIdx.x, threadIdx.x, pw_stgwait, pw_ld);
#endif
    fence_before();
    __threadfence();
    cluster_sync();  // neither CTA frees TMEM / exits while its peer may still signal it
    if (warp == 2) {
        fence_after();
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
    }
    if (threadIdx.x == 0) atomicExch(&p.slot_flags[slot_sh], 0);
}

static PFN_cuTensorMapEncodeTiled_v12000 crt_encode() {
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

static bool crt_map(CUtensorMap* m, const int8_t* base, uint64_t planes, uint64_t rows, uint64_t cols,
                    uint64_t plane_stride, uint32_t box_rows) {
    auto fn = crt_encode();
    if (!fn) return false;
    cuuint64_t dims[3] = {cols, rows, planes};
    cuuint64_t strides[2] = {cols, plane_stride};
    cuuint32_t box[3] = {(cuuint32_t)BK, box_rows, 1};
    cuuint32_t es[3] = {1, 1, 1};
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, const_cast<int8_t*>(base), dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static bool crt_cmap(CUtensorMap* m, const void* base, uint64_t rows, uint64_t cols, bool f32) {
    auto fn = crt_encode();
    if (!fn) return false;
    cuuint64_t dims[2] = {cols, rows};
    cuuint64_t strides[1] = {cols * (f32 ? 4 : 8)};
    cuuint32_t box[2] = {8, 32};
    cuuint32_t es[2] = {1, 1};
    return fn(m, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<void*>(base), dims,
              strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, f32 ? CU_TENSOR_MAP_SWIZZLE_NONE : CU_TENSOR_MAP_SWIZZLE_64B,
              CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static int sm_count() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

int crt_scratch_slots() { return 2 * sm_count(); }
bool crt_available() { return crt_encode() != nullptr; }

cudaError_t crt_gemm_launch(const CrtArgs& a, int njobs, cudaStream_t s) {
    if (njobs <= 0) return cudaSuccess;
    // instantiations: 16 moduli (FP64 class: trailing update, DSYRK) and 8 moduli (the FP32-class
    // TRSM product A_mk W^T, reading C12'), both with an FP64 C
    if (a.nb % 256 || a.nb > 8192 || !a.scratch || !a.slot_flags) return cudaErrorInvalidValue;
    if (a.c.nmod != 16 && a.c.nmod != 8) return cudaErrorInvalidValue;
    const int ki = a.c.nmod == 16 ? 0 : 1;
    auto kern = ki == 0 ? crt_gemm_kernel<16> : crt_gemm_kernel<8>;
    static bool attr[2] = {false, false};
    if (!attr[ki]) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
        if (e != cudaSuccess) return e;
        attr[ki] = true;
    }
    CrtParams p;
    memset(&p, 0, sizeof p);
    const uint64_t rows = (uint64_t)a.nt * a.nb;
    if (!crt_map(&p.a, a.planes, (uint64_t)a.c.nmod, rows, a.nb, a.plane_stride, BM) ||
        !crt_map(&p.b, a.planes, (uint64_t)a.c.nmod, rows, a.nb, a.plane_stride, BN / 2) || !a.cbase ||
        !crt_cmap(&p.cmap, a.cbase, a.crows, a.nb, false))
        return cudaErrorInvalidValue;
    p.cbase = a.cbase;
    p.jobs = a.jobs;
    p.exps = a.exps;
    p.scratch = a.scratch;
    p.slot_flags = a.slot_flags;
    p.nslots = crt_scratch_slots();
    p.nb = a.nb;
    p.tiles_n = a.nb / BN;
    p.lower = a.lower;
    p.store = a.store;
    p.tile_counter = a.counter;
    p.phase_lock = a.phase_lock;
    if (!a.counter) return cudaErrorInvalidValue;
    p.tiles_per_job = a.lower ? p.tiles_n * (p.tiles_n + 1) / 2 : p.tiles_n * p.tiles_n;
    p.c = a.c;
    const long long total = (long long)njobs * p.tiles_per_job;
    if (total >= (1LL << 28)) return cudaErrorInvalidConfiguration;  // tile index | phase << 28 in the ring
    p.total = (int)total;
    const int max_pairs = a.max_pairs > 0 ? std::min(a.max_pairs, sm_count() / 2) : sm_count() / 2;
    const int pairs = (int)std::min<long long>(total, max_pairs);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(2 * pairs));
    cfg.blockDim = dim3(THREADS);
    cfg.dynamicSmemBytes = SMEM;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, p);
}

}  // namespace mpgeo
