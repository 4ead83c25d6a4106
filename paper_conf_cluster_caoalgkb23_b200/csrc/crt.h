// K5c — FP64-class tile GEMM on INT8 tcgen05 tensor cores by modular (CRT) integer emulation
// ("Ozaki scheme II"), see crt.cu.  SURVEY §8(f) item 4; the FP64 class of Algorithm 1 (GEMM/SYRK at
// FP64).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>


namespace mpgeo {

constexpr int CRT_NMAX = 16;

// Host-computed constants of one moduli set (passed by value to the kernels).
struct CrtConst {
    int nmod;                  // number of moduli N (even, <= 16)
    int bits;                  // operand integers: x' = rint(x 2^(bits - e_row)), |x'| <= 2^bits
    int p[CRT_NMAX];           // pairwise coprime moduli <= 256
    unsigned bm[CRT_NMAX];     // ceil(2^38 / p): exact Barrett floor((a + p 2^20) / p) for |a| <= 2^27 (crt.cu)
    double invp[CRT_NMAX];     // 1/p (FP64, for the operand residues)
    int ia[CRT_NMAX / 2];      // p_2j^-1 mod p_2j+1
    unsigned shoup[CRT_NMAX / 2];  // floor(ia_j 2^32 / p_2j+1): Shoup's modular multiplication by ia_j
    int mpair[CRT_NMAX / 2];   // m_j = p_2j p_2j+1
    double H[CRT_NMAX / 2];    // w_j = (M/m_j) ((M/m_j)^-1 mod m_j) = H_j + L_j, H_j a multiple of 2^sh
    double L[CRT_NMAX / 2];    //   with < 2^33 units (sum_j R_j H_j exact), L_j < 2^sh
    double Mh, Ml, invM;       // M = prod p_t = Mh + Ml (same split), 1/M
    // Reconstruction in integer + FP32 arithmetic (crt_recon_bits): the FP64 pipe is unusable inside the
    // GEMM — it shares the tensor core's datapath and runs ~25x slower while tcgen05 MMAs are in flight
    // (tools/dbg/mma_contention.cu, profiles/r02/mma_contention.txt).
    int ld;                        // low 32-bit limbs of w_j and M dropped (1 when M >= 2^64, else 0)
    uint32_t W[CRT_NMAX / 2][3];   // limbs of w_j >> 32 ld (w_j < M)
    uint32_t Mw[3];                // limbs of M >> 32 ld
    float cw[CRT_NMAX / 2];        // fl32(w_j / M): the quotient estimate's weights
    float hoff[CRT_NMAX / 2];      // 2^23 + h_j, h_j = floor(m_j / 2) (centred residues R_j - h_j in FP32)
    float fD;                      // frac(D) in FP32 and
    int Dq;                        //   floor(D), D = sum_j h_j w_j / M (exact, host big-integer arithmetic)
};

// Constants for the first `nmod` moduli and inner dimension K (bits = largest b with K 2^{2b} <=
// 0.3 M, so |sum_k x'_ik y'_jk| <= 0.3 M: the CRT result is unique and the FP32 quotient estimate of
// crt_recon_bits, off by <= 0.125, still rounds to the exact quotient).
bool crt_constants(int nmod, int K, CrtConst* c);

#if defined(__CUDACC__)
#define CRT_HD __host__ __device__ __forceinline__
#else
#define CRT_HD inline
#endif
CRT_HD float crt_fadd(float a, float b) {
#ifdef __CUDA_ARCH__
    return __fadd_rn(a, b);
#else
    return a + b;  // host: IEEE single, -ffp-contract=off
#endif
}
CRT_HD float crt_fma(float a, float b, float c) {
#ifdef __CUDA_ARCH__
    return __fmaf_rn(a, b, c);
#else
    return __builtin_fmaf(a, b, c);
#endif
}
CRT_HD int crt_clz32(uint32_t v) {
#ifdef __CUDA_ARCH__
    return __clz((int)v);
#else
    return v ? __builtin_clz(v) : 32;
#endif
}
CRT_HD int crt_clz64(uint64_t v) {
#ifdef __CUDA_ARCH__
    return __clzll((long long)v);
#else
    return v ? __builtin_clzll(v) : 64;
#endif
}
CRT_HD float crt_bits_f(uint32_t v) {
#ifdef __CUDA_ARCH__
    return __uint_as_float(v);
#else
    float f;
    __builtin_memcpy(&f, &v, 4);
    return f;
#endif
}
CRT_HD uint32_t crt_f_bits(float f) {
#ifdef __CUDA_ARCH__
    return __float_as_uint(f);
#else
    uint32_t v;
    __builtin_memcpy(&v, &f, 4);
    return v;
#endif
}

// CRT reconstruction of one element, without FP64 arithmetic.  R[j] in [0, m_j) are the combined
// residues of the NP = nmod/2 paired moduli; the integer X = sum_j R_j w_j - q M (|X| <= 0.3 M) is
// returned as the FP64 bit pattern of (-1)^neg X 2^e0.
//  1. quotient: q = Dq + rint(frac(D) + sum_j (R_j - h_j) fl32(w_j/M)) in FP32 (two chains of NP/2
//     FFMAs; |R_j - h_j| <= 2^15 so the partial sums stay <= 2^17 and the estimate errs by <= 2^-3 —
//     within the 0.5 - 0.3 margin of the exact S/M = q + X/M).
//  2. X' = (S - q M) / 2^(32 ld) modulo 2^96 in three 32-bit limbs (products R_j W_j,l: 48 bits, sums
//     of NP in 64-bit registers; the top limb only modulo 2^32).  The dropped low limbs cost
//     < NP 2^16 2^32 + q 2^32 <= 2^51.6 absolute on X (ld = 1), against the operand rounding bound
//     K 2^b = 2^67 of the engine (crt.cu) — 2^-15 of it; with ld = 0 X' = X exactly.
//  3. |X'| normalised by count-leading-zeros, rounded to 53 bits (half up) and packed with the
//     exponent 32 ld + e0 + (position of the leading bit): plain integer instructions.
// Values below 2^-1022 flush to zero (a CRT product that small is far below FP64 resolution of C).
template <int NP>
CRT_HD uint64_t crt_recon_bits(const uint32_t (&R)[NP], const CrtConst& c, int e0, uint32_t neg) {
    uint64_t a0 = 0, a1 = 0;
    uint32_t a2 = 0;
    float ue = c.fD, uo = 0.0f;
#pragma unroll
    for (int j = 0; j < NP; ++j) {
        a0 += (uint64_t)R[j] * c.W[j][0];
        a1 += (uint64_t)R[j] * c.W[j][1];
        a2 += R[j] * c.W[j][2];
        const float rc = crt_fadd(crt_bits_f(R[j] | 0x4B000000u), -c.hoff[j]);  // R_j - h_j, exact
        if (j & 1) uo = crt_fma(rc, c.cw[j], uo);
        else ue = crt_fma(rc, c.cw[j], ue);
    }
    // rint by the 1.5 2^23 magic (|ue + uo| < 2^19): the integer sits in the low mantissa bits
    const uint32_t q = (uint32_t)(c.Dq + (int)(crt_f_bits(crt_fadd(crt_fadd(ue, uo), 12582912.0f)) - 0x4B400000u));
    const int64_t t0 = (int64_t)(a0 - (uint64_t)q * c.Mw[0]);
    const int64_t t1 = (int64_t)(a1 - (uint64_t)q * c.Mw[1]) + (t0 >> 32);
    const uint32_t x2 = a2 - q * c.Mw[2] + (uint32_t)((uint64_t)t1 >> 32);
    // |X'| as hi:lo (96 bits, hi < 2^28), sign s
    const uint32_t s = (uint32_t)((int32_t)x2 >> 31);
    const uint64_t s64 = ((uint64_t)s << 32) | s;
    const uint64_t lx = (((uint64_t)(uint32_t)t1 << 32) | (uint32_t)t0) ^ s64;
    const uint64_t lo = lx + (s & 1u);
    const uint32_t hi = (x2 ^ s) + (uint32_t)(lo < lx);
    // |X'| = T 2^k with T in [2^63, 2^64); both normalisations computed, one selected (no branch)
    const int n32 = crt_clz32(hi), n64 = crt_clz64(lo);  // hi != 0: n32 >= 4
    const uint64_t Tb = ((uint64_t)hi << ((32 + n32) & 63)) | (lo >> ((32 - n32) & 63));
    const uint64_t Ts = lo << (n64 & 63);
    const bool big = hi != 0;
    const uint64_t T = big ? Tb : Ts;
    const int k = big ? 32 - n32 : -n64;
    const int ef = 63 + k + 32 * c.ld + e0 + 1022;  // biased exponent - 1 (T >> 11 carries the leading 1)
    const uint64_t sign = (uint64_t)((s ^ neg) & 1u) << 63;
    const uint64_t bits = sign | (((uint64_t)(uint32_t)ef << 52) + (T >> 11) + ((T >> 10) & 1u));
    return (!big && lo == 0) || ef < 0 ? sign : bits;
}

struct CrtJob {
    int m, n;   // panel rows of the operands (residue-cache rows m*nb.., n*nb..)
    void* C;    // nb x nb output tile (FP64)
};
struct CrtSplitItem {
    const double* src;     // FP64 nb x nb tile (panel slot)
    int8_t* dst;           // residue planes: plane i at dst + i * plane_stride, row-major nb x nb
    int* exps;             // per-row exponents e (max_j |x_ij| < 2^e), nb
    int64_t plane_stride;  // bytes between planes
};
struct CrtArgs {
    const CrtJob* jobs;
    const int8_t* planes;  // residue cache: nmod planes of [nt*nb][nb] int8
    const int* exps;       // [nt*nb] row exponents
    int64_t plane_stride;  // = nt*nb*nb
    int nb, nt, lower;
    uint8_t* scratch;      // residue staging: crt_scratch_slots() x CRT_SLOT_BYTES
    int* slot_flags;       // crt_scratch_slots() ints, zero-initialised
    CrtConst c;            // copied into the launch parameters
    const void* cbase;     // C tiles lie inside [cbase, cbase + crows * nb) at whole-row offsets
    uint64_t crows;        //   (a view of the tile pool in C's type; C is updated by TMA reduce-add)
    int max_pairs;         // persistent grid in CTA pairs (0: one pair per 2 SMs)
    int store = 0;         // 1: C = P_m P_n^T (overwrite), 0: C -= P_m P_n^T
    int* counter = nullptr;  // 2 device ints of this launch, zero at launch: tile counter, modulus phase
    int phase_lock = 1;    // 1: each tile starts at the modulus pair the other CTAs are on
};
// One CTA's residue staging: per 128-column half, 2 KB blocks (128 rows x one 8-column group of one
// moduli pair, uint16 residues); a tile needs N/2 x 16 blocks per half and the epilogue recycles the
// blocks tile T-1's reconstruction frees for tile T's residues, so one tile + 16 spare blocks suffice
// (the block permutation is tracked per warp in shared memory, crt.cu)
constexpr int CRT_SCR_BLOCK = 128 * 16;
constexpr int CRT_SCR_BLOCKS = CRT_NMAX / 2 * 16 + 16;  // per column half
constexpr size_t CRT_SLOT_BYTES = (size_t)2 * CRT_SCR_BLOCKS * CRT_SCR_BLOCK;
int crt_scratch_slots();                                         // 2 x SM count
bool crt_available();
cudaError_t crt_split_launch(const CrtSplitItem* items, int n, int nb, const CrtConst& c, cudaStream_t s);
cudaError_t crt_gemm_launch(const CrtArgs& a, int njobs, cudaStream_t s);
}  // namespace mpgeo
