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
    int mpair[CRT_NMAX / 2];   // m_j = p_2j p_2j+1
    double H[CRT_NMAX / 2];    // w_j = (M/m_j) ((M/m_j)^-1 mod m_j) = H_j + L_j, H_j a multiple of 2^sh
    double L[CRT_NMAX / 2];    //   with < 2^33 units (sum_j R_j H_j exact), L_j < 2^sh
    double Mh, Ml, invM;       // M = prod p_t = Mh + Ml (same split), 1/M
};

// Constants for the first `nmod` moduli and inner dimension K (bits = largest b with
// 2b + log2(K) + 1 < log2(M), so |sum_k x'_ik y'_jk| < M/2 and the CRT result is unique).
bool crt_constants(int nmod, int K, CrtConst* c);

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
