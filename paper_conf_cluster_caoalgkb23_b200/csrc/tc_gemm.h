// K6 / K7 — tcgen05 tensor-core GEMMs for the trailing update of FP32-class and FP16-class tiles
// (GEMM(m,n,k) at kernel(m,n)):   C_mn (FP32 tile) -= L_mk L_nk^T
//   FP16 class  (the paper's FP16_32): FP16 operands, FP32 accumulation in TMEM (kind::f16); the
//                operands are the row-scaled FP16 hi planes of the 3xFP16 split (x = 2^e hi up to
//                FP16 rounding), so FP16-class entries far below 2^-14 do not underflow;
//   FP32 class : 3xTF32 — hi = rna_tf32(a), lo = rna_tf32(a - hi), C -= hi.hi + hi.lo + lo.hi with
//                an FP32 TMEM accumulator (kind::tf32), reading C13 in DESIGN.md.
// Operands are the consumer-side conversions of the panel (K2), stored as [nt*nb][nb] row-major
// caches and fetched with TMA (128-byte swizzle) into a multi-stage mbarrier pipeline.
#pragma once
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

namespace mpgeo {
struct TcJob {
    int m, n;    // panel rows of the two operands (tiles (m,k) and (n,k) of the current panel)
    void* C;     // nb x nb output tile (row-major): FP32, or FP16 with TcArgs::c16 (FP16 storage class)
    int cscale;  // c16: the C tile's exponent (stored value fp16(x 2^cscale))
    int pad;
};
struct TcArgs {
    const TcJob* jobs;
    const float* hi;      // TF32 hi panel cache, [nt * nb][nb]
    const float* lo;      // TF32 lo panel cache
    int nb, nt;
    // row-scaled FP16 hi / lo panel caches [nt * nb][nb] (split16_kernel) and the per-row exponents e
    // (x = 2^e (hi + lo) up to the split error): hi + lo for the 3xFP16 FP32 class, hi alone for the
    // FP16 class
    const __half* h16hi = nullptr;
    const __half* h16lo = nullptr;
    const int* e16 = nullptr;
    int persistent = 0;  // 3xFP16: persistent CTA-pair kernel (mp_config::f16x3_persistent)
    int pairs = 0;       // persistent 3xFP16 kernel: CTA pairs to use (0: all SMs / 2)
    // every TcJob::C lies in [cbase, cbase + crows rows of nb elements) at a whole row offset (the
    // epilogue reduces into C through one TMA tensor map over this range)
    const void* cbase;
    uint64_t crows;
    int c16 = 0;  // FP16-class GEMM only: C tiles are FP16 (reduce-added in FP16, scaled by 2^cscale)
};
bool tc_gemm_available();
cudaError_t tc_gemm_tf32x3_launch(const TcArgs& a, int njobs, cudaStream_t s);
cudaError_t tc_gemm_f16_launch(const TcArgs& a, int njobs, cudaStream_t s);
// pure-FP16 class (four-level maps): h16hi = the hs planes (split16_kernel, extra 2^-13 per row), F16
// accumulation in TMEM over the whole K, FP32 C
cudaError_t tc_gemm_f16h_launch(const TcArgs& a, int njobs, cudaStream_t s);
cudaError_t tc_gemm_f16x3_launch(const TcArgs& a, int njobs, cudaStream_t s);
}  // namespace mpgeo
