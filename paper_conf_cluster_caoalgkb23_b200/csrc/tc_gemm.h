// K6 / K7 — tcgen05 tensor-core GEMMs for the FP32 class (3xTF32) and the FP16 class
// (FP16 x FP16 -> FP32) trailing updates:  C_mn (FP32 tile) -= L_m L_n^T.
#pragma once
#include <cuda_fp16.h>
#include <cuda_runtime.h>

namespace mpgeo {
struct TcJob {
    int m, n;   // panel rows of the two operands (tiles (m,k) and (n,k) of the current panel)
    float* C;   // FP32 nb x nb output tile (row-major)
};
struct TcArgs {
    const TcJob* jobs;
    const float* hi;      // TF32 hi panel cache, [nt * nb][nb]
    const float* lo;      // TF32 lo panel cache
    int nb, nt;
    const __half* p16;    // FP16 panel cache, [nt * nb][nb]
};
bool tc_gemm_available();
cudaError_t tc_gemm_tf32x3_launch(const TcArgs& a, int njobs, cudaStream_t s);
cudaError_t tc_gemm_f16_launch(const TcArgs& a, int njobs, cudaStream_t s);
}  // namespace mpgeo
