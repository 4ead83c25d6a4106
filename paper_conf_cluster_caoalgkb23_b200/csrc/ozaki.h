// K5b — FP64-class GEMM on INT8 tcgen05 tensor cores (Ozaki splitting), see ozaki.cu.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace mpgeo {
struct OzSplitItem {
    const double* src;     // FP64 nb x nb tile (panel slot)
    int8_t* dst;           // slice planes: plane s at dst + s * plane_stride, row-major nb x nb
    int* exps;             // per-row exponents (nb)
    int64_t plane_stride;  // bytes between slice planes
};
struct OzJob {
    int m, n;   // panel rows of the operands (slice-cache rows m*nb.., n*nb..)
    void* C;    // nb x nb output tile (FP64, or FP32 when c_f32)
};
struct OzArgs {
    const OzJob* jobs;
    const int8_t* slices;  // slice cache: S planes of [nt*nb][nb] int8
    const int* exps;       // [nt*nb] row exponents
    int64_t plane_stride;  // = nt*nb*nb
    int nb, nt, S, lower;
    int c_f32;             // C tiles are FP32 (FP32 class, S = 4) instead of FP64 (S = 8)
};
bool ozaki_available();
cudaError_t ozaki_split_launch(const OzSplitItem* items, int n, int nb, int S, cudaStream_t s);
cudaError_t ozaki_gemm_launch(const OzArgs& a, int njobs, cudaStream_t s);
}  // namespace mpgeo
