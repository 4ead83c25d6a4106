// Shared device/host helpers for libmpgeo (sm_100a only).
#pragma once
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <stdint.h>

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ < 1000)
#error "libmpgeo is built for sm_100a only (-gencode arch=compute_100a,code=sm_100a)"
#endif

namespace mpgeo {

enum Prec : uint8_t { P64 = 0, P32 = 1, P16 = 2 };

// One tile-level job for the batched kernels: operands and output pointers.
struct GemmJob {
    const void* A;
    const void* B;
    void* C;
};

// Round-to-nearest-even of an FP64 value to `prec`, returned as FP64 (cvt.rn).
__device__ __forceinline__ double round_to(double v, int prec) {
    if (prec == P32) return (double)__double2float_rn(v);
    if (prec == P16) return (double)__half2float(__double2half(v));
    return v;
}

// Warp / block reductions (fixed order => deterministic).
__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

}  // namespace mpgeo

// Kernel launch wrappers return cudaError_t; the host engine checks each one.
#define MPGEO_LAUNCH_CHECK() cudaGetLastError()
