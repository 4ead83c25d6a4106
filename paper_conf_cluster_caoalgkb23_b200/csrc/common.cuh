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

// FP16 storage class (mp_config::fp16_storage): an FP16-class tile is stored as
// fp16(x 2^t) with one power-of-two exponent t per tile (chosen from the tile norm so the stored values
// stay far inside the FP16 range, engine.cu), read back as fp16 2^-t: 11 significant bits per entry
// without FP16's underflow.  2^t is built from its exponent bits (|t| <= 1000).
__device__ __forceinline__ double pow2d(int t) { return __hiloint2double((t + 1023) << 20, 0); }
__device__ __forceinline__ __half store16(double v, int t) { return __double2half(v * pow2d(t)); }
__device__ __forceinline__ double load16(__half h, int t) { return (double)__half2float(h) * pow2d(-t); }

// Warp / block reductions (fixed order => deterministic).
__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

}  // namespace mpgeo

// Kernel launch wrappers return cudaError_t; the host engine checks each one.
#define MPGEO_LAUNCH_CHECK() cudaGetLastError()
