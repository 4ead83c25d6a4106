// Peer-memory panel exchange kernels (dist.cu).
#pragma once
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

namespace mpgeo {
struct WaitItem {
    const uint64_t* flag;  // a peer's (or own) stamp
    uint64_t target;       // wait until *flag >= target
};
struct PackItem {
    const double* src;  // FP64 values already rounded to `prec`
    void* dst;          // own send slot
    int prec;
    int scale;          // P16 payload: fp16(x 2^scale) (0 = the plain FP16 of STC; the FP16 storage class's exponent)
};
struct PullItem {
    const void* src;       // peer payload (comm precision)
    const uint64_t* flag;  // peer stamp for that payload
    uint64_t target;
    double* p64;           // local FP64 panel slot (the operand formats are derived from it later)
    int prec;
    int scale;             // P16 payload exponent (see PackItem)
};
constexpr int MAX_PEERS = 8;
struct GatherItem {
    const double* base;            // z_k (may be null)
    const double* src[MAX_PEERS];  // partial vectors (already negative sums)
    int n;
    double* dst;                   // base + sum src (fixed order)
};
cudaError_t wait_flags_launch(const WaitItem* items, int n, cudaStream_t s);
cudaError_t set_flag_launch(uint64_t* flag, uint64_t v, cudaStream_t s);
cudaError_t pack_launch(const PackItem* items, int n, int64_t elems, cudaStream_t s);
cudaError_t pull_launch(const PullItem* items, int n, int64_t elems, cudaStream_t s);
cudaError_t gather_add_launch(const GatherItem& g, int len, cudaStream_t s);
}  // namespace mpgeo
