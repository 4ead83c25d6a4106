// Multi-GPU panel exchange over peer memory.
//
// Every rank owns the tiles (m, k) with owner(m, k) = (m mod P) * Q + (k mod Q).  When a
// panel tile is final (L~_kk after POTRF, L_mk after TRSM) its producer PACKS it into its send area
// in the communication precision of Algorithm 2 (FP64 / FP32 / FP16 bytes: tiles travel in
// storage or comm precision, never wider) and PUBLISHES a stamp (k + 1) with a system-scope
// release store.  Each consumer runs one fused kernel that waits for the stamp with a
// system-scope acquire load, reads the payload straight from the producer's memory (NVLink
// peer load; across processes on one device it is the same-device IPC mapping) and converts it
// on the fly into its own FP64 panel slot and, if its successors need them, the FP16 and TF32
// hi/lo operand caches — the transfer and the target-side conversion (TTC) are one kernel.
// A consumer stamps `done` when it has pulled everything of a panel; a producer waits for every
// peer's `done` of panel k-2 before reusing that send slot (two slot sets, panel parity).
#include "common.cuh"
#include "dist.h"

namespace mpgeo {

__device__ __forceinline__ uint64_t ld_acquire_sys(const volatile uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(volatile uint64_t* p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ float tf32_rna_d(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return __uint_as_float(r);
}

// Wait until every flag[i] >= target[i] (one thread; the list is short).
__global__ void wait_flags_kernel(const WaitItem* items, int n) {
    if (threadIdx.x != 0) return;
    for (int i = 0; i < n; ++i) {
        const volatile uint64_t* f = items[i].flag;
        const uint64_t t = items[i].target;
        while (ld_acquire_sys(f) < t) __nanosleep(256);
    }
}

__global__ void set_flag_kernel(uint64_t* flag, uint64_t v) {
    __threadfence_system();
    st_release_sys(flag, v);
}

// Pack FP64 sources (already rounded to their communication precision) into payloads.
__global__ void pack_kernel(const PackItem* items, int64_t elems) {
    const PackItem it = items[blockIdx.y];
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < elems; i += stride) {
        const double v = it.src[i];
        if (it.prec == P64) ((double*)it.dst)[i] = v;
        else if (it.prec == P32) ((float*)it.dst)[i] = __double2float_rn(v);
        else ((__half*)it.dst)[i] = __double2half(v);
    }
}

// Fused pull + convert: peer payload (comm precision) -> local FP64 panel slot (+ caches).
__global__ void pull_kernel(const PullItem* items, int64_t elems) {
    const PullItem it = items[blockIdx.y];
    if (threadIdx.x == 0) {  // acquire the producer's stamp (already reached: wait_flags ran first)
        while (ld_acquire_sys(it.flag) < it.target) __nanosleep(64);
    }
    __syncthreads();
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < elems; i += stride) {
        double v;
        if (it.prec == P64) v = ((const double*)it.src)[i];
        else if (it.prec == P32) v = (double)((const float*)it.src)[i];
        else v = (double)__half2float(((const __half*)it.src)[i]);
        it.p64[i] = v;
        if (it.p16) it.p16[i] = __double2half(v);
        if (it.hi) {
            const float f = __double2float_rn(v);
            const float h = tf32_rna_d(f);
            it.hi[i] = h;
            it.lo[i] = tf32_rna_d(f - h);
        }
    }
}

// dst[i] = base[i] + sum_r src_r[i] over the peers' partial vectors, in fixed rank order.
__global__ void gather_add_kernel(const GatherItem g, int len) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= len) return;
    double s = g.base ? g.base[i] : 0.0;
    for (int r = 0; r < g.n; ++r) s += g.src[r][i];
    g.dst[i] = s;
}

cudaError_t wait_flags_launch(const WaitItem* items, int n, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    wait_flags_kernel<<<1, 32, 0, s>>>(items, n);
    return cudaGetLastError();
}

cudaError_t set_flag_launch(uint64_t* flag, uint64_t v, cudaStream_t s) {
    set_flag_kernel<<<1, 1, 0, s>>>(flag, v);
    return cudaGetLastError();
}

cudaError_t pack_launch(const PackItem* items, int n, int64_t elems, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    dim3 grid((unsigned)std::min<int64_t>((elems + 255) / 256, 64), n);
    pack_kernel<<<grid, 256, 0, s>>>(items, elems);
    return cudaGetLastError();
}

cudaError_t pull_launch(const PullItem* items, int n, int64_t elems, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    dim3 grid((unsigned)std::min<int64_t>((elems + 255) / 256, 64), n);
    pull_kernel<<<grid, 256, 0, s>>>(items, elems);
    return cudaGetLastError();
}

cudaError_t gather_add_launch(const GatherItem& g, int len, cudaStream_t s) {
    gather_add_kernel<<<(len + 255) / 256, 256, 0, s>>>(g, len);
    return cudaGetLastError();
}

}  // namespace mpgeo
