// Multi-GPU panel exchange over peer memory.
//
// Every rank owns the tiles (m, k) with owner(m, k) = (m mod P) * Q + (k mod Q).  When a
// panel tile is final (L~_kk after POTRF, L_mk after TRSM) its producer PACKS it into its send area
// in the communication precision of Algorithm 2 (FP64 / FP32 / FP16 bytes: tiles travel in
// storage or comm precision, never wider) and PUBLISHES a stamp (k + 1) with a system-scope
// release store.  Each consumer runs one fused kernel that waits for the stamp with a
// system-scope acquire load, reads the payload straight from the producer's memory (NVLink
// peer load; across processes on one device it is the same-device IPC mapping) and up-converts it
// on the fly into its own FP64 panel slot — the transfer and the target-side conversion (TTC,
// P:156) are one kernel; the consumer's operand formats are derived from that slot once per panel
// (engine.cu, step 5e).  Both kernels move 32 bytes of FP64 (4 elements) per thread and iteration
// and size their grids to a few waves of the SMs.
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

// Pack FP64 sources (already rounded to their communication precision) into payloads (elems % 4 == 0).
__global__ void __launch_bounds__(256) pack_kernel(const PackItem* items, int64_t elems) {
    const PackItem it = items[blockIdx.y];
    const int64_t stride = (int64_t)gridDim.x * blockDim.x * 4;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 4; i < elems; i += stride) {
        const double2 a = *(const double2*)(it.src + i), b = *(const double2*)(it.src + i + 2);
        if (it.prec == P64) {
            *(double2*)((double*)it.dst + i) = a;
            *(double2*)((double*)it.dst + i + 2) = b;
        } else if (it.prec == P32) {
            *(float4*)((float*)it.dst + i) =
                make_float4(__double2float_rn(a.x), __double2float_rn(a.y), __double2float_rn(b.x), __double2float_rn(b.y));
        } else {
            __half2 h[2] = {__halves2half2(store16(a.x, it.scale), store16(a.y, it.scale)),
                            __halves2half2(store16(b.x, it.scale), store16(b.y, it.scale))};
            *(uint2*)((__half*)it.dst + i) = *(const uint2*)h;
        }
    }
}

// Fused pull + up-convert: peer payload (comm precision) -> local FP64 panel slot (elems % 4 == 0).
__global__ void __launch_bounds__(256) pull_kernel(const PullItem* items, int64_t elems) {
    const PullItem it = items[blockIdx.y];
    if (threadIdx.x == 0) {  // acquire the producer's stamp (already reached: wait_flags ran first)
        while (ld_acquire_sys(it.flag) < it.target) __nanosleep(64);
    }
    __syncthreads();
    const int64_t stride = (int64_t)gridDim.x * blockDim.x * 4;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 4; i < elems; i += stride) {
        double2 a, b;
        if (it.prec == P64) {
            a = *(const double2*)((const double*)it.src + i);
            b = *(const double2*)((const double*)it.src + i + 2);
        } else if (it.prec == P32) {
            const float4 f = *(const float4*)((const float*)it.src + i);
            a = make_double2(f.x, f.y);
            b = make_double2(f.z, f.w);
        } else {
            const uint2 u = *(const uint2*)((const __half*)it.src + i);
            const __half2 h0 = *(const __half2*)&u.x, h1 = *(const __half2*)&u.y;
            a = make_double2(load16(__low2half(h0), it.scale), load16(__high2half(h0), it.scale));
            b = make_double2(load16(__low2half(h1), it.scale), load16(__high2half(h1), it.scale));
        }
        *(double2*)(it.p64 + i) = a;
        *(double2*)(it.p64 + i + 2) = b;
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

// grid: about four waves of 148 SMs x 8 CTAs over all items, at least one CTA per item
static dim3 xfer_grid(int64_t elems, int n) {
    int64_t per = (4LL * 148 * 8 + n - 1) / n;
    const int64_t maxc = (elems / 4 + 255) / 256;
    per = std::max<int64_t>(1, std::min(per, maxc));
    return dim3((unsigned)per, n);
}

cudaError_t pack_launch(const PackItem* items, int n, int64_t elems, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    if (elems % 4) return cudaErrorInvalidValue;
    pack_kernel<<<xfer_grid(elems, n), 256, 0, s>>>(items, elems);
    return cudaGetLastError();
}

cudaError_t pull_launch(const PullItem* items, int n, int64_t elems, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    if (elems % 4) return cudaErrorInvalidValue;
    pull_kernel<<<xfer_grid(elems, n), 256, 0, s>>>(items, elems);
    return cudaGetLastError();
}

cudaError_t gather_add_launch(const GatherItem& g, int len, cudaStream_t s) {
    gather_add_kernel<<<(len + 255) / 256, 256, 0, s>>>(g, len);
    return cudaGetLastError();
}

}  // namespace mpgeo
