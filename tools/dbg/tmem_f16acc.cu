// Probe: where does tcgen05.mma kind::f16 with an F16 accumulator (idesc dtype = 0) put D in TMEM?
// One CTA, M = 128, N = 64, K = 16: A[i][0] = fp16(i + 1), B[j][0] = fp16((j + 1) / 64), zero elsewhere, so
// D[i][j] = (i + 1)(j + 1) / 64 (exact in FP16 for small i, j).  Reads TMEM lanes 0..31 columns 0..63 with
// tcgen05.ld.32x32b.x32 and prints the raw 32-bit words of a few lanes, then the same with an F32
// accumulator (dtype = 1) for comparison.  Operands: K-major, 128-byte swizzle (16-byte chunk c of row r
// at chunk c ^ (r % 8)), like the library's kernels.
#include <cstdint>
#include <cstdio>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
    uint64_t d = (uint64_t)((saddr & 0x3FFFFu) >> 4);
    d |= (uint64_t)1 << 16;
    d |= (uint64_t)(1024 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}

template <int DT>
__global__ void probe(uint32_t* out) {
    __shared__ __align__(1024) uint8_t sA[128 * 128];
    __shared__ __align__(1024) uint8_t sB[64 * 128];
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bar;
    const int t = threadIdx.x, warp = t >> 5;
    for (int i = t; i < 128 * 128; i += blockDim.x) sA[i] = 0;
    for (int i = t; i < 64 * 128; i += blockDim.x) sB[i] = 0;
    __syncthreads();
    if (t < 128) *(__half*)(sA + t * 128 + ((0 ^ (t % 8)) * 16)) = __float2half((float)(t + 1));
    if (t < 64) *(__half*)(sB + t * 128 + ((0 ^ (t % 8)) * 16)) = __float2half((float)(t + 1) / 64.0f);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (t == 0) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" ::"r"(su32(&tslot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tslot;
    if (t == 0) {
        const uint32_t idesc = ((uint32_t)DT << 4) | ((64u >> 3) << 17) | ((128u >> 4) << 24);
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, 0, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
                     "l"(desc_sw128(su32(sA))), "l"(desc_sw128(su32(sB))), "r"(idesc));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
        asm volatile("{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t@!p bra W_%=;\n\t}" ::"r"(su32(&bar)) : "memory");
    }
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (warp == 0) {
        uint32_t r[32];
        for (int half = 0; half < 2; ++half) {
            asm volatile(
                "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                  "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
                  "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
                  "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                : "r"(tmem + half * 32));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
            for (int c = 0; c < 32; ++c) out[t * 64 + half * 32 + c] = r[c];
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" ::"r"(tmem) : "memory");
}

int main() {
    uint32_t* d;
    cudaMalloc(&d, 32 * 64 * 4);
    for (int dt = 0; dt < 2; ++dt) {
        cudaMemset(d, 0, 32 * 64 * 4);
        if (dt == 0) probe<0><<<1, 128>>>(d); else probe<1><<<1, 128>>>(d);
        cudaError_t e = cudaDeviceSynchronize();
        uint32_t h[32 * 64];
        cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
        printf("== dtype %s (%s); expected D[i][j] = (i+1)(j+1)/64\n", dt ? "F32" : "F16", cudaGetErrorString(e));
        for (int lane : {0, 1, 2, 31}) {
            printf("lane %2d:", lane);
            for (int c = 0; c < 12; ++c) {
                const uint32_t w = h[lane * 64 + c];
                if (dt) {
                    float f;
                    memcpy(&f, &w, 4);
                    printf(" %g", f);
                } else {
                    __half_raw lo, hi;
                    lo.x = (unsigned short)(w & 0xffff);
                    hi.x = (unsigned short)(w >> 16);
                    printf(" [%g|%g]", __half2float(__half(lo)), __half2float(__half(hi)));
                }
            }
            printf("\n");
        }
        if (!dt) {  // find which word holds D[1][5] = 2*6/64
            for (int c = 0; c < 64; ++c) {
                const uint32_t w = h[1 * 64 + c];
                __half_raw lo, hi;
                lo.x = (unsigned short)(w & 0xffff);
                hi.x = (unsigned short)(w >> 16);
                if (__half2float(__half(lo)) == 12.0f / 64 || __half2float(__half(hi)) == 12.0f / 64)
                    printf("D[1][5] found in column word %d (%s half)\n", c, __half2float(__half(lo)) == 12.0f / 64 ? "low" : "high");
            }
        }
    }
    return 0;
}
