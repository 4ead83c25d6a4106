// Microbenchmark: does a running tcgen05 MMA stream slow the SM's ALU pipes?  One CTA per SM; warp 0
// issues back-to-back tcgen05.mma (kind::i8 or kind::f16, M = 128, N = 256, K = 32, cta_group::1) on
// garbage shared-memory operands while warps 4..11 run independent chains of one ALU op (DFMA, FFMA,
// IMAD, IMAD.HI, DADD+cvt) and time themselves with clock64.  Prints lane-ops per clock per SM and
// the MMA rate (MACs per clock per SM) for every (op, mma) combination.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mc mma_contention.cu
#include <cstdint>
#include <cstdio>
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
constexpr uint32_t ID_I8 = (2u << 4) | (1u << 7) | (1u << 10) | ((256u >> 3) << 17) | ((128u >> 4) << 24);
constexpr uint32_t ID_F16 = (1u << 4) | ((256u >> 3) << 17) | ((128u >> 4) << 24);

struct Res { long long alu_cyc; long long mma_cyc; long long mmas; };

template <int OP, int MMA>  // MMA: 0 none, 1 i8, 2 f16
__global__ void __launch_bounds__(384, 1) k(Res* out, int iters, double a, double b, volatile int* stop_flag) {
    extern __shared__ __align__(1024) uint8_t sm[];
    uint8_t* s = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bar;
    __shared__ volatile int alu_done;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
        alu_done = 0;
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&tslot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tslot;
    if (warp == 0) {
        if (MMA && lane == 0) {
            const uint64_t ad = desc_sw128(su32(s)), bd = desc_sw128(su32(s + 16384));
            long long t0 = clock64(), n = 0;
            uint32_t ph = 0;
            while (!alu_done) {
                for (int i = 0; i < 64; ++i) {
                    if (MMA == 1)
                        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                     "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
                                     "l"(ad), "l"(bd), "r"(ID_I8), "r"(i));
                    else
                        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                     "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
                                     "l"(ad), "l"(bd), "r"(ID_F16), "r"(i));
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
                asm volatile("{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}" ::"r"(su32(&bar)), "r"(ph) : "memory");
                ph ^= 1u;
                n += 64;
            }
            if (blockIdx.x == 0) { out->mma_cyc = clock64() - t0; out->mmas = n; }
        }
    } else if (warp >= 4) {
        double x[8];
        float f[8];
        uint32_t y[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) { x[i] = threadIdx.x * 1e-3 + i; f[i] = (float)x[i]; y[i] = threadIdx.x * 7 + i; }
        // let the MMA stream start
        for (long long w = clock64(); clock64() - w < 20000;) {}
        long long t0 = clock64();
        for (int it = 0; it < iters; ++it) {
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                if (OP == 0) x[i] = fma(x[i], a, b);
                if (OP == 1) f[i] = __fmaf_rn(f[i], (float)a, (float)b);
                if (OP == 2) y[i] = y[i] * (uint32_t)iters + (uint32_t)i;
                if (OP == 3) y[i] = __umulhi(y[i], 0x9E3779B9u) + (uint32_t)i;
                if (OP == 4) x[i] = x[i] + b;
                if (OP == 5 && (i & 1) == 0) {  // DMMA m8n8k4: 2 FP64 MACs x 64 per thread-instruction pair
                    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
                                 : "+d"(x[i]), "+d"(x[i + 1]) : "d"(a), "d"(b));
                }
            }
        }
        long long t1 = clock64();
        double sum = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) sum += x[i] + f[i] + y[i];
        if (sum == 1.2345) out->mmas = -1;
        if (blockIdx.x == 0 && threadIdx.x == 128) out->alu_cyc = t1 - t0;
        asm volatile("bar.sync 1, 256;" ::: "memory");
        if (threadIdx.x == 128) alu_done = 1;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 2) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tmem) : "memory");
    }
}

template <int OP, int MMA>
void run(const char* name, int sms, Res* d) {
    const int smem = 64 * 1024;
    cudaFuncSetAttribute(k<OP, MMA>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    const int iters = 20000;
    k<OP, MMA><<<sms, 384, 200 * 1024>>>(d, iters, 1.0000001, 1e-9, nullptr);
    cudaDeviceSynchronize();
    cudaMemset(d, 0, sizeof(Res));
    k<OP, MMA><<<sms, 384, 200 * 1024>>>(d, iters, 1.0000001, 1e-9, nullptr);
    cudaError_t e = cudaDeviceSynchronize();
    Res h;
    cudaMemcpy(&h, d, sizeof h, cudaMemcpyDeviceToHost);
    // lane-ops per clock per SM (8 warps); DMMA: FP64 MACs per clock per SM (4 mma per iteration and warp, 256 MACs each)
    const double alu_rate = OP == 5 ? 8.0 * iters * 4 * 256 / (double)h.alu_cyc : 8.0 * 32 * iters * 8 / (double)h.alu_cyc;
    const double mac = MMA ? (double)h.mmas * 128 * 256 * 32 / (double)h.mma_cyc : 0.0;
    printf("%-8s mma=%-4s: ALU %6.1f lane-op/clk/SM   MMA %7.0f MAC/clk/SM  (%s)\n", name, MMA == 0 ? "none" : MMA == 1 ? "i8" : "f16",
           alu_rate, mac, cudaGetErrorString(e));
    (void)smem;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    Res* d;
    cudaMalloc(&d, sizeof(Res));
    run<0, 0>("DFMA", sms, d); run<0, 1>("DFMA", sms, d); run<0, 2>("DFMA", sms, d);
    run<4, 0>("DADD", sms, d); run<4, 1>("DADD", sms, d);
    run<1, 0>("FFMA", sms, d); run<1, 1>("FFMA", sms, d); run<1, 2>("FFMA", sms, d);
    run<2, 0>("IMAD", sms, d); run<2, 1>("IMAD", sms, d); run<2, 2>("IMAD", sms, d);
    run<3, 0>("IMAD.HI", sms, d); run<3, 1>("IMAD.HI", sms, d);
    run<5, 0>("DMMA", sms, d); run<5, 1>("DMMA", sms, d); run<5, 2>("DMMA", sms, d);
    return 0;
}
