// Microbenchmark of the operations of the CRT-16 epilogue (crt.cu) on B200: lane-ops per clock per SM
// of IMAD, IMAD.WIDE (s32 x s32 -> s64), IMAD.HI, IADD3, LOP3, PRMT, FFMA, DFMA, DADD and of the whole
// mod_canon() reduction.  8 independent chains per thread, many warps (throughput, not latency).
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ int mod_canon(int a, int p, int mq) {
    const int q = (int)(((long long)a * mq + 0x80000000LL) >> 32);
    int r = a - q * p;
    return r < 0 ? r + p : r;
}

template <int OP>
__global__ void k(int* out, int iters, int p, int mq) {
    int x[8];
    long long w[8];
    float f[8];
    double d[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        x[i] = threadIdx.x * 7 + i;
        w[i] = x[i];
        f[i] = (float)x[i];
        d[i] = (double)x[i];
    }
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if (OP == 0) x[i] = x[i] * p + mq;                                 // IMAD
            if (OP == 1) w[i] = (long long)x[i] * mq + w[i], x[i] ^= (int)w[i]; // IMAD.WIDE
            if (OP == 2) x[i] = __mulhi(x[i], mq) + i;                         // IMAD.HI
            if (OP == 3) x[i] = x[i] + p + (int)it;                            // IADD3
            if (OP == 4) x[i] = (x[i] & 0xffff) | (p << 3) ^ it;               // LOP3
            if (OP == 5) f[i] = fmaf(f[i], 1.0000001f, 1e-7f);                  // FFMA
            if (OP == 6) d[i] = fma(d[i], 1.0000001, 1e-9);                    // DFMA
            if (OP == 7) d[i] = d[i] + 1e-9;                                   // DADD
            if (OP == 8) x[i] = mod_canon(x[i] + (int)it * 977, p, mq) + 1;    // mod_canon
            if (OP == 9) x[i] = __byte_perm(x[i], p, 0x0541) + it;             // PRMT
        }
    }
    long long s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) s += x[i] + w[i] + (long long)f[i] + (long long)d[i];
    if (s == 12345) out[0] = (int)s;
}

int main() {
    int* o;
    cudaMalloc(&o, 8);
    int sms, clk;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    const char* names[] = {"IMAD", "IMAD.WIDE", "IMAD.HI", "IADD3", "LOP3", "FFMA", "DFMA", "DADD", "mod_canon", "PRMT"};
    for (int op = 0; op < 10; ++op) {
        for (int warps : {8, 16, 32}) {
            const int iters = 4096;
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0);
            cudaEventCreate(&e1);
            auto launch = [&]() {
                switch (op) {
                    case 0: k<0><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 1: k<1><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 2: k<2><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 3: k<3><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 4: k<4><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 5: k<5><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 6: k<6><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 7: k<7><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 8: k<8><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                    case 9: k<9><<<sms, warps * 32>>>(o, iters, 251, 17111111); break;
                }
            };
            launch();
            cudaEventRecord(e0);
            for (int r = 0; r < 5; ++r) launch();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            double ops = 5.0 * sms * warps * 32.0 * iters * 8;
            printf("%-10s warps/SM %2d: %8.1f Gop/s = %6.1f op/clk/SM at %.0f MHz\n", names[op], warps,
                   ops / (ms * 1e-3) / 1e9, ops / (ms * 1e-3) / sms / (clk * 1e3), clk / 1e3);
        }
    }
    return 0;
}
