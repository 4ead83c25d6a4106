// Microbenchmark: DFMA / DADD / IMAD throughput per SM on this GPU (independent chains, many warps).
#include <cstdio>
#include <cuda_runtime.h>
template <int OP>
__global__ void k(double* out, int iters, double a, double b) {
    double x[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x * 1e-3 + i;
    long long y[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) y[i] = threadIdx.x + i;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if (OP == 0) x[i] = fma(x[i], a, b);
            if (OP == 1) x[i] = x[i] + b;
            if (OP == 2) y[i] = y[i] * (long long)iters + (unsigned)i;
            if (OP == 3) { float f = (float)x[i]; f = __fmaf_rn(f, (float)a, (float)b); x[i] = f; }
        }
    }
    double s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) s += x[i] + (double)y[i];
    if (s == 1.2345) out[0] = s;
}
int main() {
    double* o;
    cudaMalloc(&o, 8);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    const char* names[] = {"DFMA", "DADD", "IMAD64", "FFMA+cvt"};
    for (int op = 0; op < 4; ++op) {
        for (int warps : {4, 8, 16, 32}) {
            const int iters = 4096;
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0);
            cudaEventCreate(&e1);
            auto launch = [&]() {
                if (op == 0) k<0><<<sms, warps * 32>>>(o, iters, 1.0000001, 1e-9);
                if (op == 1) k<1><<<sms, warps * 32>>>(o, iters, 1.0000001, 1e-9);
                if (op == 2) k<2><<<sms, warps * 32>>>(o, iters, 1.0000001, 1e-9);
                if (op == 3) k<3><<<sms, warps * 32>>>(o, iters, 1.0000001, 1e-9);
            };
            launch();
            cudaEventRecord(e0);
            for (int r = 0; r < 5; ++r) launch();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            double ops = 5.0 * sms * warps * 32.0 * iters * 8;
            printf("%-9s warps/SM %2d: %.1f Gop/s = %.1f op/clk/SM at max clock %.0f MHz\n", names[op], warps,
                   ops / (ms * 1e-3) / 1e9, ops / (ms * 1e-3) / sms / (clk * 1e3), clk / 1e3);
        }
    }
    return 0;
}
