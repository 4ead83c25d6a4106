// Microbenchmark: per-SM throughput of DFMA, DADD, FFMA, IMAD, I2F.F64 on sm_100a.
#include <cstdio>
#include <cuda_runtime.h>
template <int OP>
__global__ void k(double* out, int iters) {
    double a[8];
    float f[8];
    int iv[8];
    for (int i = 0; i < 8; ++i) { a[i] = threadIdx.x * 1e-3 + i; f[i] = (float)a[i]; iv[i] = threadIdx.x + i; }
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if (OP == 0) a[i] = fma(a[i], 1.0000001, 0.5);
            if (OP == 1) a[i] = a[i] + 1.0000001;
            if (OP == 2) f[i] = fmaf(f[i], 1.0000001f, 0.5f);
            if (OP == 3) iv[i] = iv[i] * 3 + 7;
            if (OP == 4) a[i] += (double)(iv[i] + it);
        }
    }
    double s = 0;
    for (int i = 0; i < 8; ++i) s += a[i] + f[i] + iv[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
int main() {
    double* o;
    cudaMalloc(&o, 148 * 8 * 1024 * 8);
    const char* names[] = {"DFMA", "DADD", "FFMA", "IMAD", "I2F.F64+DADD"};
    for (int op = 0; op < 5; ++op) {
        auto run = [&](int iters) {
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0);
            cudaEventCreate(&e1);
            cudaEventRecord(e0);
            if (op == 0) k<0><<<148 * 4, 512>>>(o, iters);
            if (op == 1) k<1><<<148 * 4, 512>>>(o, iters);
            if (op == 2) k<2><<<148 * 4, 512>>>(o, iters);
            if (op == 3) k<3><<<148 * 4, 512>>>(o, iters);
            if (op == 4) k<4><<<148 * 4, 512>>>(o, iters);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            return ms;
        };
        run(100);
        const int iters = 4000;
        float ms = run(iters);
        double ops = 148.0 * 4 * 512 * iters * 8;
        int clk;
        cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
        printf("%-14s %8.2f Gop/s  = %6.1f ops/clk/SM (at %d MHz)\n", names[op], ops / ms / 1e6, ops / (ms * 1e-3) / 148 / (clk * 1e3), clk / 1000);
    }
    return 0;
}
