// DFMA throughput with few warps (8 per SM) and 16 independent chains per thread, like the CRT
// reconstruction; also the dependent-chain latency.
#include <cstdio>
#include <cuda_runtime.h>
template <int CH>
__global__ void k(double* out, int iters, long long* cyc) {
    double a[CH];
    for (int i = 0; i < CH; ++i) a[i] = threadIdx.x * 1e-3 + i;
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < CH; ++i) a[i] = fma(a[i], 1.0000001, 0.5);
    }
    long long t1 = clock64();
    double s = 0;
    for (int i = 0; i < CH; ++i) s += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}
int main() {
    double* o;
    long long* c;
    cudaMalloc(&o, 148 * 1024 * 8);
    cudaMalloc(&c, 8);
    for (int warps : {1, 2, 4, 8, 16}) {
        for (int ch : {1, 16}) {
            const int iters = 2000;
            if (ch == 1) k<1><<<148, warps * 32>>>(o, iters, c); else k<16><<<148, warps * 32>>>(o, iters, c);
            cudaDeviceSynchronize();
            if (ch == 1) k<1><<<148, warps * 32>>>(o, iters, c); else k<16><<<148, warps * 32>>>(o, iters, c);
            long long h;
            cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
            const double per = (double)h / iters;  // cycles per iteration (ch DFMAs per thread)
            printf("warps/SM %2d chains %2d: %.1f cycles/iter -> %.1f DFMA/clk/SM (latency-bound %s)\n", warps, ch, per,
                   warps * 32.0 * ch / per, ch == 1 ? "yes" : "?");
        }
    }
    return 0;
}
