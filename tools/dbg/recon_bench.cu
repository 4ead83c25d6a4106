// Isolated cost of the CRT reconstruction arithmetic (8 warps / SM, one CTA per SM): per group of
// 8 elements, 8 moduli pairs -> X, scaled, as in crt_gemm_kernel.  Variants: ldexp vs exponent bits.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
struct C8 { double H[8], L[8], Mh, Ml, invM; int bits; };
template <int V>
__global__ void __launch_bounds__(256, 1) k(const __grid_constant__ C8 c, const int* ecol, double* out, int groups, long long* cyc) {
    uint4 w[8];
    for (int j = 0; j < 8; ++j) w[j] = make_uint4(threadIdx.x * 7 + j, threadIdx.x * 3 + j, j * 11, j * 13);
    double acc = 0;
    long long t0 = clock64();
    for (int gi = 0; gi < groups; ++gi) {
        double sh[8], sl[8];
#pragma unroll
        for (int v = 0; v < 8; ++v) sh[v] = sl[v] = 0.0;
#pragma unroll
        for (int jj = 0; jj < 8; ++jj) {
            const double Hj = c.H[jj], Lj = c.L[jj];
            const uint32_t wv[4] = {w[jj].x, w[jj].y, w[jj].z, w[jj].w};
#pragma unroll
            for (int v = 0; v < 8; ++v) {
                const uint32_t Rv = (v & 1) ? (wv[v >> 1] >> 16) : (wv[v >> 1] & 0xffffu);
                const double d = __hiloint2double(0x43300000, (int)Rv) - 4503599627370496.0;
                sh[v] = fma(d, Hj, sh[v]);
                sl[v] = fma(d, Lj, sl[v]);
            }
        }
#pragma unroll
        for (int v = 0; v < 8; ++v) {
            const double qm = rint((sh[v] + sl[v]) * c.invM);
            const double X = fma(-qm, c.Mh, sh[v]) + fma(-qm, c.Ml, sl[v]);
            const int e = __ldg(ecol + ((gi * 8 + v) & 255)) - c.bits;
            double s;
            if (V == 0) s = ldexp(1.0, e);
            else s = __hiloint2double((e + 1023) << 20, 0);
            acc += X * 1.5 * s;
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) w[j].x += 1;
    }
    long long t1 = clock64();
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}
int main() {
    C8 c;
    for (int j = 0; j < 8; ++j) { c.H[j] = 1e30 * (j + 1); c.L[j] = 1e20 * (j + 3); }
    c.Mh = 5e37; c.Ml = 1e24; c.invM = 1.0 / 5e37; c.bits = 56;
    int* ec; double* o; long long* cy;
    cudaMalloc(&ec, 256 * 4); cudaMemset(ec, 0, 256 * 4);
    cudaMalloc(&o, 148 * 256 * 8); cudaMalloc(&cy, 8);
    for (int V = 0; V < 2; ++V) {
        const int groups = 2000;
        for (int rep = 0; rep < 2; ++rep) {
            if (V == 0) k<0><<<148, 256>>>(c, ec, o, groups, cy); else k<1><<<148, 256>>>(c, ec, o, groups, cy);
            cudaDeviceSynchronize();
        }
        long long h; cudaMemcpy(&h, cy, 8, cudaMemcpyDeviceToHost);
        printf("variant %d (%s): %.0f cycles per group (8 warps each doing 8 elements)\n", V, V ? "exp bits" : "ldexp", (double)h / groups);
    }
    return 0;
}
