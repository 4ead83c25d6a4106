// Probe: does cp.reduce.async.bulk.tensor .add work on a FLOAT64 tensor map (sm_100a)?
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdio.h>
#include <vector>
__global__ void k(const __grid_constant__ CUtensorMap map) {
    __shared__ __align__(1024) double buf[32 * 16];
    for (int i = threadIdx.x; i < 32 * 16; i += blockDim.x) buf[i] = 1.0 + i * 0.25;  // row-major 32 x 16, no swizzle
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t s = (uint32_t)__cvta_generic_to_shared(buf);
        asm volatile("cp.reduce.async.bulk.tensor.2d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3}], [%1];" ::"l"(&map),
                     "r"(s), "r"(16), "r"(8)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
}
int main() {
    const int R = 64, Cc = 64;
    std::vector<double> h(R * Cc, 100.0);
    double* d;
    cudaMalloc(&d, R * Cc * 8);
    cudaMemcpy(d, h.data(), R * Cc * 8, cudaMemcpyHostToDevice);
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
    auto enc = (PFN_cuTensorMapEncodeTiled_v12000)f;
    CUtensorMap m;
    cuuint64_t dims[2] = {Cc, R}, strides[1] = {Cc * 8};
    cuuint32_t box[2] = {16, 32}, es[2] = {1, 1};
    CUresult cr = enc(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, d, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode %d\n", (int)cr);
    k<<<1, 128>>>(m);
    cudaError_t e = cudaDeviceSynchronize();
    printf("kernel %s\n", cudaGetErrorString(e));
    cudaMemcpy(h.data(), d, R * Cc * 8, cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int r = 0; r < R; ++r)
        for (int c = 0; c < Cc; ++c) {
            double exp = 100.0;
            if (r >= 8 && r < 40 && c >= 16 && c < 32) exp += 1.0 + ((r - 8) * 16 + (c - 16)) * 0.25;
            if (h[r * Cc + c] != exp) ++bad;
        }
    printf("bad %d sample %g %g\n", bad, h[8 * Cc + 16], h[9 * Cc + 17]);
    return 0;
}
