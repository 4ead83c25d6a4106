// Kernel-level test hooks (include/mpgeo_test.h).  Not on the hot path.
#include "../../include/mpgeo_test.h"
#include <vector>

#include "kernels.h"
#include "tc_gemm.h"
#include "ozaki.h"

using namespace mpgeo;

extern "C" {

mp_status mp_test_bessel_k(double nu, const double* d_x, double* d_out, int n) {
    if (bessel_k_launch(nu, d_x, d_out, n, 0) != cudaSuccess) return MP_ERR_CUDA;
    return cudaDeviceSynchronize() == cudaSuccess ? MP_OK : MP_ERR_CUDA;
}

mp_status mp_test_dgemm(const double* d_A, const double* d_B, void* d_C, int M, int N, int K, int lda, int ldb,
                        int ldc, int lower, double alpha, double beta, int round, int c_f32) {
    GemmJob j{d_A, d_B, d_C};
    GemmJob* dj = nullptr;
    if (cudaMalloc(&dj, sizeof j) != cudaSuccess) return MP_ERR_CUDA;
    cudaMemcpy(dj, &j, sizeof j, cudaMemcpyHostToDevice);
    DgemmArgs a{};
    a.jobs = dj;
    a.M = M;
    a.N = N;
    a.K = K;
    a.lda = lda;
    a.ldb = ldb;
    a.ldc = ldc;
    a.lower = lower;
    a.alpha = alpha;
    a.beta = beta;
    cudaError_t e = dgemm_nt_launch(a, 1, round, c_f32 != 0, 0);
    cudaError_t e2 = cudaDeviceSynchronize();
    cudaFree(dj);
    if (e == cudaErrorInvalidValue) return MP_ERR_ARG;
    return (e == cudaSuccess && e2 == cudaSuccess) ? MP_OK : MP_ERR_CUDA;
}

mp_status mp_test_tc_gemm(int kind, const void* d_panel, const void* d_panel_lo, float* d_C, int nb, int nt, int m,
                          int n) {
    if (!tc_gemm_available()) return MP_ERR_UNSUPPORTED;
    TcJob j{m, n, d_C};
    TcJob* dj = nullptr;
    if (cudaMalloc(&dj, sizeof j) != cudaSuccess) return MP_ERR_CUDA;
    cudaMemcpy(dj, &j, sizeof j, cudaMemcpyHostToDevice);
    TcArgs a{};
    a.jobs = dj;
    a.nb = nb;
    a.nt = nt;
    a.cbase = d_C;
    a.crows = (uint64_t)nb;
    cudaError_t e;
    if (kind == 1) {
        a.hi = (const float*)d_panel;
        a.lo = (const float*)d_panel_lo;
        e = tc_gemm_tf32x3_launch(a, 1, 0);
    } else {
        a.p16 = (const __half*)d_panel;
        e = tc_gemm_f16_launch(a, 1, 0);
    }
    cudaError_t e2 = cudaDeviceSynchronize();
    cudaFree(dj);
    return (e == cudaSuccess && e2 == cudaSuccess) ? MP_OK : MP_ERR_CUDA;
}

int mp_tc_available(void) { return tc_gemm_available() ? 1 : 0; }

mp_status mp_test_ozaki_gemm(const double* d_panel, double* d_C, int nb, int nt, int m, int n, int S, int lower) {
    if (!ozaki_available()) return MP_ERR_UNSUPPORTED;
    const int64_t plane = (int64_t)nt * nb * nb;
    int8_t* sl = nullptr;
    int* ex = nullptr;
    OzSplitItem* it = nullptr;
    OzJob* dj = nullptr;
    if (cudaMalloc(&sl, plane * 8) || cudaMalloc(&ex, sizeof(int) * nt * nb) ||
        cudaMalloc(&it, sizeof(OzSplitItem) * nt) || cudaMalloc(&dj, sizeof(OzJob)))
        return MP_ERR_CUDA;
    std::vector<OzSplitItem> h(nt);
    for (int t = 0; t < nt; ++t)
        h[t] = OzSplitItem{d_panel + (size_t)t * nb * nb, sl + (size_t)t * nb * nb, ex + (size_t)t * nb, plane};
    cudaMemcpy(it, h.data(), sizeof(OzSplitItem) * nt, cudaMemcpyHostToDevice);
    OzJob j{m, n, d_C};
    cudaMemcpy(dj, &j, sizeof j, cudaMemcpyHostToDevice);
    cudaError_t e = ozaki_split_launch(it, nt, nb, 8, 0);  // the cache always holds 8 planes
    OzArgs a{dj, sl, ex, plane, nb, nt, S, lower, S == 4 ? 1 : 0};  // S = 4: FP32 class, C is float
    if (e == cudaSuccess) e = ozaki_gemm_launch(a, 1, 0);
    cudaError_t e2 = cudaDeviceSynchronize();
    cudaFree(sl);
    cudaFree(ex);
    cudaFree(it);
    cudaFree(dj);
    return (e == cudaSuccess && e2 == cudaSuccess) ? MP_OK : MP_ERR_CUDA;
}

}  // extern "C"
