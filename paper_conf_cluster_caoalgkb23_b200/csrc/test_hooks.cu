// Kernel-level test hooks (include/mpgeo_test.h).  Not on the hot path.
#include "../../include/mpgeo_test.h"
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <algorithm>
#include <vector>

#include "kernels.h"
#include "tc_gemm.h"
#include "crt.h"

using namespace mpgeo;

namespace mpgeo {
template <int NP>
static void recon_rows(const CrtConst& c, const uint32_t* R, const int* e0, int n, int neg, double* out) {
    for (int i = 0; i < n; ++i) {
        uint32_t r[NP];
        for (int j = 0; j < NP; ++j) r[j] = R[(size_t)i * NP + j];
        const uint64_t b = crt_recon_bits<NP>(r, c, e0[i], (uint32_t)neg);
        memcpy(out + i, &b, 8);
    }
}

}  // namespace mpgeo

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
    if (kind != 1) return MP_ERR_ARG;  // 3xTF32 only; the FP16 kinds take an FP64 panel (mp_test_tc_gemm_split)
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
    a.hi = (const float*)d_panel;
    a.lo = (const float*)d_panel_lo;
    cudaError_t e = tc_gemm_tf32x3_launch(a, 1, 0);
    cudaError_t e2 = cudaDeviceSynchronize();
    cudaFree(dj);
    return (e == cudaSuccess && e2 == cudaSuccess) ? MP_OK : MP_ERR_CUDA;
}

mp_status mp_test_tc_gemm_split(int kind, const double* d_panel, float* d_C, int nb, int nt, int m, int n,
                                int persistent) {
    if (!tc_gemm_available()) return MP_ERR_UNSUPPORTED;
    if (kind != 0 && kind != 2 && kind != 3) return MP_ERR_ARG;  // 3: pure FP16 (F16 accumulation, hs planes)
    const size_t elems = (size_t)nt * nb * nb;
    __half *hi = nullptr, *lo = nullptr;
    int* ex = nullptr;
    TcJob j{m, n, d_C};
    TcJob* dj = nullptr;
    Split16Item* di = nullptr;
    std::vector<Split16Item> items;
    cudaError_t e = cudaMalloc(&hi, elems * 2);
    if (e == cudaSuccess) e = cudaMalloc(&lo, elems * 2);
    if (e == cudaSuccess) e = cudaMalloc(&ex, (size_t)nt * nb * sizeof(int));
    if (e == cudaSuccess) e = cudaMalloc(&dj, sizeof j);
    if (e == cudaSuccess) e = cudaMalloc(&di, nt * sizeof(Split16Item));
    if (e == cudaSuccess) {
        for (int t = 0; t < nt; ++t)  // the FP16 class derives hi only (lo stays untouched)
            items.push_back({d_panel + (size_t)t * nb * nb, kind == 3 ? nullptr : hi + (size_t)t * nb * nb,
                             kind == 2 ? lo + (size_t)t * nb * nb : nullptr, ex + (size_t)t * nb,
                             kind == 3 ? hi + (size_t)t * nb * nb : nullptr});
        cudaMemcpy(dj, &j, sizeof j, cudaMemcpyHostToDevice);
        cudaMemcpy(di, items.data(), nt * sizeof(Split16Item), cudaMemcpyHostToDevice);
        e = split16_launch(di, nt, nb, 0);
    }
    if (e == cudaSuccess) {
        TcArgs a{};
        a.jobs = dj;
        a.nb = nb;
        a.nt = nt;
        a.h16hi = hi;
        a.h16lo = lo;
        a.e16 = ex;
        a.cbase = d_C;
        a.crows = (uint64_t)nb;
        a.persistent = persistent;
        e = kind == 2 ? tc_gemm_f16x3_launch(a, 1, 0) : kind == 3 ? tc_gemm_f16h_launch(a, 1, 0) : tc_gemm_f16_launch(a, 1, 0);
    }
    cudaError_t e2 = cudaDeviceSynchronize();
    cudaFree(hi);
    cudaFree(lo);
    cudaFree(ex);
    cudaFree(dj);
    cudaFree(di);
    return (e == cudaSuccess && e2 == cudaSuccess) ? MP_OK : MP_ERR_CUDA;
}

int mp_tc_available(void) { return tc_gemm_available() ? 1 : 0; }

mp_status mp_test_crt_gemm(const double* d_panel, double* d_C, int nb, int nt, int m, int n, int nmod, int lower,
                           int store) {
    if (!crt_available()) return MP_ERR_UNSUPPORTED;
    CrtConst c;
    if (!crt_constants(nmod, nb, &c)) return MP_ERR_ARG;
    const int64_t plane = (int64_t)nt * nb * nb;
    const int slots = crt_scratch_slots();
    int8_t* pl = nullptr;
    int* ex = nullptr;
    CrtSplitItem* it = nullptr;
    CrtJob* dj = nullptr;
    uint8_t* scr = nullptr;
    int* flags = nullptr;
    if (cudaMalloc(&pl, plane * nmod) || cudaMalloc(&ex, sizeof(int) * nt * nb) ||
        cudaMalloc(&it, sizeof(CrtSplitItem) * nt) || cudaMalloc(&dj, sizeof(CrtJob)) ||
        cudaMalloc(&scr, (size_t)slots * CRT_SLOT_BYTES) || cudaMalloc(&flags, sizeof(int) * (slots + 2)))
        return MP_ERR_CUDA;
    cudaMemset(flags, 0, sizeof(int) * (slots + 2));  // slot flags + the tile counter and phase
    std::vector<CrtSplitItem> h(nt);
    for (int t = 0; t < nt; ++t)
        h[t] = CrtSplitItem{d_panel + (size_t)t * nb * nb, pl + (size_t)t * nb * nb, ex + (size_t)t * nb, plane};
    cudaMemcpy(it, h.data(), sizeof(CrtSplitItem) * nt, cudaMemcpyHostToDevice);
    CrtJob j{m, n, d_C};
    cudaMemcpy(dj, &j, sizeof j, cudaMemcpyHostToDevice);
    cudaError_t e = crt_split_launch(it, nt, nb, c, 0);
    CrtArgs a{};
    a.jobs = dj;
    a.planes = pl;
    a.exps = ex;
    a.plane_stride = plane;
    a.nb = nb;
    a.nt = nt;
    a.lower = lower;
    a.scratch = scr;
    a.slot_flags = flags;
    a.c = c;
    a.cbase = d_C;
    a.crows = (uint64_t)nb;
    a.store = store;
    a.counter = flags + slots;
    if (e == cudaSuccess) e = crt_gemm_launch(a, 1, 0);
    cudaError_t e2 = cudaDeviceSynchronize();
    cudaFree(pl);
    cudaFree(ex);
    cudaFree(it);
    cudaFree(dj);
    cudaFree(scr);
    cudaFree(flags);
    if (e == cudaErrorInvalidValue) return MP_ERR_ARG;
    return (e == cudaSuccess && e2 == cudaSuccess) ? MP_OK : MP_ERR_CUDA;
}

/* Isolated timing of the CRT FP64-class engine on a batched trailing-update-like launch: a
 * deterministic FP64 panel of nt tiles, njobs tile-GEMMs C_j -= P_{m_j} P_{n_j}^T (distinct C tiles)
 * with nmod moduli.  ms[0] = split of the nt panel tiles, ms[1] = one GEMM launch (mean over reps
 * after one warm-up). */
mp_status mp_bench_fp64_engine(int nb, int nt, int njobs, int nmod, int reps, float* ms) {
    const int64_t plane = (int64_t)nt * nb * nb;
    double *P = nullptr, *Cb = nullptr;
    int8_t* pl = nullptr;
    int* ex = nullptr;
    CrtSplitItem* it = nullptr;
    CrtJob* dj = nullptr;
    uint8_t* scr = nullptr;
    int* flags = nullptr;
    const int slots = crt_scratch_slots();
    if (cudaMalloc(&P, plane * 8) || cudaMalloc(&Cb, (size_t)njobs * nb * nb * 8) || cudaMalloc(&pl, plane * nmod) ||
        cudaMalloc(&ex, sizeof(int) * nt * nb) || cudaMalloc(&it, sizeof(CrtSplitItem) * nt) ||
        cudaMalloc(&dj, sizeof(CrtJob) * njobs) || cudaMalloc(&scr, (size_t)slots * CRT_SLOT_BYTES) ||
        cudaMalloc(&flags, sizeof(int) * (slots + 2 * (1 + reps))))
        return MP_ERR_CUDA;
    cudaMemset(flags, 0, sizeof(int) * (slots + 2 * (1 + reps)));  // slot flags + counter pair per launch
    cudaMemset(Cb, 0, (size_t)njobs * nb * nb * 8);
    {   // deterministic non-trivial panel: x = sin(i * 0.37 + j * 0.11) scaled per row
        std::vector<double> h((size_t)nb * nb);
        for (int t = 0; t < nt; ++t) {
            for (int i = 0; i < nb; ++i)
                for (int j = 0; j < nb; ++j) h[(size_t)i * nb + j] = sin(0.37 * (i + t * nb) + 0.11 * j) * (1.0 + (i % 7));
            cudaMemcpy(P + (size_t)t * nb * nb, h.data(), h.size() * 8, cudaMemcpyHostToDevice);
        }
    }
    std::vector<CrtJob> jobs(njobs);
    for (int j = 0; j < njobs; ++j) jobs[j] = CrtJob{j % nt, (j / nt + j + 1) % nt, Cb + (size_t)j * nb * nb};
    cudaMemcpy(dj, jobs.data(), sizeof(CrtJob) * njobs, cudaMemcpyHostToDevice);
    CrtConst c;
    if (!crt_constants(nmod, nb, &c)) return MP_ERR_ARG;
    std::vector<CrtSplitItem> hs(nt);
    for (int t = 0; t < nt; ++t) hs[t] = CrtSplitItem{P + (size_t)t * nb * nb, pl + (size_t)t * nb * nb, ex + (size_t)t * nb, plane};
    cudaMemcpy(it, hs.data(), sizeof(CrtSplitItem) * nt, cudaMemcpyHostToDevice);
    int launch_no = 0;
    auto gemm = [&]() {
        CrtArgs a{};
        a.jobs = dj;
        a.planes = pl;
        a.exps = ex;
        a.plane_stride = plane;
        a.nb = nb;
        a.nt = nt;
        a.scratch = scr;
        a.slot_flags = flags;
        a.c = c;
        a.cbase = Cb;
        a.crows = (uint64_t)njobs * nb;
        a.counter = flags + slots + 2 * std::min(launch_no++, reps);
        return crt_gemm_launch(a, njobs, 0);
    };
    cudaEvent_t e0, e1, e2;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventCreate(&e2);
    cudaError_t e = crt_split_launch(it, nt, nb, c, 0);
    if (e == cudaSuccess) e = gemm();
    cudaDeviceSynchronize();
    cudaEventRecord(e0, 0);
    for (int r = 0; r < reps && e == cudaSuccess; ++r) e = crt_split_launch(it, nt, nb, c, 0);
    cudaEventRecord(e1, 0);
    for (int r = 0; r < reps && e == cudaSuccess; ++r) e = gemm();
    cudaEventRecord(e2, 0);
    cudaError_t es = cudaEventSynchronize(e2);
    float a = 0, b = 0;
    cudaEventElapsedTime(&a, e0, e1);
    cudaEventElapsedTime(&b, e1, e2);
    ms[0] = a / reps;
    ms[1] = b / reps;
    cudaFree(P);
    cudaFree(Cb);
    cudaFree(pl);
    cudaFree(ex);
    cudaFree(it);
    cudaFree(dj);
    cudaFree(scr);
    cudaFree(flags);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaEventDestroy(e2);
    return (e == cudaSuccess && es == cudaSuccess) ? MP_OK : MP_ERR_CUDA;
}

mp_status mp_test_crt_recon(int nmod, int K, const uint32_t* R, const int* e0, int n, int neg, double* out) {
    CrtConst c;
    if (!crt_constants(nmod, K, &c)) return MP_ERR_ARG;
    if (nmod == 16) mpgeo::recon_rows<8>(c, R, e0, n, neg, out);
    else if (nmod == 14) mpgeo::recon_rows<7>(c, R, e0, n, neg, out);
    else if (nmod == 8) mpgeo::recon_rows<4>(c, R, e0, n, neg, out);
    else return MP_ERR_ARG;
    return MP_OK;
}

/* Host constants of the CRT engine (pinned on CPU against big-integer arithmetic). */
mp_status mp_test_crt_constants(int nmod, int K, int* bits, int* moduli, double* H, double* L, double* Mhl) {
    CrtConst c;
    if (!crt_constants(nmod, K, &c)) return MP_ERR_ARG;
    *bits = c.bits;
    for (int t = 0; t < nmod; ++t) moduli[t] = c.p[t];
    for (int j = 0; j < nmod / 2; ++j) {
        H[j] = c.H[j];
        L[j] = c.L[j];
    }
    Mhl[0] = c.Mh;
    Mhl[1] = c.Ml;
    return MP_OK;
}

}  // extern "C"
