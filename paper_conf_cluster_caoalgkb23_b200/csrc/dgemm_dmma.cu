// K5 — batched FP64 tile GEMM on the DMMA tensor-core path of sm_100a.
//
//   C  = beta*C + alpha * A * B^T        (alpha = -1, beta = 1: trailing update;
//                                         alpha = +1, beta = 0: in-place TRSM block)
// for a batch of jobs of identical shape M x N x K, all operands row-major with the
// contraction index contiguous ("NT": both A and B are K-major).  This is the
// DSYRK / GEMM of Algorithm 1 (§V) for FP64-class tiles, and the
// building block of the blocked DPOTRF and TRSM.
//
// There is no tcgen05 kind::f64 on sm_100a; FP64 tensor-core math is the warp-level
// mma.sync.m16n8k4.f64 (SASS DMMA).  Design:
//   * CTA tile 128 x 128 x 32, 256 threads = 8 warps (2 x 4), warp tile 64 x 32,
//     16 DMMA m16n8k4 per k4-step held in 64 FP64 accumulators per thread;
//   * 3-stage cp.async (LDGSTS) pipeline (192 KB), 16-byte chunks, zero-fill past M / N;
//   * shared tiles are [128][32] doubles with the 16-byte chunk index XOR-swizzled
//     by 2*(row & 3) (see dg_swz): every fragment load is two 128-byte wavefronts, the
//     minimum for 256 bytes; fragments are double-buffered in registers;
//   * optional operand rounding to FP32 / FP16 (the FP32- and FP16-class GEMM of
//     P:146 evaluated as FP64 arithmetic on rounded operands) and an FP32 C tile.
// Jobs of one launch are laid out job-major so the CTAs resident at one time share
// the job's operand tiles in L2.
#include "common.cuh"
#include "kernels.h"

namespace mpgeo {

constexpr int DG_BM = 128, DG_BN = 128, DG_BK = 32, DG_STAGES = 3, DG_THREADS = 256;
constexpr int DG_CH = DG_BK / 2;  // 16-byte chunks per smem row
constexpr int DG_STAGE_ELEMS = (DG_BM + DG_BN) * DG_BK;  // doubles per stage
constexpr int DG_SMEM = DG_STAGES * DG_STAGE_ELEMS * 8;  // 192 KB

// 16-byte chunk c of row r lives at chunk c ^ ((r & 3) << 1).  A DMMA fragment load reads 8 rows
// (g = lane / 4) x 2 chunks; 64-bit shared loads are served per half-warp (g = 0..3 and 4..7), and
// within a half-warp the 8 (row, chunk) pairs land on 8 distinct 16-byte bank groups: 2 wavefronts
// per warp load, the minimum for 256 bytes.
__device__ __forceinline__ int dg_swz(int row, int col) {
    return row * DG_BK + ((((col >> 1) ^ ((row & 3) << 1))) << 1) + (col & 1);
}

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, bool valid) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    int bytes = valid ? 16 : 0;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(bytes));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

__device__ __forceinline__ void dmma_16x8x4(double (&d)[4], const double (&a)[2], double b) {
    asm volatile(
        "mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};\n"
        : "+d"(d[0]), "+d"(d[1]), "+d"(d[2]), "+d"(d[3])
        : "d"(a[0]), "d"(a[1]), "d"(b));
}

template <int ROUND>
__device__ __forceinline__ double ld_op(const double* p) {
    double v = *p;
    if (ROUND == P32) v = (double)__double2float_rn(v);
    if (ROUND == P16) v = (double)__half2float(__double2half(v));
    return v;
}

template <int ROUND, bool CF32>
__global__ void __launch_bounds__(DG_THREADS, 1) dgemm_nt_kernel(DgemmArgs p) {
    extern __shared__ __align__(128) double smem[];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = lane >> 2, t = lane & 3;
    const int wm = warp >> 2, wn = warp & 3;

    // ---- which job / CTA tile
    const long long bid = blockIdx.x;
    const int job = (int)(bid / p.tiles_per_job);
    int tt = (int)(bid - (long long)job * p.tiles_per_job);
    int bi, bj;
    if (p.lower) {
        bi = (int)((sqrt(8.0 * tt + 1.0) - 1.0) * 0.5);
        while ((bi + 1) * (bi + 2) / 2 <= tt) ++bi;
        while (bi * (bi + 1) / 2 > tt) --bi;
        bj = tt - bi * (bi + 1) / 2;
    } else {
        bi = tt / p.tiles_n;
        bj = tt - bi * p.tiles_n;
    }
    const GemmJob jb = p.jobs[job];
    const double* __restrict__ A = (const double*)jb.A;
    const double* __restrict__ B = (const double*)jb.B;
    const int bm = bi * DG_BM, bn = bj * DG_BN;

    // ---- loader: BM x BK/2 16-byte chunks per operand per stage (zero-fill past M, N, K)
    auto load_stage = [&](int stage, int kt) {
        double* As = smem + stage * DG_STAGE_ELEMS;
        double* Bs = As + DG_BM * DG_BK;
        const int k0 = kt * DG_BK;
#pragma unroll
        for (int i = 0; i < DG_BM * DG_CH / DG_THREADS; ++i) {
            const int c = tid + i * DG_THREADS;
            const int row = c / DG_CH, ch = c % DG_CH;
            const int ra = bm + row, rb = bn + row;
            const bool kv = k0 + ch * 2 < p.K;  // K is even: a chunk is all-in or all-out
            const bool va = ra < p.M && kv, vb = rb < p.N && kv;
            const double* ga = va ? A + (size_t)ra * p.lda + k0 + ch * 2 : A;
            const double* gb = vb ? B + (size_t)rb * p.ldb + k0 + ch * 2 : B;
            const int sw = (ch ^ ((row & 3) << 1)) << 1;
            cp_async16(As + row * DG_BK + sw, ga, va);
            cp_async16(Bs + row * DG_BK + sw, gb, vb);
        }
    };

    double acc[4][4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
            for (int r = 0; r < 4; ++r) acc[i][j][r] = 0.0;

    const int KT = (p.K + DG_BK - 1) / DG_BK;  // zero-filled past K
#pragma unroll
    for (int s = 0; s < DG_STAGES - 1; ++s) {
        if (s < KT) load_stage(s, s);
        cp_async_commit();
    }

    for (int kt = 0; kt < KT; ++kt) {
        cp_async_wait<DG_STAGES - 2>();
        __syncthreads();
        {
            const int nk = kt + DG_STAGES - 1;
            if (nk < KT) load_stage(nk % DG_STAGES, nk);
            cp_async_commit();
        }
        const double* As = smem + (kt % DG_STAGES) * DG_STAGE_ELEMS;
        const double* Bs = As + DG_BM * DG_BK;
        // fragments double-buffered across k4-steps: loads of step ks+1 overlap the DMMAs of ks
        double a[2][4][2], b[2][4];
        auto load_frag = [&](int buf, int ks) {
            const int kk = ks * 4 + t;
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int r = wm * 64 + i * 16 + g;
                a[buf][i][0] = ld_op<ROUND>(As + dg_swz(r, kk));
                a[buf][i][1] = ld_op<ROUND>(As + dg_swz(r + 8, kk));
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) b[buf][j] = ld_op<ROUND>(Bs + dg_swz(wn * 32 + j * 8 + g, kk));
        };
        load_frag(0, 0);
#pragma unroll
        for (int ks = 0; ks < DG_BK / 4; ++ks) {
            if (ks + 1 < DG_BK / 4) load_frag((ks + 1) & 1, ks + 1);
#pragma unroll
            for (int i = 0; i < 4; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) dmma_16x8x4(acc[i][j], a[ks & 1][i], b[ks & 1][j]);
        }
    }
    cp_async_wait<0>();

    // ---- epilogue: C = beta*C + alpha*acc, two adjacent columns per fragment row
    const double alpha = p.alpha;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int r = bm + wm * 64 + i * 16 + g + h * 8;
            if (r >= p.M) continue;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int c = bn + wn * 32 + j * 8 + 2 * t;
                if (c >= p.N) continue;
                const double v0 = alpha * acc[i][j][2 * h], v1 = alpha * acc[i][j][2 * h + 1];
                if (CF32) {
                    float2* cp = (float2*)((float*)jb.C + (size_t)r * p.ldc + c);
                    float2 o;
                    if (p.beta != 0.0) {
                        const float2 cv = *cp;
                        o.x = __double2float_rn((double)cv.x + v0);
                        o.y = __double2float_rn((double)cv.y + v1);
                    } else {
                        o.x = __double2float_rn(v0);
                        o.y = __double2float_rn(v1);
                    }
                    *cp = o;
                } else {
                    double2* cp = (double2*)((double*)jb.C + (size_t)r * p.ldc + c);
                    double2 o;
                    if (p.beta != 0.0) {
                        const double2 cv = *cp;
                        o.x = cv.x + v0;
                        o.y = cv.y + v1;
                    } else {
                        o.x = v0;
                        o.y = v1;
                    }
                    *cp = o;
                }
            }
        }
    }
}

template <int ROUND, bool CF32>
static cudaError_t launch_one(const DgemmArgs& a, long long grid, cudaStream_t s) {
    static bool attr_done = false;
    if (!attr_done) {
        cudaError_t e = cudaFuncSetAttribute(dgemm_nt_kernel<ROUND, CF32>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, DG_SMEM);
        if (e != cudaSuccess) return e;
        attr_done = true;
    }
    dgemm_nt_kernel<ROUND, CF32><<<(unsigned)grid, DG_THREADS, DG_SMEM, s>>>(a);
    return cudaGetLastError();
}

cudaError_t dgemm_nt_launch(DgemmArgs a, int njobs, int round_ops, bool c_f32, cudaStream_t s) {
    if (njobs <= 0 || a.M <= 0 || a.N <= 0 || a.K <= 0) return cudaSuccess;
    if (a.K % 16) return cudaErrorInvalidValue;
    a.tiles_m = (a.M + DG_BM - 1) / DG_BM;
    a.tiles_n = (a.N + DG_BN - 1) / DG_BN;
    if (a.lower) {
        if (a.tiles_m != a.tiles_n) return cudaErrorInvalidValue;
        a.tiles_per_job = a.tiles_m * (a.tiles_m + 1) / 2;
    } else {
        a.tiles_per_job = a.tiles_m * a.tiles_n;
    }
    const long long grid = (long long)njobs * a.tiles_per_job;
    if (grid > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    if (c_f32) {
        if (round_ops == P32) return launch_one<P32, true>(a, grid, s);
        if (round_ops == P16) return launch_one<P16, true>(a, grid, s);
        return launch_one<P64, true>(a, grid, s);
    }
    if (round_ops == P32) return launch_one<P32, false>(a, grid, s);
    if (round_ops == P16) return launch_one<P16, false>(a, grid, s);
    return launch_one<P64, false>(a, grid, s);
}

}  // namespace mpgeo
