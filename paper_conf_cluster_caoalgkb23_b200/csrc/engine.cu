// Host engine and C ABI of libmpgeo (include/mpgeo.h).
//
// The tile DAG of Algorithm 1 is executed as a static per-panel schedule on the
// handle's CUDA stream: for panel k
//   1. DPOTRF(k,k): blocked by 128 columns — diagonal block Cholesky + inverse (1 CTA), the
//      block column as an in-place DMMA GEMM with the inverse, the trailing block SYRK;
//   2. L~_kk = L_kk rounded to comm(k,k) (what the TRSMs receive, Alg. 2) + block inverses;
//   3. panel in: the column's tiles (m,k), m > k, up-converted into the FP64 panel buffer;
//   4. TRSM(m,k): FP64-class tiles by blocked DMMA substitution, FP32/FP16-class tiles as the
//      FP32-class product A_mk W^T with W = L~_kk^-1 (reading C12');
//   5. panel out (K2): write back in storage precision, round to comm(m,k); multi-rank: publish /
//      pull the panel tiles in comm precision;
//   5e. operand formats (K2), once per panel and GPU: row-scaled FP16 hi/lo, TF32 pairs, CRT
//      residue planes — single-buffered, produced on the update stream right before the update;
//   6. trailing update: DSYRK(m,k) + GEMM(m,n,k) grouped by the kernel precision of the
//      output tile: FP64 class (CRT INT8 / DMMA), FP32 class, FP16 class.
// Everything for one call is planned on the host first (job arrays for the batched kernels),
// uploaded once into the control arena of the workspace, then enqueued.
#include <unistd.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <functional>
#include <string>
#include <vector>

#include "../../include/mpgeo.h"
#include "kernels.h"
#include "tc_gemm.h"
#include "dist.h"
#include "crt.h"

using namespace mpgeo;

// ------------------------------------------------------------------ objects
struct ProfRec {
    cudaEvent_t e0, e1;
    int cls;
    double flops;
    int stream;
};
struct mp_handle {
    int device = 0, rank = 0, nranks = 1, P = 1, Q = 1;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    std::string err;
    int64_t launches = 0;
    int* d_info = nullptr;
    cudaEvent_t ev[8] = {};
    bool broken = false;
    mp_config cfg{};       // engines and schedule switches (mp_init_config)
    uint8_t id[128] = {};  // communicator id (mp_get_unique_id); all zero = none
    bool has_id = false;
    cudaStream_t pstream = nullptr;
    std::vector<cudaEvent_t> sync_ev;
    // profiling (mp_set_profiling): event pairs per launch, resolved in mp_get_profile
    bool profiling = false;
    unsigned prof_mask = 0;  // classes whose launches get event pairs (mp_set_profiling_mask)
    std::vector<cudaEvent_t> prof_pool;
    size_t prof_free = 0;
    std::vector<ProfRec> prof_pending;
    mp_profile prof = {};
};

// The engines one matrix runs with: the handle's configuration where the tile size allows it
// (the tcgen05 kernels tile nb by 256).  plan_potrf, the workspace layout and mp_matrix_engines all
// read this one predicate.
struct Engines {
    bool crt = false;        // FP64 class: CRT (16 moduli) on INT8 tcgen05; else DMMA
    bool tc16 = false;       // FP16 class: row-scaled FP16 on tcgen05; else DMMA on FP16-rounded operands
    int f32 = MP_F32_DMMA;   // FP32 class engine (mp_fp32_engine)
    bool ctrsm = false;      // FP32/FP16-class TRSM as the CRT-8 product with the inverse factor
    bool h16 = false;        // row-scaled FP16 hi (+ lo) caches exist
    bool s16 = false;        // FP16 storage class for FP16-class tiles (mp_config::fp16_storage)
    bool p64_double = false; // the update reads the FP64 panel buffer (a DMMA class): two panel sets
};
static Engines engines_for(const mp_handle* h, int nb) {
    Engines e;
    const bool tcok = tc_gemm_available() && nb % 256 == 0;
    e.crt = h->cfg.fp64_engine == MP_F64_CRT16 && crt_available() && nb % 256 == 0;
    e.tc16 = h->cfg.fp16_tensor != 0 && tcok;
    e.f32 = (h->cfg.fp32_engine == MP_F32_3XFP16 || h->cfg.fp32_engine == MP_F32_3XTF32) && tcok ? h->cfg.fp32_engine
                                                                                                : MP_F32_DMMA;
    e.ctrsm = e.crt && h->cfg.lowp_trsm_product != 0;
    e.h16 = e.tc16 || e.f32 == MP_F32_3XFP16;
    e.s16 = h->cfg.fp16_storage != 0;
    e.p64_double = h->cfg.lookahead != 0 && (!e.crt || !e.tc16 || e.f32 == MP_F32_DMMA);
    return e;
}

struct Regions {
    size_t total = 0;
    size_t inputs = 0, p64 = 0, h16 = 0, h16s = 0, e16 = 0, phi = 0, plo = 0, oz32 = 0, e32 = 0, ltilde = 0, wbuf = 0,
           wbuf2 = 0, wfac = 0, oz = 0, ozexp = 0, wdiag = 0, mtab = 0, crt = 0, crtflags = 0, crtctr = 0;
    int p64_sets = 1;              // 2 when the update reads the FP64 panel buffer (Engines::p64_double)
    size_t vec_r = 0, vec_y = 0, partials = 0, norms = 0, ctrl = 0, ctrl_bytes = 0;
    std::vector<size_t> tile_off;  // per (m*nt+k), SIZE_MAX if not stored here
    size_t pool = 0;               // start of the tile pool
};

// Peer-memory exchange area of one matrix (multi-GPU only; cudaMalloc'ed by the library so it
// can be exported with cudaIpcGetMemHandle).  Offsets are identical on every rank.
struct Comm {
    char* base = nullptr;
    size_t bytes = 0;
    std::vector<char*> peer;  // base of every rank's area (own = base)
    bool connected = false;
    uint64_t epoch = 0;       // incremented per collective call; stamps = epoch << 24 | step
    size_t hdr = 0, send = 0, pub = 0, done = 0, bar = 0, part = 0, yv = 0, pflag = 0, yflag = 0, norms = 0,
           nflag = 0, scal = 0, sflag = 0, tmp = 0;
};

struct mp_matrix {
    mp_handle* h = nullptr;
    Comm comm;
    int64_t n = 0;
    int nb = 0, nt = 0;
    char* ws = nullptr;
    size_t ws_bytes = 0;
    bool bound = false, generated = false, factored = false;
    int cov = MP_COV_MATERN;
    std::vector<uint8_t> storage, kmap, cmap;
    std::vector<double> sqn;      // tile sums of squares of the last generation pass 1 (NT*NT, all-gathered)
    std::vector<int> tscale;      // FP16 storage class: per-tile exponent t (stored value fp16(x 2^t))
    bool h16h = false;            // the bound map has pure-FP16 (MP_FP16H) tiles: the hs operand planes exist
    int ts(int m, int k) const { return tscale.empty() ? 0 : tscale[(size_t)m * nt + k]; }
    Regions R;
    int owner(int m, int k) const { return (m % h->P) * h->Q + (k % h->Q); }
    bool mine(int m, int k) const { return h->nranks == 1 || owner(m, k) == h->rank; }
    size_t nb2() const { return (size_t)nb * nb; }
    void* tile(int m, int k) const { return ws + R.tile_off[(size_t)m * nt + k]; }
    uint8_t st(int m, int k) const { return storage[(size_t)m * nt + k]; }
    template <class T>
    T* at(size_t off) const { return (T*)(ws + off); }
};

#define FAIL(h, code, ...)                                            \
    do {                                                              \
        char _b[512];                                                 \
        snprintf(_b, sizeof _b, __VA_ARGS__);                         \
        if (h) (h)->err = _b;                                         \
        return code;                                                  \
    } while (0)
#define CK(h, x)                                                                          \
    do {                                                                                  \
        cudaError_t _e = (x);                                                             \
        if (_e != cudaSuccess) {                                                          \
            if (h) (h)->broken = true;                                                    \
            FAIL(h, MP_ERR_CUDA, "%s failed: %s (%s:%d)", #x, cudaGetErrorString(_e), __FILE__, __LINE__); \
        }                                                                                 \
    } while (0)

static size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }
// CRT launches of one factorisation: <= 4 update launches (two parts x SYRK / GEMM) + 1 FP32-class +
// 1 TRSM per panel
static size_t crt_counters(int nt) { return 2 * (8 * (size_t)nt + 64); }
constexpr int MT_PIECES_MAX = 512;
static int ceil_div(int a, int b) { return (a + b - 1) / b; }

// Upper bound of control-arena bytes for one call on an nt x nt tile matrix.
static size_t ctrl_bytes_for(int nt, int nb) {
    const size_t T = nt;
    const size_t nblk = ceil_div(nb, POTRF_IB);
    size_t jobs = T * (T + 1) * (T + 2) / 6 + T + 2 * nblk * T + 2 * nblk * T * T;
    size_t bytes = jobs * sizeof(GemmJob);
    bytes += T * T * sizeof(PanelTile) * 2;
    bytes += T * (T + 1) / 2 * sizeof(GenTile);
    bytes += T * T * sizeof(GemvTile);
    bytes += T * (sizeof(double*) + sizeof(int));
    bytes += T * T * (sizeof(PackItem) + sizeof(PullItem) + 2 * sizeof(WaitItem)) + T * 8 * sizeof(WaitItem);
    bytes += T * T * (sizeof(CrtSplitItem) + sizeof(Split16Item) + sizeof(Tf32Item)) + T * (T + 1) * (T + 2) / 6 * sizeof(CrtJob);
    bytes += 64 * 1024 + 32 * 256;  // alignment slack
    return bytes;
}

// storage == NULL: all FP64 (the worst case); storage == NO_POOL: no tile pool (mp_matrix_attach)
static const uint8_t* const NO_POOL = (const uint8_t*)1;

static Regions layout(const mp_matrix* A, const uint8_t* storage) {
    // Map-independent regions first (their offsets depend only on n, nb, NT and the engines), then
    // the tile pool, whose slots depend on the storage map (re-laid out per evaluation).
    Regions R;
    const int nt = A->nt;
    const size_t nb2 = A->nb2();
    const Engines E = engines_for(A->h, A->nb);
    size_t off = 0;
    auto take = [&](size_t bytes) {
        off = align_up(off, 256);
        const size_t o = off;
        off += bytes;
        return o;
    };
    const size_t nvec = (size_t)nt * A->nb;
    const size_t slots = (size_t)nt * nb2;  // one panel: slot m holds tile (m, k)
    R.inputs = take(3 * nvec * 8);
    R.vec_r = take(nvec * 8);
    R.vec_y = take(nvec * 8);
    const size_t ntl = (size_t)nt * (nt + 1) / 2;
    R.partials = take(std::max(ntl * (A->nb / GEN_ROWS), (size_t)2 * nt + nvec / 4096 + 64) * 8);
    R.norms = take(std::max(ntl, (size_t)nt * 4 + 64) * 8);
    R.ctrl_bytes = ctrl_bytes_for(nt, A->nb);
    R.ctrl = take(R.ctrl_bytes);
    R.ltilde = take(nb2 * 8);
    R.wbuf = take((size_t)POTRF_IB * POTRF_IB * 8);
    R.wbuf2 = take((size_t)ceil_div(A->nb, POTRF_IB) * POTRF_IB * POTRF_IB * 8);
    R.wdiag = take((size_t)nt * ceil_div(A->nb, POTRF_IB) * POTRF_IB * POTRF_IB * 8);  // solve: block inverses
    R.mtab = take((size_t)MT_PIECES_MAX * (MT_DEG + 1) * 8);  // general-nu Matern table
    // FP64 panel buffer: written by panel k+1's POTRF/TRSM (panel stream) while update k runs, so
    // two sets only if update k reads it (a DMMA class); the operand formats below are derived from
    // it after update k and are single-buffered
    R.p64_sets = E.p64_double ? 2 : 1;
    R.p64 = take(R.p64_sets * slots * 8);
    if (E.h16) {  // row-scaled FP16 hi and lo planes + row exponents (3xFP16 FP32 class, FP16 class)
        R.h16 = take(2 * slots * 2);
        R.e16 = take(nvec * 4);
        if (A->h16h) R.h16s = take(slots * 2);  // four-level maps: pure-FP16 operands (split16 hs)
    }
    if (E.f32 == MP_F32_3XTF32) {
        R.phi = take(slots * 4);
        R.plo = take(slots * 4);
    }
    if (E.crt) {  // FP64 class: 16 residue planes + row exponents; per-CTA residue staging slots
        R.oz = take(slots * CRT_NMAX);
        R.ozexp = take(nvec * 4);
        R.crt = take((size_t)crt_scratch_slots() * CRT_SLOT_BYTES);
        R.crtflags = take((size_t)crt_scratch_slots() * sizeof(int));
        R.crtctr = take(crt_counters(nt) * sizeof(int));
    }
    if (E.ctrsm) {  // the TRSM product's operands (8 residue planes, own exponents) and W = L~_kk^-1
        R.oz32 = take(slots * 8);
        R.e32 = take(nvec * 4);
        R.wfac = take(nb2 * 8);
    }
    R.tile_off.assign((size_t)nt * nt, SIZE_MAX);
    R.pool = align_up(off, 256);  // tile pool start (tile offsets from here are whole nb-float rows when 256 | nb)
    if (storage != NO_POOL)
        for (int k = 0; k < nt; ++k)
            for (int m = k; m < nt; ++m)
                if (A->mine(m, k)) {
                    const uint8_t p = storage ? storage[(size_t)m * nt + k] : (uint8_t)MP_FP64;
                    R.tile_off[(size_t)m * nt + k] = take(nb2 * (p == MP_FP64 ? 8 : p == MP_FP32 ? 4 : 2));
                }
    R.total = align_up(off, 256);
    return R;
}

// Control arena: host staging of job / descriptor arrays, uploaded in one copy.
struct Arena {
    std::vector<char> host;
    char* dev_base = nullptr;
    size_t cap = 0;
    template <class T>
    T* push(const T* items, size_t n) {  // returns the device address of the copy
        size_t off = align_up(host.size(), 16);
        host.resize(off + n * sizeof(T));
        if (n) memcpy(host.data() + off, items, n * sizeof(T));
        return (T*)(dev_base + off);
    }
    template <class T>
    T* push(const std::vector<T>& v) { return push(v.data(), v.size()); }
};

// One enqueued kernel: launcher, profiling class (mp_profile) and its algorithmic flops.
struct Op {
    std::function<cudaError_t(cudaStream_t)> fn;
    int cls;
    double flops;
    int stream = 0;  // 0: the handle's stream, 1: the high-priority panel stream (lookahead)
    int kind = 0;    // 0: launch, 1: record event `ev` on `stream`, 2: make `stream` wait for `ev`
    int ev = -1;
    int nlaunch = 1;  // kernels this op launches (for the launch count)
};
static Op op_record(int stream, int ev) { Op o{nullptr, 0, 0}; o.stream = stream; o.kind = 1; o.ev = ev; return o; }
static Op op_wait(int stream, int ev) { Op o{nullptr, 0, 0}; o.stream = stream; o.kind = 2; o.ev = ev; return o; }
enum { C_UPD64 = 0, C_UPD32 = 1, C_UPD16 = 2, C_POTRF = 3, C_TRSM = 4, C_CONV = 5, C_GEN = 6, C_SOLVE = 7 };

static cudaEvent_t prof_event(mp_handle* h) {
    if (h->prof_free < h->prof_pool.size()) return h->prof_pool[h->prof_free++];
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    h->prof_pool.push_back(e);
    h->prof_free++;
    return e;
}

static mp_status run_plan(mp_handle* h, mp_matrix* A, Arena& ar, std::vector<Op>& ops) {
    if (ar.host.size() > A->R.ctrl_bytes)
        FAIL(h, MP_ERR_NOMEM, "control arena overflow (%zu > %zu)", ar.host.size(), A->R.ctrl_bytes);
    if (!ar.host.empty())
        CK(h, cudaMemcpyAsync(ar.dev_base, ar.host.data(), ar.host.size(), cudaMemcpyHostToDevice, h->stream));
    int max_ev = -1;
    for (auto& op : ops) max_ev = std::max(max_ev, op.ev);
    while ((int)h->sync_ev.size() <= max_ev) {
        cudaEvent_t e;
        CK(h, cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        h->sync_ev.push_back(e);
    }
    for (auto& op : ops) {
        cudaStream_t st = op.stream ? h->pstream : h->stream;
        if (op.kind == 1) {
            CK(h, cudaEventRecord(h->sync_ev[op.ev], st));
            continue;
        }
        if (op.kind == 2) {
            CK(h, cudaStreamWaitEvent(st, h->sync_ev[op.ev], 0));
            continue;
        }
        if (h->profiling && ((h->prof_mask >> op.cls) & 1u)) {
            cudaEvent_t e0 = prof_event(h), e1 = prof_event(h);
            CK(h, cudaEventRecord(e0, st));
            CK(h, op.fn(st));
            CK(h, cudaEventRecord(e1, st));
            h->prof_pending.push_back(ProfRec{e0, e1, op.cls, op.flops, op.stream});
        } else {
            CK(h, op.fn(st));
        }
        h->launches += op.nlaunch;
    }
    return MP_OK;
}

// ------------------------------------------------------------------ lifecycle
extern "C" {

const char* mp_version(void) {
    return "mpgeo 0.2 sm_100a (FP64 class: CRT INT8 tcgen05 | DMMA; FP32 class: 3xFP16 | 3xTF32 tcgen05 | DMMA; "
           "FP16 class: row-scaled f16 tcgen05 | DMMA; four-level pure FP16: f16-accumulator tcgen05)";
}

void mp_config_default(mp_config* c) {
    if (!c) return;
    c->fp64_engine = MP_F64_CRT16;
    c->fp32_engine = MP_F32_3XFP16;
    c->fp16_tensor = 1;
    c->lookahead = 1;
    c->reserve_pairs = 6;
    c->lowp_trsm_product = 1;
    c->matern_table = 1;
    c->f16x3_persistent = 0;
    c->crt_phase_lock = 1;
    c->fp16_storage = 0;
}

mp_status mp_get_unique_id(uint8_t id[128]) {
    if (!id) return MP_ERR_ARG;
    memset(id, 0, 128);
    FILE* f = fopen("/dev/urandom", "rb");
    if (!f || fread(id, 1, 32, f) != 32) {
        if (f) fclose(f);
        return MP_ERR_UNSUPPORTED;
    }
    fclose(f);
    const long pid = (long)getpid();
    memcpy(id + 32, &pid, sizeof pid);
    gethostname((char*)id + 48, 79);
    id[127] = 0;
    return MP_OK;
}

mp_status mp_init_config(int device, int rank, int nranks, int P, int Q, const uint8_t* id, void* cuda_stream,
                         const mp_config* cfg, mp_handle** out) {
    if (!out || nranks < 1 || rank < 0 || rank >= nranks || P < 1 || Q < 1 || P * Q != nranks || P > Q)
        return MP_ERR_ARG;
    *out = nullptr;
    if (nranks > MAX_PEERS) return MP_ERR_UNSUPPORTED;
    if (nranks > 1 && !id) return MP_ERR_ARG;  // multi-rank: the communicator id of mp_get_unique_id
    mp_handle* h = new mp_handle();
    h->device = device;
    h->rank = rank;
    h->nranks = nranks;
    h->P = P;
    h->Q = Q;
    mp_config_default(&h->cfg);
    if (cfg) h->cfg = *cfg;
    if (h->cfg.reserve_pairs < 0) h->cfg.reserve_pairs = 0;
    if (id) {
        memcpy(h->id, id, 128);
        h->has_id = true;
    }
    auto fail = [&](mp_status s) {  // release everything created so far
        for (auto& e : h->ev)
            if (e) cudaEventDestroy(e);
        if (h->d_info) cudaFree(h->d_info);
        if (h->pstream) cudaStreamDestroy(h->pstream);
        if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
        delete h;
        return s;
    };
    if (cudaSetDevice(device) != cudaSuccess) return fail(MP_ERR_CUDA);
    if (cuda_stream) {
        h->stream = (cudaStream_t)cuda_stream;
    } else {
        if (cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking) != cudaSuccess) return fail(MP_ERR_CUDA);
        h->own_stream = true;
    }
    {
        int lo = 0, hi = 0;
        cudaDeviceGetStreamPriorityRange(&lo, &hi);
        if (cudaStreamCreateWithPriority(&h->pstream, cudaStreamNonBlocking, hi) != cudaSuccess) return fail(MP_ERR_CUDA);
    }
    if (cudaMalloc(&h->d_info, sizeof(int)) != cudaSuccess) return fail(MP_ERR_CUDA);
    for (auto& e : h->ev)
        if (cudaEventCreate(&e) != cudaSuccess) return fail(MP_ERR_CUDA);
    *out = h;
    return MP_OK;
}

mp_status mp_init(int device, int rank, int nranks, int P, int Q, const uint8_t* id, void* cuda_stream,
                  mp_handle** out) {
    return mp_init_config(device, rank, nranks, P, Q, id, cuda_stream, nullptr, out);
}

mp_status mp_handle_get_config(const mp_handle* h, mp_config* cfg) {
    if (!h || !cfg) return MP_ERR_ARG;
    *cfg = h->cfg;
    return MP_OK;
}

mp_status mp_finalize(mp_handle* h) {
    if (!h) return MP_ERR_ARG;
    cudaSetDevice(h->device);
    if (h->stream) cudaStreamSynchronize(h->stream);
    for (auto& e : h->ev)
        if (e) cudaEventDestroy(e);
    for (auto& e : h->prof_pool)
        if (e) cudaEventDestroy(e);
    for (auto& e : h->sync_ev)
        if (e) cudaEventDestroy(e);
    if (h->pstream) cudaStreamDestroy(h->pstream);
    if (h->d_info) cudaFree(h->d_info);
    if (h->own_stream) cudaStreamDestroy(h->stream);
    delete h;
    return MP_OK;
}

const char* mp_last_error(const mp_handle* h) { return h ? h->err.c_str() : "null handle"; }

mp_status mp_set_profiling_mask(mp_handle* h, unsigned mask) {
    if (!h) return MP_ERR_ARG;
    if (!h->prof_pending.empty()) CK(h, cudaStreamSynchronize(h->stream));
    h->prof_pending.clear();
    h->prof_free = 0;
    h->prof = mp_profile{};
    h->prof_mask = mask & ((1u << MP_PROF_CLASSES) - 1);
    h->profiling = h->prof_mask != 0;
    return MP_OK;
}

mp_status mp_set_profiling(mp_handle* h, int enable) {
    return mp_set_profiling_mask(h, enable ? (1u << MP_PROF_CLASSES) - 1 : 0u);
}

mp_status mp_get_profile(mp_handle* h, mp_profile* out) {
    if (!h || !out) return MP_ERR_ARG;
    CK(h, cudaStreamSynchronize(h->stream));
    // MPGEO_TIMELINE=<path>: append every profiled launch as "class stream start_ms end_ms flops"
    // (relative to the first one) — the schedule of one call, for tuning the lookahead overlap
    if (const char* path = getenv("MPGEO_TIMELINE"))
        if (!h->prof_pending.empty())
            if (FILE* f = fopen(path, "a")) {
                const cudaEvent_t t0 = h->prof_pending.front().e0;
                for (const ProfRec& r : h->prof_pending) {
                    float a = 0.f, b = 0.f;
                    cudaEventElapsedTime(&a, t0, r.e0);
                    cudaEventElapsedTime(&b, t0, r.e1);
                    fprintf(f, "%d %d %.4f %.4f %.6g\n", r.cls, r.stream, a, b, r.flops);
                }
                fprintf(f, "--\n");
                fclose(f);
            }
    for (const ProfRec& r : h->prof_pending) {
        float ms = 0.f;
        CK(h, cudaEventElapsedTime(&ms, r.e0, r.e1));
        h->prof.ms[r.cls] += ms;
        h->prof.flops[r.cls] += r.flops;
        h->prof.launches[r.cls] += 1;
    }
    h->prof_pending.clear();
    h->prof_free = 0;
    *out = h->prof;
    return MP_OK;
}
int64_t mp_launch_count(const mp_handle* h) { return h ? h->launches : 0; }

mp_status mp_matrix_engines(const mp_matrix* A, int* fp64, int* fp32, int* fp16, int* lowp_trsm) {
    if (!A) return MP_ERR_ARG;
    const Engines e = engines_for(A->h, A->nb);
    if (fp64) *fp64 = e.crt ? MP_F64_CRT16 : MP_F64_DMMA;
    if (fp32) *fp32 = e.f32;
    if (fp16) *fp16 = e.tc16 ? 1 : 0;
    if (lowp_trsm) *lowp_trsm = e.ctrsm ? 1 : 0;
    return MP_OK;
}

// ------------------------------------------------------------------ matrices
mp_status mp_matrix_create(mp_handle* h, int64_t n, int nb, mp_matrix** A) {
    if (!h || !A) return MP_ERR_ARG;
    if (n < 1 || nb < 16 || nb > 8192 || nb % 16) FAIL(h, MP_ERR_ARG, "invalid n=%lld nb=%d", (long long)n, nb);
    const int64_t nt = (n + nb - 1) / nb;
    if (nt > 4096) FAIL(h, MP_ERR_ARG, "too many tiles (NT=%lld)", (long long)nt);
    mp_matrix* M = new mp_matrix();
    M->h = h;
    M->n = n;
    M->nb = nb;
    M->nt = (int)nt;
    *A = M;
    return MP_OK;
}

mp_status mp_matrix_destroy(mp_matrix* A) {
    if (!A) return MP_ERR_ARG;
    for (size_t r = 0; r < A->comm.peer.size(); ++r)
        if (A->comm.peer[r] && A->comm.peer[r] != A->comm.base) cudaIpcCloseMemHandle(A->comm.peer[r]);
    if (A->comm.base) cudaFree(A->comm.base);
    delete A;
    return MP_OK;
}

static size_t comm_layout(mp_matrix* A) {
    Comm& c = A->comm;
    const size_t nt = A->nt, nb = A->nb, nb2 = A->nb2();
    size_t off = 0;
    auto take = [&](size_t bytes) {
        off = align_up(off, 256);
        const size_t o = off;
        off += bytes;
        return o;
    };
    c.hdr = take(128);  // the communicator id (mp_get_unique_id), checked by every peer at connect
    c.send = take(2 * nt * nb2 * 8);
    c.pub = take(2 * nt * 8);
    c.done = take(2 * 8);
    c.bar = take(8);
    c.part = take(nt * nb * 8);
    c.yv = take(nt * nb * 8);
    c.pflag = take(nt * 8);
    c.yflag = take(nt * 8);
    c.norms = take(nt * nt * 8);
    c.nflag = take(8);
    c.scal = take(4 * 8);
    c.sflag = take(8);
    c.tmp = take(nb * 8);
    return align_up(off, 256);
}

mp_status mp_matrix_comm_export(mp_matrix* A, void* handle_out) {
    if (!A || !handle_out) return MP_ERR_ARG;
    mp_handle* h = A->h;
    if (h->nranks < 2) FAIL(h, MP_ERR_STATE, "single-rank handle has no exchange area");
    Comm& c = A->comm;
    if (!c.base) {
        c.bytes = comm_layout(A);
        CK(h, cudaMalloc(&c.base, c.bytes));
        CK(h, cudaMemset(c.base, 0, c.bytes));
        CK(h, cudaMemcpy(c.base + c.hdr, h->id, 128, cudaMemcpyHostToDevice));
        CK(h, cudaDeviceSynchronize());
    }
    cudaIpcMemHandle_t ih;
    CK(h, cudaIpcGetMemHandle(&ih, c.base));
    memcpy(handle_out, &ih, sizeof ih);
    return MP_OK;
}

mp_status mp_matrix_comm_connect(mp_matrix* A, const void* all_handles) {
    if (!A || !all_handles) return MP_ERR_ARG;
    mp_handle* h = A->h;
    Comm& c = A->comm;
    if (!c.base) FAIL(h, MP_ERR_STATE, "call mp_matrix_comm_export first");
    c.peer.assign(h->nranks, nullptr);
    for (int r = 0; r < h->nranks; ++r) {
        if (r == h->rank) {
            c.peer[r] = c.base;
            continue;
        }
        cudaIpcMemHandle_t ih;
        memcpy(&ih, (const char*)all_handles + (size_t)r * sizeof ih, sizeof ih);
        void* p = nullptr;
        CK(h, cudaIpcOpenMemHandle(&p, ih, cudaIpcMemLazyEnablePeerAccess));
        c.peer[r] = (char*)p;
        uint8_t pid[128];
        CK(h, cudaMemcpy(pid, c.peer[r] + c.hdr, 128, cudaMemcpyDeviceToHost));
        if (memcmp(pid, h->id, 128) != 0)
            FAIL(h, MP_ERR_COMM, "rank %d's exchange area carries another communicator id (mp_get_unique_id)", r);
    }
    c.connected = true;
    return MP_OK;
}

int mp_matrix_nt(const mp_matrix* A) { return A ? A->nt : 0; }
int mp_matrix_owner(const mp_matrix* A, int m, int k) { return A ? A->owner(m, k) : -1; }

mp_status mp_matrix_bytes(const mp_matrix* A, const uint8_t* storage_prec, size_t* bytes) {
    if (!A || !bytes) return MP_ERR_ARG;
    *bytes = layout(A, storage_prec).total;
    return MP_OK;
}

mp_status mp_matrix_bind(mp_matrix* A, const uint8_t* storage_prec, void* d_workspace, size_t bytes) {
    if (!A || !d_workspace) return MP_ERR_ARG;
    mp_handle* h = A->h;
    if ((uintptr_t)d_workspace % 256) FAIL(h, MP_ERR_ARG, "workspace must be 256-byte aligned");
    const int nt = A->nt;
    if (storage_prec)
        for (int k = 0; k < nt; ++k)
            for (int m = k; m < nt; ++m) {
                const uint8_t p = storage_prec[(size_t)m * nt + k];
                if (p > MP_FP16) FAIL(h, MP_ERR_ARG, "storage map entry (%d,%d)=%d", m, k, p);
                if (m == k && p != MP_FP64) FAIL(h, MP_ERR_ARG, "diagonal tiles are stored in FP64 (P:117)");
            }
    Regions R = layout(A, storage_prec);
    if (R.total > bytes) FAIL(h, MP_ERR_NOMEM, "workspace %zu bytes < required %zu", bytes, R.total);
    A->R = std::move(R);
    A->ws = (char*)d_workspace;
    A->ws_bytes = bytes;
    A->storage.assign((size_t)nt * nt, 255);
    for (int k = 0; k < nt; ++k)
        for (int m = k; m < nt; ++m)
            A->storage[(size_t)m * nt + k] = storage_prec ? storage_prec[(size_t)m * nt + k] : (uint8_t)MP_FP64;
    // FP16 storage class: per-tile exponent t with ||A_mk||_F 2^t <= 2^10, from the norms of the last
    // generation pass 1 (every entry is below the tile's Frobenius norm, so the stored values stay 2^6 below
    // the FP16 maximum, leaving headroom for the trailing updates; without norms t = 0)
    A->tscale.assign((size_t)nt * nt, 0);
    for (int k = 0; k < nt; ++k)
        for (int m = k + 1; m < nt; ++m) {
            const size_t i = (size_t)m * nt + k;
            if (A->storage[i] != MP_FP16 || A->sqn.size() != (size_t)nt * nt || !(A->sqn[i] > 0)) continue;
            const int e = (int)std::floor(std::log2(std::sqrt(A->sqn[i])));
            A->tscale[i] = std::max(-900, std::min(900, 10 - e - 1));
        }
    A->bound = true;
    A->generated = A->factored = false;
    return MP_OK;
}

mp_status mp_matrix_attach(mp_matrix* A, void* d_workspace, size_t bytes) {
    if (!A || !d_workspace) return MP_ERR_ARG;
    mp_handle* h = A->h;
    if ((uintptr_t)d_workspace % 256) FAIL(h, MP_ERR_ARG, "workspace must be 256-byte aligned");
    Regions R = layout(A, NO_POOL);
    if (R.total > bytes) FAIL(h, MP_ERR_NOMEM, "workspace %zu bytes < map-independent regions %zu", bytes, R.total);
    A->R = std::move(R);
    A->ws = (char*)d_workspace;
    A->ws_bytes = bytes;
    A->storage.assign((size_t)A->nt * A->nt, 255);
    A->bound = true;  // pass 1 of the generation (norms) needs only the map-independent regions
    A->generated = A->factored = false;
    return MP_OK;
}

mp_status mp_matrix_maps(const mp_matrix* A, uint8_t* kernel_prec, uint8_t* storage_prec, uint8_t* comm_prec) {
    if (!A) return MP_ERR_ARG;
    const size_t NN = (size_t)A->nt * A->nt;
    if (kernel_prec && A->kmap.size() == NN) memcpy(kernel_prec, A->kmap.data(), NN);
    if (storage_prec && A->storage.size() == NN) memcpy(storage_prec, A->storage.data(), NN);
    if (comm_prec && A->cmap.size() == NN) memcpy(comm_prec, A->cmap.data(), NN);
    return MP_OK;
}

mp_status mp_matrix_get_tile(mp_handle* h, const mp_matrix* A, int m, int k, double* h_tile) {
    if (!h || !A || !h_tile || !A->bound || m < k || m >= A->nt || k < 0) return MP_ERR_ARG;
    if (!A->mine(m, k)) FAIL(h, MP_ERR_ARG, "tile (%d,%d) not owned by rank %d", m, k, h->rank);
    if (A->R.tile_off[(size_t)m * A->nt + k] == SIZE_MAX) FAIL(h, MP_ERR_STATE, "no tile pool laid out");
    const size_t nb2 = A->nb2();
    if (A->st(m, k) == MP_FP64) {
        CK(h, cudaMemcpyAsync(h_tile, A->tile(m, k), nb2 * 8, cudaMemcpyDeviceToHost, h->stream));
        CK(h, cudaStreamSynchronize(h->stream));
    } else if (A->st(m, k) == MP_FP16) {
        std::vector<__half> tmp(nb2);
        CK(h, cudaMemcpyAsync(tmp.data(), A->tile(m, k), nb2 * 2, cudaMemcpyDeviceToHost, h->stream));
        CK(h, cudaStreamSynchronize(h->stream));
        const double sc = std::ldexp(1.0, -A->ts(m, k));
        for (size_t i = 0; i < nb2; ++i) h_tile[i] = (double)__half2float(tmp[i]) * sc;
    } else {
        std::vector<float> tmp(nb2);
        CK(h, cudaMemcpyAsync(tmp.data(), A->tile(m, k), nb2 * 4, cudaMemcpyDeviceToHost, h->stream));
        CK(h, cudaStreamSynchronize(h->stream));
        for (size_t i = 0; i < nb2; ++i) h_tile[i] = tmp[i];
    }
    return MP_OK;
}

mp_status mp_matrix_set_tile(mp_handle* h, mp_matrix* A, int m, int k, const double* h_tile) {
    if (!h || !A || !h_tile || !A->bound || m < k || m >= A->nt || k < 0) return MP_ERR_ARG;
    if (!A->mine(m, k)) FAIL(h, MP_ERR_ARG, "tile (%d,%d) not owned by rank %d", m, k, h->rank);
    if (A->R.tile_off[(size_t)m * A->nt + k] == SIZE_MAX) FAIL(h, MP_ERR_STATE, "no tile pool laid out");
    const size_t nb2 = A->nb2();
    if (A->st(m, k) == MP_FP64) {
        CK(h, cudaMemcpyAsync(A->tile(m, k), h_tile, nb2 * 8, cudaMemcpyHostToDevice, h->stream));
        CK(h, cudaStreamSynchronize(h->stream));
    } else if (A->st(m, k) == MP_FP16) {
        std::vector<__half> tmp(nb2);
        const double sc = std::ldexp(1.0, A->ts(m, k));
        for (size_t i = 0; i < nb2; ++i) tmp[i] = __float2half((float)(h_tile[i] * sc));
        CK(h, cudaMemcpyAsync(A->tile(m, k), tmp.data(), nb2 * 2, cudaMemcpyHostToDevice, h->stream));
        CK(h, cudaStreamSynchronize(h->stream));
    } else {
        std::vector<float> tmp(nb2);
        for (size_t i = 0; i < nb2; ++i) tmp[i] = (float)h_tile[i];
        CK(h, cudaMemcpyAsync(A->tile(m, k), tmp.data(), nb2 * 4, cudaMemcpyHostToDevice, h->stream));
        CK(h, cudaStreamSynchronize(h->stream));
    }
    A->generated = true;
    A->factored = false;
    return MP_OK;
}

// ------------------------------------------------------------------ multi-rank host helpers
// Host wait for a peer stamp (used by the host-synchronous collectives: norm gather, scalars).
static mp_status host_wait_stamp(mp_handle* h, const uint64_t* dflag, uint64_t target) {
    for (long it = 0;; ++it) {
        uint64_t v = 0;
        CK(h, cudaMemcpy(&v, dflag, 8, cudaMemcpyDeviceToHost));
        if (v >= target) return MP_OK;
        if (it > 20000000) FAIL(h, MP_ERR_COMM, "timeout waiting for a peer stamp");
        if (it > 100) usleep(50);
    }
}

// Barrier among all ranks through device flags (host-synchronous).
static mp_status dist_barrier(mp_handle* h, mp_matrix* A, uint64_t stamp) {
    Comm& X = A->comm;
    CK(h, set_flag_launch((uint64_t*)(X.base + X.bar), stamp, h->stream));
    CK(h, cudaStreamSynchronize(h->stream));
    for (int r = 0; r < h->nranks; ++r)
        if (r != h->rank)
            if (mp_status st = host_wait_stamp(h, (const uint64_t*)(X.peer[r] + X.bar), stamp)) return st;
    return MP_OK;
}

// ------------------------------------------------------------------ (1) generation
static mp_status check_theta(mp_handle* h, const double* th, int cov = MP_COV_MATERN) {
    if (!th || !(th[0] > 0) || !(th[1] > 0) || !std::isfinite(th[0]) || !std::isfinite(th[1]))
        FAIL(h, MP_ERR_ARG, "invalid theta (sigma2, beta > 0)");
    if (cov == MP_COV_MATERN && (!(th[2] > 0) || !(th[2] <= 20.0)))
        FAIL(h, MP_ERR_ARG, "invalid theta (Matern: 0 < nu <= 20)");
    return MP_OK;
}

mp_status mp_matrix_set_covariance(mp_matrix* A, mp_covariance kind) {
    if (!A || (kind != MP_COV_MATERN && kind != MP_COV_SQEXP)) return MP_ERR_ARG;
    A->cov = kind;
    A->generated = A->factored = false;
    return MP_OK;
}

static MaternArgs matern_args(const mp_matrix* A, const double* x, const double* y, const double* th) {
    MaternArgs a{};
    a.x = x;
    a.y = y;
    a.n = A->n;
    a.nb = A->nb;
    a.sigma2 = th[0];
    a.beta = th[1];
    a.nu = th[2];
    if (A->cov == MP_COV_SQEXP) {
        a.kind = 4;
        a.nu = 0.0;
        a.coef = 0.0;
    } else {
        a.kind = th[2] == 0.5 ? 0 : th[2] == 1.5 ? 1 : th[2] == 2.5 ? 2 : 3;
        a.coef = std::pow(2.0, 1.0 - th[2]) / std::tgamma(th[2]);
    }
    return a;
}

mp_status mp_matern_gen(mp_handle* h, mp_matrix* A, const double* d_x, const double* d_y, const double theta[3],
                        const uint8_t* storage_prec, double* tile_sqnorm) {
    if (!h || !A || !d_x || !d_y) return MP_ERR_ARG;
    if (h->broken) FAIL(h, MP_ERR_STATE, "handle unusable after an earlier CUDA failure");
    if (mp_status s = check_theta(h, theta, A->cov)) return s;
    if (h->nranks > 1 && !A->comm.connected) FAIL(h, MP_ERR_COMM, "multi-rank matrix not connected");
    const int nt = A->nt;
    MaternArgs a = matern_args(A, d_x, d_y, theta);
    if (a.kind == 3 && A->bound && h->cfg.matern_table) {
        // pieces of width w = 1/8 in u = log(r/2) on [-w*split, log(r_max/2)]; r_max bounds every
        // distance of points in the unit square (sqrt 2) — outside points fall back to direct K_nu
        const double w = 0.125;
        const double rmax = 1.5 / a.beta;
        const int split = 96;  // 12 units of u below log 2: r down to 2 e^-12 ~ 1.2e-5
        const int above = std::max(1, (int)std::ceil((std::log(rmax) - std::log(2.0)) / w));
        if (split + above <= MT_PIECES_MAX) {
            a.u0 = std::log(2.0) - w * split;
            a.w = w;
            a.inv_w = 1.0 / w;
            a.split = split;
            a.npieces = split + above;
            double* tab = A->at<double>(A->R.mtab);
            a.tab = nullptr;  // the table kernel samples the direct formula
            CK(h, matern_table_launch(a, tab, h->stream));
            h->launches++;
            a.tab = tab;
        }
    }
    if (!storage_prec) {
        // pass 1: norms.  Needs scratch for partials: use the bound workspace if present,
        // otherwise the caller must bind first (norm scratch lives in the workspace).
        if (!A->bound) FAIL(h, MP_ERR_STATE, "bind a workspace before mp_matern_gen");
        if (!tile_sqnorm) return MP_ERR_ARG;
        std::vector<GenTile> tl;
        for (int k = 0; k < nt; ++k)
            for (int m = k; m < nt; ++m)
                if (A->mine(m, k)) tl.push_back(GenTile{m, k, 0, 0, nullptr});
        Arena ar;
        ar.dev_base = A->ws + A->R.ctrl;
        GenTile* d_tl = ar.push(tl);
        double* part = A->at<double>(A->R.partials);
        double* norms = A->at<double>(A->R.norms);
        const int per = A->nb / GEN_ROWS;
        std::vector<Op> ops;
        const int ntl = (int)tl.size();
        ops.push_back({[=](cudaStream_t s) { return matern_norm_launch(a, d_tl, ntl, part, s); }, C_GEN, 0});
        ops.push_back({[=](cudaStream_t s) { return reduce_partials_launch(part, ntl, per, norms, s); }, C_GEN, 0});
        if (mp_status st = run_plan(h, A, ar, ops)) return st;
        std::vector<double> v(ntl);
        CK(h, cudaMemcpyAsync(v.data(), norms, ntl * 8, cudaMemcpyDeviceToHost, h->stream));
        CK(h, cudaStreamSynchronize(h->stream));
        for (size_t i = 0; i < (size_t)nt * nt; ++i) tile_sqnorm[i] = 0.0;
        for (int i = 0; i < ntl; ++i) tile_sqnorm[(size_t)tl[i].m * nt + tl[i].k] = v[i];
        A->sqn.clear();
        if (h->nranks > 1) {
            // all-gather over peer memory: every tile has exactly one owner, so the merge is exact
            Comm& X = A->comm;
            const uint64_t stamp = (++X.epoch << 24) + 1;
            if (mp_status st = dist_barrier(h, A, stamp)) return st;
            CK(h, cudaMemcpy(X.base + X.norms, tile_sqnorm, (size_t)nt * nt * 8, cudaMemcpyHostToDevice));
            CK(h, set_flag_launch((uint64_t*)(X.base + X.nflag), stamp, h->stream));
            CK(h, cudaStreamSynchronize(h->stream));
            std::vector<double> tmp((size_t)nt * nt);
            for (int r = 0; r < h->nranks; ++r) {
                if (r == h->rank) continue;
                if (mp_status st = host_wait_stamp(h, (const uint64_t*)(X.peer[r] + X.nflag), stamp)) return st;
                CK(h, cudaMemcpy(tmp.data(), X.peer[r] + X.norms, tmp.size() * 8, cudaMemcpyDeviceToHost));
                for (size_t i = 0; i < tmp.size(); ++i) tile_sqnorm[i] += tmp[i];
            }
            if (mp_status st = dist_barrier(h, A, stamp + 1)) return st;
        }
        A->sqn.assign(tile_sqnorm, tile_sqnorm + (size_t)nt * nt);  // the FP16 storage class's tile exponents
        return MP_OK;
    }
    if (!A->bound) FAIL(h, MP_ERR_STATE, "matrix not bound");
    for (int k = 0; k < nt; ++k)
        for (int m = k; m < nt; ++m)
            if (storage_prec[(size_t)m * nt + k] != A->st(m, k))
                FAIL(h, MP_ERR_ARG, "storage map differs from the bound one at (%d,%d)", m, k);
    std::vector<GenTile> tl;
    for (int k = 0; k < nt; ++k)
        for (int m = k; m < nt; ++m)
            if (A->mine(m, k)) tl.push_back(GenTile{m, k, A->st(m, k), A->ts(m, k), A->tile(m, k)});
    Arena ar;
    ar.dev_base = A->ws + A->R.ctrl;
    GenTile* d_tl = ar.push(tl);
    const int ntl = (int)tl.size();
    std::vector<Op> ops;
    ops.push_back({[=](cudaStream_t s) { return matern_write_launch(a, d_tl, ntl, s); }, C_GEN, 0});
    if (mp_status st = run_plan(h, A, ar, ops)) return st;
    A->generated = true;
    A->factored = false;
    return MP_OK;
}

// ------------------------------------------------------------------ (3) factorisation
struct FlopCount {
    double potrf = 0, trsm = 0, upd[4] = {0, 0, 0, 0};  // upd[MP_FP16H]: four-level maps
};

static mp_status plan_potrf(mp_handle* h, mp_matrix* A, const uint8_t* km, const uint8_t* cm, Arena& ar,
                            std::vector<Op>& ops, FlopCount& fc, uint64_t epoch) {
    const int nt = A->nt, nb = A->nb, IB = POTRF_IB, OB = 4 * POTRF_IB;
    const size_t nb2 = A->nb2();
    const size_t slots = (size_t)nt * nb2;  // elements of one panel's worth of slots
    const Engines E = engines_for(h, nb);
    const Regions& RG = A->R;
    double* const p64b = A->at<double>(RG.p64);
    __half* const h16hi = E.h16 ? A->at<__half>(RG.h16) : nullptr;  // [nt*nb][nb] hi planes, then lo
    __half* const h16lo = E.h16 ? h16hi + slots : nullptr;
    __half* const h16s = RG.h16s ? A->at<__half>(RG.h16s) : nullptr;  // pure-FP16 operands (four-level maps)
    int* const e16 = E.h16 ? A->at<int>(RG.e16) : nullptr;
    float* const phi = RG.phi ? A->at<float>(RG.phi) : nullptr;
    float* const plo = RG.plo ? A->at<float>(RG.plo) : nullptr;
    double* ltil = A->at<double>(RG.ltilde);
    double* wb = A->at<double>(RG.wbuf);
    double* wb2 = A->at<double>(RG.wbuf2);
    int* d_info = h->d_info;
    const float* const cpool = A->at<float>(RG.pool);  // tcgen05 epilogue C map range (FP32 view of the pool)
    const uint64_t crows = (RG.total - RG.pool) / ((size_t)nb * 4);
    const double* const cpool64 = A->at<double>(RG.pool);  // FP64 view of the pool (CRT epilogue C map)
    const uint64_t crows64 = (RG.total - RG.pool) / ((size_t)nb * 8);
    CrtConst crtc, crtc32;
    if (E.crt && !crt_constants(CRT_NMAX, nb, &crtc)) FAIL(h, MP_ERR_ARG, "CRT constants for nb=%d", nb);
    if (E.ctrsm && !crt_constants(8, nb, &crtc32)) FAIL(h, MP_ERR_ARG, "CRT-8 constants for nb=%d", nb);
    int8_t* const ozs = E.crt ? A->at<int8_t>(RG.oz) : nullptr;
    int* const oze = E.crt ? A->at<int>(RG.ozexp) : nullptr;
    int8_t* const o32s = E.ctrsm ? A->at<int8_t>(RG.oz32) : nullptr;
    int* const e32 = E.ctrsm ? A->at<int>(RG.e32) : nullptr;
    double* const wfac = E.ctrsm ? A->at<double>(RG.wfac) : nullptr;
    const int64_t plane = (int64_t)slots;  // bytes between int8 residue planes
    uint8_t* const crt_scr = E.crt ? A->at<uint8_t>(RG.crt) : nullptr;
    int* const crt_flags = E.crt ? A->at<int>(RG.crtflags) : nullptr;
    // one tile-scheduler counter per CRT launch of this call (zeroed by potrf_run)
    int* const crt_ctr = E.crt ? A->at<int>(RG.crtctr) : nullptr;
    size_t ctr_next = 0;
    auto next_ctr = [&]() -> int* {  // two ints per launch
        if (ctr_next + 2 > crt_counters(nt)) return nullptr;
        ctr_next += 2;
        return crt_ctr + ctr_next - 2;
    };
    auto K = [&](int m, int k) { return km[(size_t)m * nt + k]; };
    auto C = [&](int m, int k) { return cm[(size_t)m * nt + k]; };
    auto xscale = [&](int m, int k) { return A->ts(m, k); };  // FP16 storage class payloads carry the tile exponent
    if (E.s16 && !E.tc16)
        for (int k = 0; k < nt; ++k)
            for (int m = k + 1; m < nt; ++m)
                if (A->st(m, k) == MP_FP16)
                    FAIL(h, MP_ERR_UNSUPPORTED, "FP16 storage class needs the tcgen05 FP16 engine (nb %% 256 == 0)");
    const double fnb = (double)nb;
    std::vector<Op>* cur = nullptr;
    auto cur_push = [&](Op o) { cur->push_back(std::move(o)); };
    // ---- multi-rank exchange helpers; unused on one rank
    const bool dist = h->nranks > 1;
    const bool la = h->cfg.lookahead != 0;  // also multi-rank: exchange waits run on the panel stream
    // persistent CRT grids: the update leaves reserve_pairs CTA pairs to the panel stream (lookahead)
    int nsm = 148;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, h->device);
    const int upd_pairs = la ? std::max(1, nsm / 2 - h->cfg.reserve_pairs) : 0;
    const int pan_pairs = 0;  // panel-stream CRT launches: any free SM (dynamic tiles, high priority)
    const int R = h->nranks, me = h->rank;
    Comm& X = A->comm;
    auto ST = [&](int step) -> uint64_t { return (epoch << 24) + (uint64_t)(step + 2); };
    auto sendslot = [&](int r, int s, int m) { return X.peer[r] + X.send + ((size_t)s * nt + m) * nb2 * 8; };
    auto pubflag = [&](int r, int s, int m) { return (uint64_t*)(X.peer[r] + X.pub) + (size_t)s * nt + m; };
    auto doneflag = [&](int r, int s) { return (uint64_t*)(X.peer[r] + X.done) + s; };
    // the exchange records this rank executes (exchange.cpp, also checked by the CPU tests)
    std::vector<std::vector<mp_xfer>> xpub(nt), xpull(nt);
    if (dist) {
        int64_t cnt = 0;
        mp_exchange_plan(nt, h->P, h->Q, me, cm, nullptr, 0, &cnt);
        std::vector<mp_xfer> xs((size_t)cnt);
        if (mp_exchange_plan(nt, h->P, h->Q, me, cm, xs.data(), cnt, &cnt)) FAIL(h, MP_ERR_ARG, "exchange plan failed");
        for (auto& x : xs) (x.dir == 0 ? xpub : xpull)[x.k].push_back(x);
    }
    // the operand classes MY successors of L_mk run at: SYRK(m,k) on (m,m), GEMM(m,n,k), GEMM(n,m,k)
    auto needs = [&](int k, int m, bool& n16, bool& n32, bool& n64, bool& n16h) {
        n16 = n32 = n16h = false;
        n64 = A->mine(m, m);
        auto cls = [&](int p) { n16 |= p == MP_FP16, n32 |= p == MP_FP32, n64 |= p == MP_FP64, n16h |= p == MP_FP16H; };
        for (int n = k + 1; n < m; ++n)
            if (A->mine(m, n)) cls(K(m, n));
        for (int n = m + 1; n < nt; ++n)
            if (A->mine(n, m)) cls(K(n, m));
    };
    auto push_wait = [&](std::vector<WaitItem>& w) {
        if (w.empty()) return;
        WaitItem* dw = ar.push(w);
        const int n = (int)w.size();
        cur_push(Op{[=](cudaStream_t s) { return wait_flags_launch(dw, n, s); }, C_CONV, 0});
    };

    // per step: pan(k) = POTRF + TRSM + panel out (+ exchange); fmt(k) = the operand formats of
    // panel k; nxt(k) = the update of column k+1 (what panel k+1 waits for); rst(k) = the rest of the
    // trailing update
    std::vector<std::vector<Op>> pan(nt), fmt(nt), nxt(nt), rst(nt);
    auto gemm = [&](std::vector<GemmJob>& jobs, int M, int N, int Kd, int lda, int ldb, int ldc, int lower,
                    double alpha, double beta, int round, bool cf32, int cls, double flops_per_job) {
        if (jobs.empty()) return;
        GemmJob* dj = ar.push(jobs);
        DgemmArgs g{};
        g.jobs = dj;
        g.M = M;
        g.N = N;
        g.K = Kd;
        g.lda = lda;
        g.ldb = ldb;
        g.ldc = ldc;
        g.lower = lower;
        g.alpha = alpha;
        g.beta = beta;
        const int nj = (int)jobs.size();
        cur->push_back({[=](cudaStream_t s) { return dgemm_nt_launch(g, nj, round, cf32, s); }, cls, flops_per_job * nj});
    };
    auto crt_args = [&](const CrtJob* dj, const int8_t* planes, const int* exps, int lower, const CrtConst& c,
                        const void* cbase, uint64_t cr, int pairs, int store) {
        CrtArgs a{};
        a.jobs = dj;
        a.planes = planes;
        a.exps = exps;
        a.plane_stride = plane;
        a.nb = nb;
        a.nt = nt;
        a.lower = lower;
        a.scratch = crt_scr;
        a.slot_flags = crt_flags;
        a.c = c;
        a.cbase = cbase;
        a.crows = cr;
        a.max_pairs = pairs;
        a.store = store;
        a.counter = next_ctr();
        a.phase_lock = h->cfg.crt_phase_lock;
        return a;
    };

    for (int k = 0; k < nt; ++k) {
        const size_t set = E.p64_double ? (size_t)(k & 1) : 0;
        const int sp = k & 1;  // send-slot parity (multi-rank)
        bool send_free_waited = false;
        auto wait_send_free = [&]() {  // every peer has pulled panel k-2 from slot set sp
            if (send_free_waited || k < 2) return;
            std::vector<WaitItem> w;
            for (int r = 0; r < R; ++r)
                if (r != me) w.push_back(WaitItem{doneflag(r, sp), ST(k - 2)});
            push_wait(w);
            send_free_waited = true;
        };
        double* p64 = p64b + set * slots;
        cur = &pan[k];
        // ---- 1. DPOTRF(k,k), FP64: two-level blocking — 128-column blocks
        //      (diagonal block Cholesky + inverse, block column as GEMM with the inverse, update
        //      inside the 512-column outer block), then one K = 512 SYRK per outer block.
        if (dist && k == 0) {  // device-side barrier: every rank finished the previous collective
            uint64_t* bar = (uint64_t*)(X.base + X.bar);
            const uint64_t bv = ST(-1);
            cur_push(Op{[=](cudaStream_t s) { return set_flag_launch(bar, bv, s); }, C_CONV, 0});
            std::vector<WaitItem> w;
            for (int r = 0; r < R; ++r)
                if (r != me) w.push_back(WaitItem{(uint64_t*)(X.peer[r] + X.bar), bv});
            push_wait(w);
        }
        if (A->mine(k, k)) {
            double* Akk = (double*)A->tile(k, k);
            for (int J0 = 0; J0 < nb; J0 += OB) {
                const int Jend = std::min(nb, J0 + OB), Jb = Jend - J0;
                for (int j0 = J0; j0 < Jend; j0 += IB) {
                    const int jb = std::min(IB, Jend - j0), jend = j0 + jb;
                    double* blk = Akk + (size_t)j0 * nb + j0;
                    const int col0 = k * nb + j0;
                    cur->push_back({[=](cudaStream_t s) { return potrf_diag_block_launch(blk, nb, jb, wb, col0, d_info, s); },
                                   C_POTRF, (double)jb * jb * jb / 3.0});
                    const int rest = nb - jend;
                    if (rest <= 0) continue;
                    double* Xb = Akk + (size_t)jend * nb + j0;
                    std::vector<GemmJob> j1{GemmJob{Xb, wb, Xb}};
                    gemm(j1, rest, jb, jb, nb, IB, nb, 0, 1.0, 0.0, P64, false, C_POTRF, (double)rest * jb * jb);
                    if (Jend > jend) {
                        std::vector<GemmJob> j2{GemmJob{Xb, Xb, Akk + (size_t)jend * nb + jend}};
                        gemm(j2, rest, Jend - jend, jb, nb, nb, nb, 0, -1.0, 1.0, P64, false, C_POTRF,
                             2.0 * rest * (Jend - jend) * jb);
                    }
                }
                const int rest = nb - Jend;
                if (rest > 0) {
                    double* Y = Akk + (size_t)Jend * nb + J0;
                    std::vector<GemmJob> j3{GemmJob{Y, Y, Akk + (size_t)Jend * nb + Jend}};
                    gemm(j3, rest, rest, Jb, nb, nb, nb, 1, -1.0, 1.0, P64, false, C_POTRF, (double)rest * rest * Jb);
                }
            }
            cur->push_back({[=](cudaStream_t s) { return zero_upper_launch(Akk, nb, s); }, C_POTRF, 0});
            fc.potrf += fnb * fnb * fnb / 3.0;
        }
        if (k == nt - 1) break;
        // ---- 2. L~_kk at comm(k,k) and its 128-block inverses (TRSM operand, Alg. 2 l.5-10);
        //      multi-rank: the owner publishes L~_kk in comm(k,k) precision, the TRSM owners of
        //      column k pull it (fused transfer + up-conversion)
        bool trsm_here = false;
        for (int m = k + 1; m < nt; ++m) trsm_here |= A->mine(m, k);
        {
            const int pc = C(k, k);
            bool pub_kk = false;
            int pull_kk = -1;
            for (auto& x : xpub[k]) pub_kk |= x.m == k;
            for (auto& x : xpull[k])
                if (x.m == k) pull_kk = x.peer;
            if (A->mine(k, k)) {
                double* Akk = (double*)A->tile(k, k);
                cur->push_back({[=](cudaStream_t s) { return round_copy_launch(Akk, ltil, (int64_t)nb2, pc, s); }, C_TRSM, 0});
                if (pub_kk) {
                    wait_send_free();
                    std::vector<PackItem> pk{PackItem{ltil, sendslot(me, sp, k), pc, 0}};
                    PackItem* dp = ar.push(pk);
                    uint64_t* f = pubflag(me, sp, k);
                    const uint64_t v = ST(k);
                    cur_push(Op{[=](cudaStream_t s) { return pack_launch(dp, 1, (int64_t)nb2, s); }, C_CONV, 0});
                    cur_push(Op{[=](cudaStream_t s) { return set_flag_launch(f, v, s); }, C_CONV, 0});
                }
            } else if (pull_kk >= 0) {
                const int o = pull_kk;
                std::vector<WaitItem> w{WaitItem{pubflag(o, sp, k), ST(k)}};
                push_wait(w);
                std::vector<PullItem> pl{PullItem{sendslot(o, sp, k), pubflag(o, sp, k), ST(k), ltil, pc, 0}};
                PullItem* dp = ar.push(pl);
                cur_push(Op{[=](cudaStream_t s) { return pull_launch(dp, 1, (int64_t)nb2, s); }, C_CONV, 0});
            }
            if (trsm_here || !dist)
                cur->push_back({[=](cudaStream_t s) { return trtri_blocks_launch(ltil, nb, wb2, s); }, C_TRSM, 0});
        }
        // ---- 3. panel in
        std::vector<PanelTile> pin;
        for (int m = k + 1; m < nt; ++m)
            if (A->mine(m, k))
                pin.push_back(PanelTile{A->tile(m, k), p64 + (size_t)m * nb2, A->st(m, k), C(m, k), A->ts(m, k), 0});
        if (!pin.empty()) {
            PanelTile* d_in = ar.push(pin);
            const int np = (int)pin.size();
            cur->push_back({[=](cudaStream_t s) { return panel_in_launch(d_in, np, (int64_t)nb2, s); }, C_CONV, 0});
            // ---- 4. TRSM(m,k): L_mk = A_mk L~_kk^{-T}.  FP64-class tiles: FP64 arithmetic (
            //      reading C12'), right-looking over 128-column blocks (X_j = X_j W_j^T) with the updates
            //      inside a 512-column outer block at K = 128 and across outer blocks at K = 512.
            //      FP32/FP16-class tiles (the paper's FP32 TRSM) with ctrsm: 4b below.
            std::vector<double*> dm;  // DMMA substitution targets (panel slots)
            std::vector<int> lo;      // low-precision-class tiles (ctrsm)
            for (auto& t : pin) {
                const int m = (int)((t.p64 - p64) / (ptrdiff_t)nb2);
                if (E.ctrsm && K(m, k) != MP_FP64) lo.push_back(m);
                else dm.push_back(t.p64);
            }
            double* const islot = p64 + (size_t)k * nb2;  // panel slot k is free in panel k
            if (!lo.empty()) {  // right-hand side I: its substitution gives L~_kk^-T
                cur->push_back({[=](cudaStream_t s) { return identity_launch(islot, nb, s); }, C_TRSM, 0});
                dm.push_back(islot);
            }
            for (int J0 = 0; J0 < nb; J0 += OB) {
                const int Jend = std::min(nb, J0 + OB), Jb = Jend - J0;
                for (int j0 = J0; j0 < Jend; j0 += IB) {
                    const int jb = std::min(IB, Jend - j0), jend = j0 + jb;
                    std::vector<GemmJob> ja, jin;
                    for (double* x : dm) {
                        ja.push_back(GemmJob{x + j0, wb2 + (size_t)(j0 / IB) * IB * IB, x + j0});
                        if (Jend > jend) jin.push_back(GemmJob{x + j0, ltil + (size_t)jend * nb + j0, x + jend});
                    }
                    gemm(ja, nb, jb, jb, nb, IB, nb, 0, 1.0, 0.0, P64, false, C_TRSM, fnb * jb * jb);
                    gemm(jin, nb, Jend - jend, jb, nb, nb, nb, 0, -1.0, 1.0, P64, false, C_TRSM, 2.0 * fnb * (Jend - jend) * jb);
                }
                if (nb > Jend) {
                    std::vector<GemmJob> jo;
                    for (double* x : dm) jo.push_back(GemmJob{x + J0, ltil + (size_t)Jend * nb + J0, x + Jend});
                    gemm(jo, nb, nb - Jend, Jb, nb, nb, nb, 0, -1.0, 1.0, P64, false, C_TRSM, 2.0 * fnb * (nb - Jend) * Jb);
                }
            }
            // ---- 4b. FP32/FP16-class TRSM as the FP32-class product L_mk = A_mk W^T with the inverse
            //      factor W = L~_kk^-1 (its FP64 substitution above, transposed): both operands as 8 CRT
            //      residue planes (b = 25 bits per row), one CRT-8 launch over the column with an FP64 C
            //      (store mode) into the panel slots, where panel out (step 5) picks the tiles up.
            if (!lo.empty()) {
                cur->push_back({[=](cudaStream_t s) { return transpose_launch(islot, wfac, nb, s); }, C_TRSM, 0});
                std::vector<CrtSplitItem> spl{CrtSplitItem{wfac, o32s + (size_t)k * nb2, e32 + (size_t)k * nb, plane}};
                std::vector<CrtJob> tj;
                for (int m : lo) {
                    spl.push_back(CrtSplitItem{p64 + (size_t)m * nb2, o32s + (size_t)m * nb2, e32 + (size_t)m * nb, plane});
                    tj.push_back(CrtJob{m, k, p64 + (size_t)m * nb2});
                }
                CrtSplitItem* dsp = ar.push(spl);
                const int nsp = (int)spl.size();
                cur->push_back({[=](cudaStream_t s) { return crt_split_launch(dsp, nsp, nb, crtc32, s); }, C_TRSM, 0});
                CrtJob* dj = ar.push(tj);
                const int nj = (int)tj.size();
                const CrtArgs ca = crt_args(dj, o32s, e32, 0, crtc32, p64b, (uint64_t)RG.p64_sets * nt * nb, pan_pairs, 1);
                cur->push_back({[=](cudaStream_t s) { return crt_gemm_launch(ca, nj, s); }, C_TRSM, 2.0 * fnb * fnb * fnb * nj});
            }
            fc.trsm += np * fnb * fnb * fnb;
            // ---- 5. panel out (K2): storage precision into the pool, comm precision in the panel slot
            cur->push_back({[=](cudaStream_t s) { return panel_out_launch(d_in, np, (int64_t)nb2, s); }, C_CONV, 0});
        }
        std::vector<char> have(nt, 0);  // panel slots holding L_mk on this GPU after step 5c
        for (auto& t : pin) have[(t.p64 - p64) / (ptrdiff_t)nb2] = 1;
        if (dist) {
            // ---- 5b. publish my L_mk (comm precision) for remote successors
            std::vector<PackItem> packs;
            std::vector<WaitItem> flags;  // (flag, value) pairs to set
            for (auto& x : xpub[k]) {
                const int m = x.m;
                if (m == k) continue;
                packs.push_back(PackItem{p64 + (size_t)m * nb2, sendslot(me, sp, m), C(m, k), A->st(m, k) == MP_FP16 ? xscale(m, k) : 0});
                flags.push_back(WaitItem{pubflag(me, sp, m), ST(k)});
            }
            if (!packs.empty()) {
                wait_send_free();
                PackItem* dp = ar.push(packs);
                const int npk = (int)packs.size();
                cur_push(Op{[=](cudaStream_t s) { return pack_launch(dp, npk, (int64_t)nb2, s); }, C_CONV, 0});
                for (auto& f : flags) {
                    uint64_t* fp = (uint64_t*)f.flag;
                    const uint64_t v = f.target;
                    cur_push(Op{[=](cudaStream_t s) { return set_flag_launch(fp, v, s); }, C_CONV, 0});
                }
            }
            // ---- 5c. pull the remote L_mk my tiles need: peer payload -> FP64 panel slot
            std::vector<WaitItem> waits;
            std::vector<PullItem> pulls;
            for (auto& x : xpull[k]) {
                const int m = x.m;
                if (m == k) continue;
                const int o = x.peer;
                PullItem it{sendslot(o, sp, m), pubflag(o, sp, m), ST(k), p64 + (size_t)m * nb2, C(m, k),
                            A->st(m, k) == MP_FP16 ? xscale(m, k) : 0};
                waits.push_back(WaitItem{it.flag, it.target});
                pulls.push_back(it);
                have[m] = 1;
            }
            push_wait(waits);
            if (!pulls.empty()) {
                PullItem* dp = ar.push(pulls);
                const int npl = (int)pulls.size();
                cur_push(Op{[=](cudaStream_t s) { return pull_launch(dp, npl, (int64_t)nb2, s); }, C_CONV, 0});
            }
            uint64_t* df = doneflag(me, sp);
            const uint64_t dv = ST(k);
            cur_push(Op{[=](cudaStream_t s) { return set_flag_launch(df, dv, s); }, C_CONV, 0});
        }
        // ---- 5e. operand formats of panel k for this GPU's successors (single-buffered: they run on
        //      the update stream after update k-1 released the caches)
        cur = &fmt[k];
        {
            std::vector<Split16Item> s16;
            std::vector<Tf32Item> t32s;
            std::vector<CrtSplitItem> c16;
            for (int m = k + 1; m < nt; ++m) {
                if (!have[m]) continue;
                bool n16, n32, n64, n16h;
                needs(k, m, n16, n32, n64, n16h);
                const double* src = p64 + (size_t)m * nb2;
                const bool lo3 = n32 && E.f32 == MP_F32_3XFP16;
                if (E.h16 && (lo3 || (n16 && E.tc16) || (n16h && h16s)))
                    s16.push_back(Split16Item{src, h16hi + (size_t)m * nb2, lo3 ? h16lo + (size_t)m * nb2 : nullptr,
                                              e16 + (size_t)m * nb, n16h && h16s ? h16s + (size_t)m * nb2 : nullptr});
                if (n32 && E.f32 == MP_F32_3XTF32) t32s.push_back(Tf32Item{src, phi + (size_t)m * nb2, plo + (size_t)m * nb2});
                if (n64 && E.crt) c16.push_back(CrtSplitItem{src, ozs + (size_t)m * nb2, oze + (size_t)m * nb, plane});
            }
            if (!s16.empty()) {
                Split16Item* di = ar.push(s16);
                const int ns = (int)s16.size();
                cur_push(Op{[=](cudaStream_t s) { return split16_launch(di, ns, nb, s); }, C_CONV, 0});
            }
            if (!t32s.empty()) {
                Tf32Item* di = ar.push(t32s);
                const int ns = (int)t32s.size();
                cur_push(Op{[=](cudaStream_t s) { return tf32_split_launch(di, ns, (int64_t)nb2, s); }, C_CONV, 0});
            }
            if (!c16.empty()) {
                CrtSplitItem* dsp = ar.push(c16);
                const int nsp = (int)c16.size();
                cur_push(Op{[=](cudaStream_t s) { return crt_split_launch(dsp, nsp, nb, crtc, s); }, C_CONV, 0});
            }
        }
        // ---- 6. trailing update: SYRK + GEMM grouped by kernel(m,n); the tiles of
        //      column k+1 (next) are emitted separately so panel k+1 can start as soon as they are done
        for (int part = 0; part < 2; ++part) {
            cur = part == 0 ? &nxt[k] : &rst[k];
            std::vector<GemmJob> syrk, g64, g32, g16;
            std::vector<CrtJob> csyrk, c64;
            std::vector<TcJob> t32, t16, t16h;
            for (int m = k + 1; m < nt; ++m) {
                if (A->mine(m, m) && ((m == k + 1) == (part == 0))) {
                    if (E.crt) csyrk.push_back(CrtJob{m, m, A->tile(m, m)});
                    else syrk.push_back(GemmJob{p64 + (size_t)m * nb2, p64 + (size_t)m * nb2, A->tile(m, m)});
                    fc.upd[MP_FP64] += fnb * fnb * fnb;
                }
                for (int n = k + 1; n < m; ++n) {
                    if (!A->mine(m, n) || ((n == k + 1) != (part == 0))) continue;
                    const int p = K(m, n);
                    fc.upd[p] += 2.0 * fnb * fnb * fnb;
                    if (p == MP_FP16H) {  // pure FP16 (four-level maps): tcgen05 with an F16 accumulator
                        t16h.push_back(TcJob{m, n, A->tile(m, n), 0, 0});
                    } else if (p == MP_FP64) {
                        if (E.crt) c64.push_back(CrtJob{m, n, A->tile(m, n)});
                        else g64.push_back(GemmJob{p64 + (size_t)m * nb2, p64 + (size_t)n * nb2, A->tile(m, n)});
                    } else if (p == MP_FP32 ? E.f32 != MP_F32_DMMA : E.tc16) {
                        (p == MP_FP32 ? t32 : t16).push_back(TcJob{m, n, A->tile(m, n), A->ts(m, n), 0});
                    } else {
                        (p == MP_FP32 ? g32 : g16).push_back(GemmJob{p64 + (size_t)m * nb2, p64 + (size_t)n * nb2, A->tile(m, n)});
                    }
                }
            }
            const double f3 = fnb * fnb * fnb;
            for (int lower = 1; lower >= 0; --lower) {  // FP64 class on INT8 tensor cores (CRT)
                std::vector<CrtJob>& cj = lower ? csyrk : c64;
                if (cj.empty()) continue;
                CrtJob* dj = ar.push(cj);
                const int nj = (int)cj.size();
                // upd_pairs of the SM/2 CTA pairs: SMs stay free for the panel stream's POTRF/TRSM (lookahead)
                const CrtArgs ca = crt_args(dj, ozs, oze, lower, crtc, cpool64, crows64, upd_pairs, 0);
                cur_push(Op{[=](cudaStream_t s) { return crt_gemm_launch(ca, nj, s); }, C_UPD64, (lower ? f3 : 2 * f3) * nj});
            }
            gemm(syrk, nb, nb, nb, nb, nb, nb, 1, -1.0, 1.0, P64, false, C_UPD64, f3);
            gemm(g64, nb, nb, nb, nb, nb, nb, 0, -1.0, 1.0, P64, false, C_UPD64, 2 * f3);
            gemm(g32, nb, nb, nb, nb, nb, nb, 0, -1.0, 1.0, P32, true, C_UPD32, 2 * f3);
            gemm(g16, nb, nb, nb, nb, nb, nb, 0, -1.0, 1.0, P16, true, C_UPD16, 2 * f3);
            if (!t32.empty()) {
                TcJob* dj = ar.push(t32);
                const int nj = (int)t32.size();
                TcArgs ta{};
                ta.jobs = dj;
                ta.nb = nb;
                ta.nt = nt;
                ta.cbase = cpool;
                ta.crows = crows;
                if (E.f32 == MP_F32_3XFP16) {
                    ta.h16hi = h16hi;
                    ta.h16lo = h16lo;
                    ta.e16 = e16;
                    ta.persistent = h->cfg.f16x3_persistent;
                    ta.pairs = upd_pairs;  // lookahead: leave SMs to the panel stream (0: all)
                    cur->push_back({[=](cudaStream_t s) { return tc_gemm_f16x3_launch(ta, nj, s); }, C_UPD32, 2 * f3 * nj});
                } else {
                    ta.hi = phi;
                    ta.lo = plo;
                    cur->push_back({[=](cudaStream_t s) { return tc_gemm_tf32x3_launch(ta, nj, s); }, C_UPD32, 2 * f3 * nj});
                }
            }
            if (!t16.empty()) {
                TcJob* dj = ar.push(t16);
                const int nj = (int)t16.size();
                TcArgs ta{};
                ta.jobs = dj;
                ta.nb = nb;
                ta.nt = nt;
                ta.h16hi = h16hi;
                ta.e16 = e16;
                ta.cbase = cpool;
                ta.crows = crows;
                if (E.s16) {  // FP16 storage class: FP16 C tiles (FP16 view of the pool)
                    ta.c16 = 1;
                    ta.crows = (RG.total - RG.pool) / ((size_t)nb * 2);
                }
                cur->push_back({[=](cudaStream_t s) { return tc_gemm_f16_launch(ta, nj, s); }, C_UPD16, 2 * f3 * nj});
            }
            if (!t16h.empty()) {
                TcJob* dj = ar.push(t16h);
                const int nj = (int)t16h.size();
                TcArgs ta{};
                ta.jobs = dj;
                ta.nb = nb;
                ta.nt = nt;
                ta.h16hi = h16s;
                ta.e16 = e16;
                ta.cbase = cpool;
                ta.crows = crows;
                cur->push_back({[=](cudaStream_t s) { return tc_gemm_f16h_launch(ta, nj, s); }, C_UPD16, 2 * f3 * nj});
            }
        }  // part
    }
    // ---- assemble the schedule
    if (!la) {
        for (int k = 0; k < nt; ++k)
            for (auto* v : {&pan[k], &fmt[k], &nxt[k], &rst[k]})
                for (auto& o : *v) ops.push_back(std::move(o));
        return MP_OK;
    }
    // events: 0 = start; 1 + 2k = panel k done; 2 + 2k = column k+1 updated
    auto on = [&](std::vector<Op>& v, int stream) {
        for (auto& o : v) {
            o.stream = stream;
            ops.push_back(std::move(o));
        }
    };
    ops.push_back(op_record(0, 0));
    ops.push_back(op_wait(1, 0));
    on(pan[0], 1);
    ops.push_back(op_record(1, 1));
    for (int k = 0; k + 1 < nt; ++k) {
        ops.push_back(op_wait(0, 1 + 2 * k));
        on(fmt[k], 0);  // panel k's operand formats: the caches were released by update k-1
        on(nxt[k], 0);
        ops.push_back(op_record(0, 2 + 2 * k));
        ops.push_back(op_wait(1, 2 + 2 * k));
        on(pan[k + 1], 1);
        ops.push_back(op_record(1, 1 + 2 * (k + 1)));
        on(rst[k], 0);
    }
    ops.push_back(op_wait(0, 1 + 2 * (nt - 1)));
    return MP_OK;
}

static mp_status potrf_run(mp_handle* h, mp_matrix* A, const uint8_t* km, const uint8_t* cm, int64_t* info,
                           FlopCount* fc_out) {
    if (!h || !A || !km || !cm) return MP_ERR_ARG;
    if (h->broken) FAIL(h, MP_ERR_STATE, "handle unusable after an earlier CUDA failure");
    if (!A->bound || !A->generated) FAIL(h, MP_ERR_STATE, "matrix not generated");
    if (h->nranks > 1 && !A->comm.connected) FAIL(h, MP_ERR_COMM, "multi-rank matrix not connected");
    const int nt = A->nt;
    for (int k = 0; k < nt; ++k)
        for (int m = k; m < nt; ++m) {
            const size_t i = (size_t)m * nt + k;
            if (km[i] > MP_FP16H || cm[i] > MP_FP16 || (m == k && km[i] != MP_FP64))
                FAIL(h, MP_ERR_ARG, "bad map entry at (%d,%d)", m, k);
            if (km[i] == MP_FP16H && !A->R.h16s)
                FAIL(h, MP_ERR_UNSUPPORTED, "pure-FP16 tile (%d,%d): needs the tcgen05 FP16 engine and a matrix laid out "
                     "for a four-level map (mp_eval with MP_MAP_ADAPTIVE4 / MP_MAP_USER)", m, k);
            if (m > k && A->st(m, k) != (km[i] == MP_FP64 ? MP_FP64 : MP_FP32) &&
                !(A->st(m, k) == MP_FP16 && km[i] == MP_FP16 && h->cfg.fp16_storage))
                FAIL(h, MP_ERR_ARG, "kernel map inconsistent with the bound storage map at (%d,%d)", m, k);
            if (m > k && cm[i] < A->st(m, k)) FAIL(h, MP_ERR_ARG, "comm precision above storage at (%d,%d)", m, k);
        }
    const int big = INT_MAX;
    CK(h, cudaMemcpyAsync(h->d_info, &big, sizeof(int), cudaMemcpyHostToDevice, h->stream));
    if (A->R.crtflags) CK(h, cudaMemsetAsync(A->ws + A->R.crtflags, 0, (size_t)crt_scratch_slots() * sizeof(int), h->stream));
    if (A->R.crtctr) CK(h, cudaMemsetAsync(A->ws + A->R.crtctr, 0, crt_counters(A->nt) * sizeof(int), h->stream));
    Arena ar;
    ar.dev_base = A->ws + A->R.ctrl;
    std::vector<Op> ops;
    FlopCount fc;
    const uint64_t epoch = ++A->comm.epoch;
    if (mp_status s = plan_potrf(h, A, km, cm, ar, ops, fc, epoch)) return s;
    if (mp_status s = run_plan(h, A, ar, ops)) return s;
    int hinfo = 0;
    CK(h, cudaMemcpyAsync(&hinfo, h->d_info, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    CK(h, cudaStreamSynchronize(h->stream));
    A->kmap.assign(km, km + (size_t)nt * nt);
    A->cmap.assign(cm, cm + (size_t)nt * nt);
    if (fc_out) *fc_out = fc;
    if (hinfo != big) {
        if (info) *info = hinfo;
        A->factored = false;
        FAIL(h, MP_ERR_NOT_SPD, "not positive definite at column %d", hinfo);
    }
    if (info) *info = 0;
    A->factored = true;
    return MP_OK;
}

mp_status mp_tile_potrf(mp_handle* h, mp_matrix* A, const uint8_t* kernel_prec, const uint8_t* comm_prec,
                        int64_t* info) {
    return potrf_run(h, A, kernel_prec, comm_prec, info, nullptr);
}

// ------------------------------------------------------------------ (4) log-likelihood
// Multi-rank forward solve (right-looking, 2D block-cyclic): rank (p, q) accumulates
// racc_m = -sum_{own (m,j)} L_mj y_j; at step k the ranks of process row k mod P publish racc_k,
// owner(k,k) forms r_k = z_k + sum_r racc_k^(r) (rank order), solves y_k = L_kk^{-1} r_k and
// publishes y_k; the ranks of process column k mod Q read y_k straight from the owner's memory in
// their GEMV.  log-determinant and y^T y partials are all-gathered and summed in rank order.
static mp_status loglik_dist(mp_handle* h, mp_matrix* A, const double* d_z, double* loglik, double* logdet,
                             double* quad) {
    if (!A->comm.connected) FAIL(h, MP_ERR_COMM, "multi-rank matrix not connected");
    Comm& X = A->comm;
    const int nt = A->nt, nb = A->nb, P = h->P, Q = h->Q, me = h->rank;
    const int myp = me / Q, myq = me % Q;
    const int64_t n = A->n;
    const uint64_t epoch = ++X.epoch;
    auto ST = [&](int step) -> uint64_t { return (epoch << 24) + (uint64_t)(step + 2); };
    if (mp_status st = dist_barrier(h, A, ST(-1))) return st;
    double* racc = A->at<double>(A->R.vec_r);
    double* zpad = A->at<double>(A->R.vec_y);
    double* part = A->at<double>(A->R.partials);
    CK(h, cudaMemsetAsync(racc, 0, (size_t)nt * nb * 8, h->stream));
    CK(h, cudaMemsetAsync(zpad, 0, (size_t)nt * nb * 8, h->stream));
    CK(h, cudaMemcpyAsync(zpad, d_z, (size_t)n * 8, cudaMemcpyDeviceToDevice, h->stream));
    auto yslot = [&](int r, int k) { return (double*)(X.peer[r] + X.yv) + (size_t)k * nb; };
    auto yflag = [&](int r, int k) { return (uint64_t*)(X.peer[r] + X.yflag) + k; };
    auto pslot = [&](int r, int k) { return (double*)(X.peer[r] + X.part) + (size_t)k * nb; };
    auto pflag = [&](int r, int k) { return (uint64_t*)(X.peer[r] + X.pflag) + k; };
    Arena ar;
    ar.dev_base = A->ws + A->R.ctrl;
    std::vector<Op> ops;
    std::vector<const double*> diag;
    std::vector<int> nreal;
    auto wait_op = [&](std::vector<WaitItem> w) {
        if (w.empty()) return;
        WaitItem* dw = ar.push(w);
        const int nw = (int)w.size();
        ops.push_back({[=](cudaStream_t s) { return wait_flags_launch(dw, nw, s); }, C_SOLVE, 0});
    };
    for (int k = 0; k < nt; ++k) {
        if (myp == k % P) {  // publish my partial of row k
            double* src = racc + (size_t)k * nb;
            double* dst = pslot(me, k);
            uint64_t* f = pflag(me, k);
            const uint64_t v = ST(k);
            ops.push_back({[=](cudaStream_t s) { return cudaMemcpyAsync(dst, src, (size_t)nb * 8, cudaMemcpyDeviceToDevice, s); },
                           C_SOLVE, 0});
            ops.push_back({[=](cudaStream_t s) { return set_flag_launch(f, v, s); }, C_SOLVE, 0});
        }
        const int o = A->owner(k, k);
        if (o == me) {
            std::vector<WaitItem> w;
            GatherItem g{};
            g.base = zpad + (size_t)k * nb;
            g.n = 0;
            for (int q = 0; q < Q; ++q) {
                const int r = (k % P) * Q + q;
                if (r != me) w.push_back(WaitItem{pflag(r, k), ST(k)});
                g.src[g.n++] = pslot(r, k);
            }
            wait_op(w);
            double* tmp = (double*)(X.base + X.tmp);
            g.dst = tmp;
            ops.push_back({[=](cudaStream_t s) { return gather_add_launch(g, nb, s); }, C_SOLVE, 0});
            const double* Lkk = (const double*)A->tile(k, k);
            double* yk = yslot(me, k);
            ops.push_back({[=](cudaStream_t s) { return trsv_tile_launch(Lkk, nb, tmp, yk, s); }, C_SOLVE, 0});
            uint64_t* f = yflag(me, k);
            const uint64_t v = ST(k);
            ops.push_back({[=](cudaStream_t s) { return set_flag_launch(f, v, s); }, C_SOLVE, 0});
            diag.push_back(Lkk);
            nreal.push_back((int)std::min<int64_t>(nb, n - (int64_t)k * nb));
        }
        if (myq == k % Q) {
            std::vector<GemvTile> gv;
            for (int m = k + 1; m < nt; ++m)
                if (A->mine(m, k)) gv.push_back(GemvTile{A->tile(m, k), A->st(m, k), A->ts(m, k), racc + (size_t)m * nb});
            if (!gv.empty()) {
                if (o != me) wait_op({WaitItem{yflag(o, k), ST(k)}});
                GemvTile* dg = ar.push(gv);
                const int ng = (int)gv.size();
                const double* yk = yslot(o, k);  // peer memory when o != me (NVLink / IPC load)
                ops.push_back({[=](cudaStream_t s) { return gemv_sub_launch(dg, ng, yk, nb, s); }, C_SOLVE, 0});
            }
        }
    }
    // local partials: log diag of my diagonal tiles, y^T y of my y_k (slots of other k are unused)
    const int nd = (int)diag.size();
    std::vector<int> myk;
    for (int k = 0; k < nt; ++k)
        if (A->owner(k, k) == me) myk.push_back(k);
    if (nd) {
        const double* const* d_diag = ar.push(diag);
        const int* d_nreal = ar.push(nreal);
        ops.push_back({[=](cudaStream_t s) { return logdiag_launch(d_diag, d_nreal, nd, nb, part, s); }, C_SOLVE, 0});
        double* ybase = yslot(me, 0);
        const int ntt = nt;
        ops.push_back({[=](cudaStream_t s) { return sumsq_chunks_launch(ybase, (int64_t)ntt * nb, nb, part + nd, s); },
                       C_SOLVE, 0});
    }
    if (mp_status st = run_plan(h, A, ar, ops)) return st;
    std::vector<double> hp(nd + nt, 0.0);
    if (nd) CK(h, cudaMemcpyAsync(hp.data(), part, hp.size() * 8, cudaMemcpyDeviceToHost, h->stream));
    CK(h, cudaStreamSynchronize(h->stream));
    double sc[2] = {0.0, 0.0};
    for (int i = 0; i < nd; ++i) sc[0] += hp[i];
    for (int k : myk) sc[1] += hp[nd + k];
    CK(h, cudaMemcpy(X.base + X.scal, sc, sizeof sc, cudaMemcpyHostToDevice));
    CK(h, set_flag_launch((uint64_t*)(X.base + X.sflag), ST(nt), h->stream));
    CK(h, cudaStreamSynchronize(h->stream));
    double ld = 0.0, q = 0.0;
    for (int r = 0; r < h->nranks; ++r) {
        double v[2];
        if (r != me) {
            if (mp_status st = host_wait_stamp(h, (const uint64_t*)(X.peer[r] + X.sflag), ST(nt))) return st;
            CK(h, cudaMemcpy(v, X.peer[r] + X.scal, sizeof v, cudaMemcpyDeviceToHost));
        } else {
            v[0] = sc[0];
            v[1] = sc[1];
        }
        ld += v[0];
        q += v[1];
    }
    ld *= 2.0;
    // closing barrier: nobody reuses the exchange area while a peer still reads it
    if (mp_status st = dist_barrier(h, A, ST(nt + 1))) return st;
    const double ll = -0.5 * (double)n * std::log(2.0 * M_PI) - 0.5 * ld - 0.5 * q;
    if (loglik) *loglik = ll;
    if (logdet) *logdet = ld;
    if (quad) *quad = q;
    return MP_OK;
}

mp_status mp_loglik(mp_handle* h, const mp_matrix* Lc, const double* d_z, double* loglik, double* logdet,
                    double* quad) {
    mp_matrix* A = const_cast<mp_matrix*>(Lc);
    if (!h || !A || !d_z) return MP_ERR_ARG;
    if (h->broken) FAIL(h, MP_ERR_STATE, "handle unusable after an earlier CUDA failure");
    if (!A->factored) FAIL(h, MP_ERR_STATE, "matrix not factored");
    if (h->nranks > 1) return loglik_dist(h, A, d_z, loglik, logdet, quad);
    const int nt = A->nt, nb = A->nb;
    const int64_t n = A->n;
    double* r = A->at<double>(A->R.vec_r);
    double* y = A->at<double>(A->R.vec_y);
    double* part = A->at<double>(A->R.partials);
    const int chunk = 4096;
    const int nchunks = (int)((n + chunk - 1) / chunk);
    CK(h, cudaMemsetAsync(r, 0, (size_t)nt * nb * 8, h->stream));
    CK(h, cudaMemcpyAsync(r, d_z, (size_t)n * 8, cudaMemcpyDeviceToDevice, h->stream));
    Arena ar;
    ar.dev_base = A->ws + A->R.ctrl;
    std::vector<Op> ops;
    std::vector<const double*> diag;
    std::vector<int> nreal;
    for (int k = 0; k < nt; ++k) diag.push_back((const double*)A->tile(k, k));
    // 128-block inverses of every diagonal tile in one launch, then a blocked TRSV per tile
    double* wdiag = A->at<double>(A->R.wdiag);
    const size_t wstride = (size_t)ceil_div(nb, POTRF_IB) * POTRF_IB * POTRF_IB;
    {
        const double* const* d_all = ar.push(diag);
        ops.push_back({[=](cudaStream_t s) { return trtri_batch_launch(d_all, nt, nb, wdiag, s); }, C_SOLVE, 0});
    }
    for (int k = 0; k < nt; ++k) {
        const double* Lkk = diag[k];
        nreal.push_back((int)std::min<int64_t>(nb, n - (int64_t)k * nb));
        double* rk = r + (size_t)k * nb;
        double* yk = y + (size_t)k * nb;
        const double* Wk = wdiag + (size_t)k * wstride;
        Op op{[=](cudaStream_t s) { return trsv_blocked_launch(Lkk, nb, Wk, rk, yk, s); }, C_SOLVE, 0};
        op.nlaunch = 2 * ceil_div(nb, POTRF_IB) - 1;
        ops.push_back(std::move(op));
        std::vector<GemvTile> gv;
        for (int m = k + 1; m < nt; ++m) gv.push_back(GemvTile{A->tile(m, k), A->st(m, k), A->ts(m, k), r + (size_t)m * nb});
        if (!gv.empty()) {
            GemvTile* dg = ar.push(gv);
            const int ng = (int)gv.size();
            ops.push_back({[=](cudaStream_t s) { return gemv_sub_launch(dg, ng, yk, nb, s); }, C_SOLVE, 0});
        }
    }
    const double* const* d_diag = ar.push(diag);
    const int* d_nreal = ar.push(nreal);
    ops.push_back({[=](cudaStream_t s) { return logdiag_launch(d_diag, d_nreal, nt, nb, part, s); }, C_SOLVE, 0});
    ops.push_back({[=](cudaStream_t s) { return sumsq_chunks_launch(y, n, chunk, part + nt, s); }, C_SOLVE, 0});
    if (mp_status s = run_plan(h, A, ar, ops)) return s;
    std::vector<double> hp(nt + nchunks);
    CK(h, cudaMemcpyAsync(hp.data(), part, hp.size() * 8, cudaMemcpyDeviceToHost, h->stream));
    CK(h, cudaStreamSynchronize(h->stream));
    double ld = 0.0, q = 0.0;
    for (int k = 0; k < nt; ++k) ld += hp[k];
    ld *= 2.0;
    for (int c = 0; c < nchunks; ++c) q += hp[nt + c];
    const double ll = -0.5 * (double)n * std::log(2.0 * M_PI) - 0.5 * ld - 0.5 * q;
    if (loglik) *loglik = ll;
    if (logdet) *logdet = ld;
    if (quad) *quad = q;
    return MP_OK;
}

mp_status mp_gp_sample(mp_handle* h, const mp_matrix* Lc, const double* d_e, double* d_z) {
    mp_matrix* A = const_cast<mp_matrix*>(Lc);
    if (!h || !A || !d_e || !d_z) return MP_ERR_ARG;
    if (!A->factored) FAIL(h, MP_ERR_STATE, "matrix not factored");
    if (h->nranks > 1) FAIL(h, MP_ERR_UNSUPPORTED, "mp_gp_sample is single-rank");
    const int nt = A->nt, nb = A->nb;
    const int64_t n = A->n;
    double* r = A->at<double>(A->R.vec_r);
    double* ye = A->at<double>(A->R.vec_y);
    CK(h, cudaMemsetAsync(r, 0, (size_t)nt * nb * 8, h->stream));
    CK(h, cudaMemsetAsync(ye, 0, (size_t)nt * nb * 8, h->stream));
    CK(h, cudaMemcpyAsync(ye, d_e, (size_t)n * 8, cudaMemcpyDeviceToDevice, h->stream));
    Arena ar;
    ar.dev_base = A->ws + A->R.ctrl;
    std::vector<Op> ops;
    // the GEMV kernel accumulates r_m -= L_mk e_k, i.e. r = -L e; the sign is flipped on the way out
    for (int k = 0; k < nt; ++k) {
        std::vector<GemvTile> gv;
        for (int m = k; m < nt; ++m) gv.push_back(GemvTile{A->tile(m, k), A->st(m, k), A->ts(m, k), r + (size_t)m * nb});
        GemvTile* dg = ar.push(gv);
        const int ng = (int)gv.size();
        const double* yk = ye + (size_t)k * nb;
        ops.push_back({[=](cudaStream_t s) { return gemv_sub_launch(dg, ng, yk, nb, s); }, C_SOLVE, 0});
    }
    // r = -(L e): negated into d_z on the device
    ops.push_back({[=](cudaStream_t s) { return scale_vec_launch(d_z, r, n, -1.0, s); }, C_SOLVE, 0});
    if (mp_status st = run_plan(h, A, ar, ops)) return st;
    CK(h, cudaStreamSynchronize(h->stream));
    return MP_OK;
}

// ------------------------------------------------------------------ one evaluation
static void band_kernel_map(int nt, const double* s, double u_req, const double* eps, std::vector<uint8_t>& km) {
    // reading C21: two-level rule, then the narrowest band holding every FP64 tile
    std::vector<uint8_t> two((size_t)nt * nt);
    const double e2[3] = {eps ? eps[0] : std::ldexp(1.0, -52), eps ? eps[1] : std::ldexp(1.0, -23), HUGE_VAL};
    mp_precision_map(nt, s, u_req, e2, MP_COMM_TTC, two.data(), nullptr, nullptr);
    int b = 1;
    for (int k = 0; k < nt; ++k)
        for (int m = k + 1; m < nt; ++m)
            if (two[(size_t)m * nt + k] == MP_FP64) b = std::max(b, m - k + 1);
    km.assign((size_t)nt * nt, 255);
    for (int k = 0; k < nt; ++k)
        for (int m = k; m < nt; ++m) km[(size_t)m * nt + k] = (m - k < b) ? MP_FP64 : MP_FP32;
}

mp_status mp_eval(mp_handle* h, mp_matrix* A, const double* x, const double* y, const double* z, int inputs_on_host,
                  const double theta[3], double u_req, const double* eps, mp_comm_policy policy, mp_map_mode mode,
                  const uint8_t* user_kernel_prec, mp_eval_report* rep) {
    if (!h || !A || !x || !y || !z || !rep) return MP_ERR_ARG;
    if (!A->bound) FAIL(h, MP_ERR_STATE, "bind or attach a workspace first (mp_matrix_bind / mp_matrix_attach)");
    if (mp_status s = check_theta(h, theta, A->cov)) return s;
    memset(rep, 0, sizeof *rep);
    const int nt = A->nt;
    const int64_t n = A->n;
    const size_t NN = (size_t)nt * nt;
    const int64_t l0 = h->launches;
    cudaEvent_t* ev = h->ev;
    CK(h, cudaEventRecord(ev[0], h->stream));
    // inputs: x, y, z live in the map-independent `inputs` region for the whole evaluation
    const size_t nvec = (size_t)nt * A->nb;
    double* xyz = A->at<double>(A->R.inputs);
    const cudaMemcpyKind kind = inputs_on_host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
    CK(h, cudaMemcpyAsync(xyz, x, n * 8, kind, h->stream));
    CK(h, cudaMemcpyAsync(xyz + nvec, y, n * 8, kind, h->stream));
    CK(h, cudaMemcpyAsync(xyz + 2 * nvec, z, n * 8, kind, h->stream));
    const double* dx = xyz;
    const double* dy = xyz + nvec;
    const double* dz = xyz + 2 * nvec;
    void* ws = A->ws;
    const size_t wsb = A->ws_bytes;
    std::vector<double> s(NN, 0.0);
    std::vector<uint8_t> km(NN, 255), sm(NN, 255), cm(NN, 255);
    if (mode == MP_MAP_ADAPTIVE || mode == MP_MAP_ADAPTIVE4 || mode == MP_MAP_BAND) {
        if (mp_status st = mp_matern_gen(h, A, dx, dy, theta, nullptr, s.data())) return st;
    }
    CK(h, cudaEventRecord(ev[1], h->stream));
    mp_status st = MP_OK;
    switch (mode) {
        case MP_MAP_ADAPTIVE:
            st = mp_precision_map(nt, s.data(), u_req, eps, policy, km.data(), sm.data(), cm.data());
            break;
        case MP_MAP_ADAPTIVE4:  // four levels: eps = 4 entries or NULL
            st = mp_precision_map4(nt, s.data(), u_req, eps, policy, km.data(), sm.data(), cm.data());
            break;
        case MP_MAP_BAND:
            band_kernel_map(nt, s.data(), u_req, eps, km);
            st = mp_precision_map(nt, nullptr, u_req, eps, policy, km.data(), sm.data(), cm.data());
            break;
        case MP_MAP_FP64:
        case MP_MAP_EXTREME:
            for (int k = 0; k < nt; ++k)
                for (int m = k; m < nt; ++m)
                    km[(size_t)m * nt + k] = (m == k || mode == MP_MAP_FP64) ? MP_FP64 : MP_FP16;
            st = mp_precision_map(nt, nullptr, u_req, eps, policy, km.data(), sm.data(), cm.data());
            break;
        case MP_MAP_USER:
            if (!user_kernel_prec) return MP_ERR_ARG;
            km.assign(user_kernel_prec, user_kernel_prec + NN);
            st = mp_precision_map4(nt, nullptr, u_req, eps, policy, km.data(), sm.data(), cm.data());
            break;
        default:
            return MP_ERR_ARG;
    }
    if (st) FAIL(h, st, "precision map failed");
    if (h->cfg.fp16_storage)  // FP16 storage class: FP16-class tiles stored in FP16, and
        for (int k = 0; k < nt; ++k)  // they travel in FP16 (Alg. 2 caps comm at storage)
            for (int m = k + 1; m < nt; ++m) {
                const size_t i = (size_t)m * nt + k;
                if (km[i] == MP_FP16) sm[i] = cm[i] = MP_FP16;
            }
    A->h16h = false;  // the pure-FP16 operand planes only for a map that has such tiles
    for (int k = 0; k < nt; ++k)
        for (int m = k + 1; m < nt; ++m) A->h16h |= km[(size_t)m * nt + k] == MP_FP16H;
    {  // the workspace this map needs (tiles in storage precision + the map-independent regions)
        const size_t need = layout(A, sm.data()).total;
        rep->workspace_bytes = need;
        if (need > wsb) FAIL(h, MP_ERR_NOMEM, "workspace %zu bytes < %zu needed by this evaluation's map", wsb, need);
    }
    if (mp_status b = mp_matrix_bind(A, sm.data(), ws, wsb)) return b;
    if (mp_status g = mp_matern_gen(h, A, dx, dy, theta, sm.data(), nullptr)) return g;
    CK(h, cudaEventRecord(ev[2], h->stream));
    FlopCount fc;
    int64_t info = 0;
    mp_status pst = potrf_run(h, A, km.data(), cm.data(), &info, &fc);
    CK(h, cudaEventRecord(ev[3], h->stream));
    rep->info = info;
    for (int k = 0; k < nt; ++k)
        for (int m = k + 1; m < nt; ++m) {
            const size_t i = (size_t)m * nt + k;
            if (km[i] == MP_FP16H) rep->tiles_fp16h++;
            else rep->tiles[km[i]]++;
            if (cm[i] > sm[i]) rep->stc_tiles++;
        }
    for (int c = 0; c < 3; ++c) rep->flops_update[c] = fc.upd[c];
    rep->flops_update_fp16h = fc.upd[MP_FP16H];
    rep->flops_potrf = fc.potrf + fc.trsm;
    if (pst == MP_ERR_NOT_SPD) {
        rep->loglik = -HUGE_VAL;
        rep->gpu_launches = h->launches - l0;
        return pst;
    }
    if (pst) return pst;
    if (mp_status l = mp_loglik(h, A, dz, &rep->loglik, &rep->logdet, &rep->quad)) return l;
    CK(h, cudaEventRecord(ev[4], h->stream));
    CK(h, cudaEventSynchronize(ev[4]));
    float t01, t12, t23, t34, t04;
    cudaEventElapsedTime(&t01, ev[0], ev[1]);
    cudaEventElapsedTime(&t12, ev[1], ev[2]);
    cudaEventElapsedTime(&t23, ev[2], ev[3]);
    cudaEventElapsedTime(&t34, ev[3], ev[4]);
    cudaEventElapsedTime(&t04, ev[0], ev[4]);
    rep->t_map_ms = 0;
    rep->t_gen_ms = t01 + t12;
    rep->t_potrf_ms = t23;
    rep->t_solve_ms = t34;
    rep->t_total_ms = t04;
    rep->gpu_launches = h->launches - l0;
    return MP_OK;
}

}  // extern "C"
