/*
 * mpgeo.h — C ABI of the B200-native mixed-precision tile-Cholesky Matérn
 * log-likelihood library (libmpgeo.so).
 *
 * Method: Cao, Abdulah, Ltaief, Genton, Keyes, Bosilca, "Reducing Data Motion
 * and Energy Consumption of Geospatial Modeling Applications Using Automated
 * Precision Conversion", IEEE CLUSTER 2023.  Citations "P:<line>" refer to
 * lines of the paper text and the section/equation/algorithm they
 * fall in.
 *
 * One evaluation of the Gaussian log-likelihood (Eq. (1), §III-A)
 *     l(theta) = -(n/2) log(2 pi) - 1/2 log|Sigma(theta)| - 1/2 Z^T Sigma(theta)^{-1} Z
 * for the 2D Matérn covariance (§III-A) is the sequence
 *     mp_matern_gen (pass 1: tile norms)  ->  mp_precision_map  ->
 *     mp_matern_gen (pass 2: tiles in storage precision)  ->  mp_tile_potrf  ->  mp_loglik
 * or the single call mp_eval, which runs that sequence.
 *
 * Conventions (all entry points):
 *  - Every function returns mp_status; MP_OK = 0.  No C++ exception crosses the
 *    ABI.  mp_last_error(h) describes the last failure on a handle.
 *  - Device pointers ("d_" prefix) are borrowed: the caller (PyTorch in the
 *    Python binding) allocates and frees them.  Host pointers ("h_" or plain)
 *    are read or written only during the call.
 *  - Work is enqueued on the CUDA stream given to mp_init.  Calls that return
 *    host results (norms, info, scalars) synchronise that stream before return.
 *  - Tiles: square nb x nb, NT = ceil(n / nb); tile (m, k) covers rows
 *    [m nb, min(n, (m+1) nb)) and columns [k nb, min(n, (k+1) nb)) (P:258,
 *    "tile size 2048").  Only the lower triangle m >= k exists.  The ragged
 *    last tile is padded in storage to nb x nb: identity on the diagonal pad,
 *    zeros elsewhere (reading C18), which leaves l unchanged.
 *  - NT x NT host maps (uint8) and the tile-norm array (double) are ROW-major
 *    with index m * NT + k, lower triangle (m >= k) meaningful; other entries
 *    are ignored on input and set to 255 (maps) / 0 (norms) on output.
 *  - Precision codes: MP_FP64 = 0, MP_FP32 = 1, MP_FP16 = 2 (smaller = higher).
 *    MP_FP16 is the paper's FP16_32 class: FP16 operands, FP32 accumulation,
 *    FP32 storage; a storage map may hold MP_FP16 only with
 *    mp_config::fp16_storage (tiles stored as fp16(x 2^t), t from the pass-1 tile norms).
 *  - Multi-GPU: one process (and one handle) per GPU, P x Q process grid with
 *    P <= Q, 2D block-cyclic tile ownership
 *    owner(m, k) = (m mod P) * Q + (k mod Q).  Results returned to the host
 *    are identical on every rank.
 *  - Threading: a handle is not thread-safe; use one handle per thread.
 */
#ifndef MPGEO_H
#define MPGEO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    MP_OK = 0,
    MP_ERR_ARG = 1,          /* invalid argument: sizes, theta <= 0, nu outside (0, 20], bad map */
    MP_ERR_NOT_SPD = 2,      /* POTRF met a non-positive pivot; see `info` of mp_tile_potrf */
    MP_ERR_CUDA = 3,         /* a CUDA call failed; the handle is unusable afterwards */
    MP_ERR_COMM = 4,         /* peer exchange not connected / IPC mapping failed */
    MP_ERR_NOMEM = 5,        /* workspace too small for the requested layout */
    MP_ERR_UNSUPPORTED = 6,  /* configuration this build does not implement */
    MP_ERR_STATE = 7         /* call order violated (e.g. potrf before generation) */
} mp_status;

/* Precision classes (smaller value = higher precision).  MP_FP16 is the paper's FP16_32 (FP16 operands,
 * FP32 accumulation); MP_FP16H is the paper's pure FP16 class (FP16 operands AND FP16
 * accumulation, "A, B, C, and operation are all in FP16"), used only by four-level maps
 * (mp_precision_map4, MP_MAP_ADAPTIVE4).  Data (storage / communication) precisions
 * are FP64, FP32 and FP16 only: an FP16H tile is stored in FP32 and receives FP16 operands. */
typedef enum { MP_FP64 = 0, MP_FP32 = 1, MP_FP16 = 2, MP_FP16H = 3 } mp_prec;

/* u_low of the FP16_32 class in four-level maps.  The paper fixes it "experimentally" (citing
 * [23]: FP16_32 has a lower error bound than FP16) and prints no value; reading C7': the
 * ratio of the measured tile-GEMM errors of the FP16_32 and pure-FP16 classes on the application's
 * FP16-class tiles times FP16's machine epsilon 2^-10 (tools/fp16_eps.py; measured on the C2 factor:
 * median ratio 0.058 -> 5.7e-5, rounded UP to a power of two: 2^-14; profiles/r02/fp16h/fp16_eps.json). */
#define MP_EPS_FP16_32 (1.0 / 16384.0)

/* Communication-precision policy.
 * MP_COMM_TTC : target-task conversion — every tile travels in its storage
 *               precision and each consumer converts (the pre-existing scheme).
 * MP_COMM_AUTO: Algorithm 2 — sender-side conversion (STC) where all
 *               successors run at lower precision, TTC otherwise. */
typedef enum { MP_COMM_TTC = 0, MP_COMM_AUTO = 1 } mp_comm_policy;

/* How mp_eval chooses the kernel-precision map. */
typedef enum {
    MP_MAP_ADAPTIVE = 0,  /* tile-norm rule of P:117 at u_req (the paper's method) */
    MP_MAP_FP64 = 1,      /* everything FP64 (the "same code forced to all-FP64" baseline) */
    MP_MAP_BAND = 2,      /* FP64 band / FP32 outside (config 2; reading C21) */
    MP_MAP_EXTREME = 3,   /* FP64 diagonal, FP16 elsewhere (performance-only) */
    MP_MAP_USER = 4,      /* kernel_prec supplied by the caller */
    MP_MAP_ADAPTIVE4 = 5  /* four-level rule (FP64, FP32, FP16_32, FP16; mp_precision_map4) at u_req */
} mp_map_mode;

/* Covariance family of the generated matrix (§III-A). */
typedef enum {
    MP_COV_MATERN = 0,  /* sigma^2 2^(1-nu)/Gamma(nu) (h/beta)^nu K_nu(h/beta), theta = {sigma^2, beta, nu} */
    MP_COV_SQEXP = 1    /* sigma^2 exp(-h^2/beta), theta = {sigma^2, beta, unused} */
} mp_covariance;

typedef struct mp_handle mp_handle;
typedef struct mp_matrix mp_matrix;

/* Per-evaluation report filled by mp_eval. Times are device times (CUDA events on
 * the handle's stream) in milliseconds; flops are algorithmic counts. */
typedef struct {
    double loglik, logdet, quad;
    int64_t info;                 /* 0, or first non-positive pivot column (1-based) */
    double t_gen_ms, t_map_ms, t_potrf_ms, t_solve_ms, t_total_ms;
    double flops_potrf;           /* n^3/3 convention is left to the caller; this is the
                                     tile count: sum over executed kernels at nb^3 units */
    double flops_update[3];       /* GEMM+SYRK flops executed per precision class */
    int64_t tiles[3];             /* lower off-diagonal tiles per kernel precision */
    int64_t stc_tiles;            /* off-diagonal tiles whose comm precision < storage */
    int64_t gpu_launches;         /* kernels launched by this call */
    uint64_t workspace_bytes;     /* bytes this evaluation's map needs (set also on MP_ERR_NOMEM) */
    int64_t tiles_fp16h;          /* four-level maps: tiles of the pure-FP16 class (counted apart from tiles[2]) */
    double flops_update_fp16h;    /*   and their GEMM flops (apart from flops_update[2]) */
} mp_eval_report;

/* ---------------------------------------------------------------- configuration */

/* Engines of the precision classes (the arithmetic each class of Algorithm 1 runs on). */
typedef enum {
    MP_F64_CRT16 = 0,  /* FP64 class (DSYRK, FP64 GEMM) as 16 exact INT8 tcgen05 GEMMs + CRT
                          reconstruction (Ozaki scheme II): per-row normwise error
                          <= K 2^-(b+1) max_l|a_il| max_l|b_jl|, b = 56 at nb = 2048 (needs nb % 256 == 0,
                          else DMMA) */
    MP_F64_DMMA = 1    /* FP64 class on the FP64 DMMA tensor cores (native FP64, componentwise bound) */
} mp_fp64_engine;
typedef enum {
    MP_F32_3XFP16 = 0, /* FP32 class as 3xFP16 on tcgen05 kind::f16: row-scaled 11 + 11-bit hi/lo split,
                          FP32 chunk sums (reading C13c); per-row normwise bound (needs nb % 256 == 0) */
    MP_F32_3XTF32 = 1, /* FP32 class as 3xTF32 on tcgen05 kind::tf32 (reading C13) */
    MP_F32_DMMA = 2    /* FP32 class on DMMA with FP32-rounded operands and an FP32 C (reference engine) */
} mp_fp32_engine;

/* Handle configuration (read once by mp_init_config; every field has a default). */
typedef struct {
    int fp64_engine;      /* mp_fp64_engine, default MP_F64_CRT16 */
    int fp32_engine;      /* mp_fp32_engine, default MP_F32_3XFP16 */
    int fp16_tensor;      /* 1 (default): FP16 class on tcgen05 kind::f16 with row-scaled FP16 operands;
                             0: DMMA with FP16-rounded operands (reference engine) */
    int lookahead;        /* 1 (default): panel k+1 (POTRF, TRSM) on a high-priority stream overlaps the
                             trailing update of panel k; 0: one stream, strict Algorithm 1 order */
    int reserve_pairs;    /* CTA pairs the persistent update kernels leave to the panel stream (default 6) */
    int lowp_trsm_product;/* 1 (default, with MP_F64_CRT16): TRSM of FP32/FP16-class tiles as the FP32-class
                             product A_mk W^T, W = L~_kk^-1 (reading C12'); 0: FP64 substitution */
    int matern_table;     /* 1 (default): general nu through the per-evaluation Chebyshev table of the
                             correlation; 0: K_nu evaluated per entry */
    int f16x3_persistent; /* 1: persistent-CTA 3xFP16 kernel; 0 (default): one CTA pair per output tile */
    int crt_phase_lock;   /* 1 (default): CRT tiles start at the modulus pair the other CTAs are on */
    int fp16_storage;     /* 1: FP16 storage class: mp_eval stores FP16-class tiles in FP16 (one
                             power-of-two exponent per tile from its norm; 2 B instead of the paper's FP32)
                             and sends them in FP16; needs the tcgen05 FP16 engine.  0 (default): P:152 */
} mp_config;

/* Fill *cfg with the defaults above. */
void mp_config_default(mp_config* cfg);

/* ---------------------------------------------------------------- lifecycle */

/* A 128-byte communicator id (SURVEY §8(b) mp_get_unique_id): random bytes from the OS plus this
 * host's name and process id.  Rank 0 creates it and broadcasts it to the other ranks (e.g.
 * torch.distributed); every rank passes it to mp_init.  The multi-rank exchange (mp_matrix_comm_*)
 * writes it into the header of each rank's exchange area and mp_matrix_comm_connect refuses to map
 * a peer whose id differs (MP_ERR_COMM), so areas of two different jobs can never be mixed.  The
 * transport itself is CUDA IPC peer memory, which needs no other bootstrap. */
mp_status mp_get_unique_id(uint8_t id[128]);

/* Create a handle on CUDA `device` for `rank` of `nranks` (P * Q == nranks,
 * P <= Q, nranks <= 8).  `id`: the communicator id of mp_get_unique_id (required when nranks > 1,
 * may be NULL for one rank).  `cuda_stream` is a cudaStream_t (NULL = a stream created and owned by
 * the handle).  `cfg` may be NULL (defaults).  *h receives the handle.  Multi-rank matrices exchange
 * panel tiles through peer memory: see mp_matrix_comm_export / mp_matrix_comm_connect. */
mp_status mp_init_config(int device, int rank, int nranks, int P, int Q, const uint8_t* id, void* cuda_stream,
                         const mp_config* cfg, mp_handle** h);
/* mp_init_config with the default configuration. */
mp_status mp_init(int device, int rank, int nranks, int P, int Q, const uint8_t* id,
                  void* cuda_stream, mp_handle** h);
/* The configuration the handle runs with. */
mp_status mp_handle_get_config(const mp_handle* h, mp_config* cfg);
mp_status mp_finalize(mp_handle* h);
const char* mp_last_error(const mp_handle* h);

/* ---------------------------------------------------------------- matrices */

/* Geometry and ownership of an n x n symmetric tile matrix with tile size nb
 * (nb % 16 == 0, 16 <= nb <= 8192, n >= 1).  No device memory is touched. */
mp_status mp_matrix_create(mp_handle* h, int64_t n, int nb, mp_matrix** A);
mp_status mp_matrix_destroy(mp_matrix* A);

/* Device bytes needed to bind A with the given storage map (NULL = all FP64, the
 * worst case): the map-independent regions (inputs, norms, control arena, the panel buffers and
 * operand caches of ONE panel — K2 formats are single-buffered) followed by the
 * owned tiles in storage precision. */
mp_status mp_matrix_bytes(const mp_matrix* A, const uint8_t* storage_prec, size_t* bytes);

/* Lay out A inside the caller's device workspace (256-byte aligned) for the
 * storage map (NULL = all FP64).  May be called again with a new map on the
 * same workspace (each MLE evaluation has its own map); contents are lost. */
mp_status mp_matrix_bind(mp_matrix* A, const uint8_t* storage_prec, void* d_workspace, size_t bytes);

/* Give A a caller-owned workspace for mp_eval without laying out a tile pool: every mp_eval then
 * binds its own map inside it.  `bytes` must cover at least the map-independent regions
 * (mp_matrix_bytes of the all-FP32 off-diagonal map is a safe minimum); an evaluation whose map
 * needs more returns MP_ERR_NOMEM with report->workspace_bytes set, so the caller can grow the
 * workspace (sized by the map, not by an all-FP64 worst case) and repeat the call. */
mp_status mp_matrix_attach(mp_matrix* A, void* d_workspace, size_t bytes);

/* Multi-rank only (nranks > 1), once per matrix, before its first use:
 * mp_matrix_comm_export allocates this rank's exchange area (send slots in
 * communication precision, stamps, solve vectors; library-owned device memory)
 * and writes its 64-byte CUDA IPC handle to handle_out.  The caller all-gathers
 * the handles (e.g. torch.distributed.all_gather_object) in rank order and
 * passes the nranks * 64 bytes to mp_matrix_comm_connect, which maps every
 * peer's area.  Consumers then read panel tiles directly from the producer's
 * memory (NVLink peer loads across GPUs; same-device IPC between processes). */
mp_status mp_matrix_comm_export(mp_matrix* A, void* handle_out);
mp_status mp_matrix_comm_connect(mp_matrix* A, const void* all_handles);

/* One transfer of the multi-rank panel exchange (host description). */
typedef struct {
    int32_t k;     /* panel */
    int32_t m;     /* tile row: m == k is L~_kk (POTRF output), m > k is L_mk (TRSM output) */
    int32_t peer;  /* producer rank for a pull, -1 for a publish */
    int32_t prec;  /* communication precision (mp_prec) the tile travels in */
    int32_t dir;   /* 0 = publish (this rank produces it for others), 1 = pull */
} mp_xfer;

/* Pure host: the exchange `rank` performs in an nt x nt factorisation on a P x Q grid
 * (POTRF(k,k) -> TRSMs of column k; TRSM(m,k) -> GEMMs of row m and column m and
 * SYRK(m,k)), given the NT*NT comm map.  Writes up to `cap` records (out may be NULL to count)
 * and the total to *count; MP_ERR_NOMEM if cap was too small.  mp_tile_potrf executes
 * exactly these records. */
mp_status mp_exchange_plan(int nt, int P, int Q, int rank, const uint8_t* comm_prec, mp_xfer* out,
                           int64_t cap, int64_t* count);

/* ---------------------------------------------------------------- the path */

/* (1) Matérn tile generation, P:82 (covariance), P:117 (tile norms)
 * (tiles generated directly in their storage precision).
 * theta = {sigma^2, beta, nu}; C(0) = sigma^2 (reading C3); h Euclidean (C5).
 * d_x, d_y: device FP64 [n] locations (replicated on every rank).
 * Pass 1 — storage_prec == NULL: computes s_mk = ||A_mk||_F^2 over real
 *   (unpadded) entries for every lower tile and writes them to the host array
 *   tile_sqnorm[NT*NT] (all-reduced over ranks, identical everywhere).  A must
 *   be bound (any map; the partial sums live in the workspace).  Deterministic
 *   (fixed reduction order).
 * Pass 2 — storage_prec != NULL (the map A is bound with): writes every owned
 *   tile in its storage precision (FP64 or FP32, round-to-nearest-even) and
 *   the padding; tile_sqnorm may be NULL. */
mp_status mp_matern_gen(mp_handle* h, mp_matrix* A, const double* d_x, const double* d_y,
                        const double theta[3], const uint8_t* storage_prec, double* tile_sqnorm);

/* (2) Precision maps — pure host, deterministic, no GPU (P:117, P:146, P:152,
 * Algorithm 2; readings C6, C7, C10, C11 in DESIGN.md).
 *   S = sum_k s_kk + 2 sum_{m>k} s_mk (each sum correctly rounded);
 *   kernel(k,k) = FP64; off-diagonal r = sqrt(s_mk) * NT / sqrt(S) and
 *   kernel = FP16 if r <= u_req/eps[2], else FP32 if r <= u_req/eps[1], else FP64;
 *   storage = FP64 if kernel is FP64 else FP32;
 *   comm per `policy` (TTC: storage, diagonal FP64; AUTO: Algorithm 2).
 * eps may be NULL (= {2^-52, 2^-23, 2^-10}).  Any output pointer may be NULL.
 * If tile_sqnorm is NULL, kernel_prec is an INPUT (a user map) and only the
 * storage and comm maps are derived from it. */
mp_status mp_precision_map(int nt, const double* tile_sqnorm, double u_req, const double* eps,
                           mp_comm_policy policy, uint8_t* kernel_prec, uint8_t* storage_prec,
                           uint8_t* comm_prec);

/* Four-level variant (P:113 / P:117: "FP64, FP32, FP16_32, and FP16"): eps[4] =
 * {FP64, FP32, FP16_32, FP16} (NULL = {2^-52, 2^-23, MP_EPS_FP16_32, 2^-10}; eps[3] >= eps[2]);
 * kernel = MP_FP16H if r <= u_req/eps[3], else MP_FP16 if r <= u_req/eps[2], else FP32 if
 * r <= u_req/eps[1], else FP64.  Storage and communication maps as above (data precisions
 * FP64 / FP32 / FP16: an FP16H successor receives FP16).  A user kernel map may contain MP_FP16H. */
mp_status mp_precision_map4(int nt, const double* tile_sqnorm, double u_req, const double* eps,
                            mp_comm_policy policy, uint8_t* kernel_prec, uint8_t* storage_prec,
                            uint8_t* comm_prec);

/* (3) In-place mixed-precision tile Cholesky A = L L^T (Algorithm 1):
 * DPOTRF (FP64) on diagonal tiles; TRSM(m,k) with L_kk received at comm(k,k): FP64 substitution
 * for FP64-class tiles, the FP32-class product A_mk L~_kk^-T for FP32/FP16-class tiles (reading
 * C12'), result rounded to storage(m,k); L_mk reaches its successors at comm(m,k) and is
 * converted once per panel on the consuming GPU to the successor's operand format;
 * DSYRK and FP64-class GEMMs on the handle's FP64 engine (default: CRT on INT8 tcgen05, see
 * mp_config), FP32-class GEMMs as 3xFP16 (default) or 3xTF32 on tcgen05, FP16-class GEMMs as
 * row-scaled FP16 x FP16 -> FP32 on tcgen05, accumulating into the FP32 tile;
 * pure-FP16 tiles (MP_FP16H, four-level maps) as row-scaled FP16 x FP16 with an F16 TMEM accumulator,
 * widened and added into the FP32 tile — these need a matrix laid out for a four-level map (mp_eval
 * with MP_MAP_ADAPTIVE4 / MP_MAP_USER), else MP_ERR_UNSUPPORTED.
 * kernel_prec / comm_prec: host maps (NT*NT, as produced by mp_precision_map / mp_precision_map4
 * and consistent with the storage map A is bound with).  Blocking.
 * *info = 0 on success, else the 1-based global column of the first
 * non-positive pivot (LAPACK convention) and MP_ERR_NOT_SPD is returned. */
mp_status mp_tile_potrf(mp_handle* h, mp_matrix* A, const uint8_t* kernel_prec,
                        const uint8_t* comm_prec, int64_t* info);

/* (4) Eq. (1) from the factor: log|Sigma| = 2 sum log L_ii (FP64 diagonal
 * tiles), y = L^{-1} Z by tile forward substitution reading L in storage
 * precision with FP64 arithmetic (reading C15), quad = y^T y,
 * l = -(n/2) log(2 pi) - logdet/2 - quad/2.  d_z: device FP64 [n].  Blocking. */
mp_status mp_loglik(mp_handle* h, const mp_matrix* L, const double* d_z,
                    double* loglik, double* logdet, double* quad);

/* Sample the Gaussian field with covariance L L^T: d_z = L d_e (device FP64 [n] each), with L the
 * factor left in A by mp_tile_potrf (read in storage precision; everything on the device).  With e ~ N(0, I) this gives the
 * synthetic measurement vectors Z = L(theta) e of the Monte-Carlo studies.  One rank only. */
mp_status mp_gp_sample(mp_handle* h, const mp_matrix* L, const double* d_e, double* d_z);

/* One whole evaluation (the call a user makes): (1) pass 1, (2), (1) pass 2,
 * (3), (4).  x, y, z are FP64 [n]; if `inputs_on_host` is nonzero they are host
 * pointers and are copied to the device inside the call (pinned memory makes
 * the copy asynchronous), else device pointers.  A must be bound to a
 * workspace (mp_matrix_bind or mp_matrix_attach); it is re-bound to the evaluation's storage map,
 * and MP_ERR_NOMEM (report->workspace_bytes = the bytes needed) if that does not fit.  `mode` picks the kernel map
 * (`user_kernel_prec` is read only for MP_MAP_USER).  Out: report.
 * Returns MP_ERR_NOT_SPD (report->info set, loglik = -inf) for a non-SPD Sigma. */
mp_status mp_eval(mp_handle* h, mp_matrix* A, const double* x, const double* y, const double* z,
                  int inputs_on_host, const double theta[3], double u_req, const double* eps,
                  mp_comm_policy policy, mp_map_mode mode, const uint8_t* user_kernel_prec,
                  mp_eval_report* report);

/* Maps used by the last mp_eval on A (host NT*NT arrays; any may be NULL). */
mp_status mp_matrix_maps(const mp_matrix* A, uint8_t* kernel_prec, uint8_t* storage_prec,
                         uint8_t* comm_prec);

/* Select the covariance family mp_matern_gen / mp_eval generate for A (default MP_COV_MATERN). */
mp_status mp_matrix_set_covariance(mp_matrix* A, mp_covariance kind);

/* Copy owned tile (m, k) of A to host as FP64 nb x nb row-major (padding
 * included), for tests.  Returns MP_ERR_ARG if (m, k) is not owned here. */
mp_status mp_matrix_get_tile(mp_handle* h, const mp_matrix* A, int m, int k, double* h_tile);

/* Overwrite owned tile (m, k) of a bound A from host FP64 nb x nb row-major data (padding
 * included), rounding to the tile's storage precision; marks A as generated.  Lets a caller
 * factor a matrix of its own instead of the Matérn covariance. */
mp_status mp_matrix_set_tile(mp_handle* h, mp_matrix* A, int m, int k, const double* h_tile);

/* Number of tiles per dimension and whether tile (m, k) is owned by this rank. */
int mp_matrix_nt(const mp_matrix* A);
int mp_matrix_owner(const mp_matrix* A, int m, int k);

/* Per-kernel-class device time accounting (CUDA events recorded on the handle's stream around
 * every launch of the class; enable before the region to measure, read after it).
 * Classes: 0 FP64-class trailing update (GEMM + SYRK), 1 FP32-class update, 2 FP16-class update,
 * 3 POTRF (diagonal tiles), 4 TRSM, 5 conversion (K2), 6 generation (K1), 7 solve (K8). */
#define MP_PROF_CLASSES 8
typedef struct {
    double ms[MP_PROF_CLASSES];      /* summed device time per class */
    double flops[MP_PROF_CLASSES];   /* algorithmic flops per class (0 where not a flop count) */
    int64_t launches[MP_PROF_CLASSES];
} mp_profile;
mp_status mp_set_profiling(mp_handle* h, int enable);  /* enable also resets the counters */
/* Profile only the classes whose bit is set in `mask` (bit c = class c; 0 = off); resets the counters.
 * bench.py times the dominant class inside its timed region this way (one event pair per launch of
 * that class only). */
mp_status mp_set_profiling_mask(mp_handle* h, unsigned mask);
mp_status mp_get_profile(mp_handle* h, mp_profile* out);  /* synchronises the stream */

/* The engines mp_tile_potrf / mp_eval actually run for this matrix (they depend on nb as well as
 * on the handle's mp_config: the tcgen05 kernels need nb % 256 == 0).  Out (any may be NULL):
 * fp64 = mp_fp64_engine, fp32 = mp_fp32_engine, fp16 = 1 for tcgen05 / 0 for DMMA, lowp_trsm = 1
 * if FP32/FP16-class TRSMs run as the CRT-8 product (reading C12'). */
mp_status mp_matrix_engines(const mp_matrix* A, int* fp64, int* fp32, int* fp16, int* lowp_trsm);

/* Total kernels launched on this handle since mp_init (for bench accounting). */
int64_t mp_launch_count(const mp_handle* h);

/* Library version string, e.g. "mpgeo 0.1 sm_100a". */
const char* mp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MPGEO_H */
