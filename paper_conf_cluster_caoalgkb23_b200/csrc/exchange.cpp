// Host-only description of the multi-rank panel exchange.
//
// 2D block-cyclic ownership owner(m, k) = (m mod P) * Q + (k mod Q).  In panel k:
//   * L~_kk (POTRF output, comm(k,k) precision) goes from owner(k,k) to the owners of the TRSM
//     tiles (m, k), m > k ("POTRF (k, k) ... broadcasts to TRSMs in column k");
//   * L_mk (TRSM output, comm(m,k) precision) goes from owner(m,k) to the owners of GEMM(m,n,k),
//     k < n < m (row m), GEMM(n,m,k), n > m (column m) and SYRK(m,k) on tile (m,m)
//     ("TRSM (m, k) broadcasts to GEMMs in row m, GEMMs in column m, and SYRK (m, k)").
// A producer publishes a tile once if any other rank needs it; each consumer pulls it once.
// The engine executes exactly these records (engine.cu plan_potrf), and tests check them.
#include <cstring>
#include <vector>

#include "../../include/mpgeo.h"

namespace {
inline int owner(int m, int k, int P, int Q) { return (m % P) * Q + (k % Q); }
}  // namespace

extern "C" mp_status mp_exchange_plan(int nt, int P, int Q, int rank, const uint8_t* comm_prec, mp_xfer* out,
                                      int64_t cap, int64_t* count) {
    if (nt <= 0 || P < 1 || Q < 1 || rank < 0 || rank >= P * Q || !comm_prec || !count) return MP_ERR_ARG;
    const int R = P * Q;
    std::vector<char> need(R);
    int64_t c = 0;
    auto emit = [&](int k, int m, int peer, int prec, int dir) {
        if (out && c < cap) out[c] = mp_xfer{k, m, peer, prec, dir};
        ++c;
    };
    for (int k = 0; k + 1 < nt; ++k) {
        // L~_kk: consumers are the owners of column k below the diagonal
        std::fill(need.begin(), need.end(), 0);
        for (int m = k + 1; m < nt; ++m) need[owner(m, k, P, Q)] = 1;
        const int okk = owner(k, k, P, Q);
        const int pkk = comm_prec[(size_t)k * nt + k];
        bool remote = false;
        for (int r = 0; r < R; ++r) remote |= (r != okk && need[r]);
        if (rank == okk && remote) emit(k, k, -1, pkk, 0);
        if (rank != okk && need[rank]) emit(k, k, okk, pkk, 1);
        // L_mk
        for (int m = k + 1; m < nt; ++m) {
            std::fill(need.begin(), need.end(), 0);
            need[owner(m, m, P, Q)] = 1;
            for (int n = k + 1; n < m; ++n) need[owner(m, n, P, Q)] = 1;
            for (int n = m + 1; n < nt; ++n) need[owner(n, m, P, Q)] = 1;
            const int o = owner(m, k, P, Q);
            const int p = comm_prec[(size_t)m * nt + k];
            remote = false;
            for (int r = 0; r < R; ++r) remote |= (r != o && need[r]);
            if (rank == o && remote) emit(k, m, -1, p, 0);
            if (rank != o && need[rank]) emit(k, m, o, p, 1);
        }
    }
    *count = c;
    return (out && c > cap) ? MP_ERR_NOMEM : MP_OK;
}
