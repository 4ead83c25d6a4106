"""Shared helpers for the -m gpu parity tests (they call the CUDA path through the C ABI)."""
import numpy as np

from oracle.tiles import tile_range


def lower_mask(nb):
    return np.tril(np.ones((nb, nb), bool))


def gpu_factor_dense(M, n):
    """Assemble the lower factor from the GPU tiles (real part only)."""
    nb, nt = M.nb, M.nt
    L = np.zeros((n, n))
    for k in range(nt):
        for m in range(k, nt):
            t = M.tile(m, k)
            r0, r1 = tile_range(m, n, nb)
            c0, c1 = tile_range(k, n, nb)
            L[r0:r1, c0:c1] = t[: r1 - r0, : c1 - c0]
    return np.tril(L)


def to_dev(a):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def near_tie_guard(s, nt, u_req, eps=(2.0**-52, 2.0**-23, 2.0**-10)):
    """Reading C6: fail loudly (not pass by luck) if a tile ratio sits within 1e-12 of a threshold."""
    from oracle.tiles import global_sqnorm
    S = global_sqnorm(s)
    worst = np.inf
    for k in range(nt):
        for m in range(k + 1, nt):
            r = np.sqrt(s[m, k]) * nt / np.sqrt(S)
            for e in eps[1:]:
                worst = min(worst, abs(r / (u_req / e) - 1.0))
    assert worst >= 1e-12, f"near tie in the precision rule (|r/thr - 1| = {worst:g}); change the seed"
    return worst


# ---------------------------------------------------------------------------------------------
# Backward-error bound of the mixed-precision factor (replaces the MP emulation as a pass criterion).
#
# The GPU factor L^ satisfies L^ L^T = A + dA.  Per tile (m, n), m >= n, standard rounding-error
# analysis of Algorithm 1 with the maps of P:117/P:152/Alg. 2 gives, up to a constant c,
#   ||dA_mn|| <= (NT+1) u_s(m,n) (||A_mn|| + sum_k ||L_mk|| ||L_nk||)          storage rounding
#              + sum_{k<n} (e_mk ||L_nk|| + ||L_mk|| e_nk + nb u_acc ||L_mk|| ||L_nk||)
#                  e_mk = operand error of L_mk: comm(m,k) rounding + the kernel(m,n) operand format
#              + [m > n] (u_s + t_nn) ||L_mn|| ||L_nn||_2 + kappa(L_nn) e(L~_nn) ||L_mn||   TRSM(m,n)
#              + [m == n] nb u64 ||A_nn||                                        POTRF
# with t_nn = nb 2^-25 kappa(L_nn) for the FP32-class TRSM product (reading C12') or nb 2^-52
# kappa(L_nn) for the FP64 substitution.  Frobenius norms; ||L_mk|| from the oracle's FP64 factor.
# ---------------------------------------------------------------------------------------------
U_PREC = {0: 2.0**-53, 1: 2.0**-24, 2: 2.0**-11}
ABS16 = 2.0**-25  # plain FP16 rounding below the normal range: absolute error <= half the subnormal spacing
# operand-format rounding of the kernel classes; class 3 (pure FP16, four-level maps): the hs planes,
# 11 bits relative to each entry + subnormals below 2^-14 of a row max in [2, 4) (<= 2^-26 of the max)
OP_REL = {0: 2.0**-52, 1: 2.0**-20, 2: 2.0**-11, 3: 2.0**-11 * 1.1}
ACC = {0: 2.0**-53, 1: 2.0**-23, 2: 2.0**-23, 3: 2.0**-11}  # accumulation unit over K (FP64 / FP32 / FP16 TMEM)


def mp_backward_check(A, Lhat, L, km, sm, cm, nt, nb, lowp_trsm=True, scaled_fp16=True, c=4.0):
    """Max over tiles of ||(L^ L^T - A)_mn||_F / bound_mn and the total ||L^ L^T - A||_F (FP64, on the GPU
    through torch when available).  A, Lhat, L: {(m, k): tile} (real parts, same shapes).
    Operand errors in Frobenius norm: e(L, p) = u_p ||L|| (+ 2^-25 sqrt(#entries) for plain FP16, whose
    small entries fall below the normal range: the communication precision FP16 of STC, and the FP16-class
    operand unless it is row-scaled as on the GPU — scaled_fp16)."""
    import torch
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    T = {key: torch.from_numpy(np.ascontiguousarray(t)).to(dev) for key, t in Lhat.items()}
    nrm = {key: float(np.linalg.norm(t)) for key, t in L.items()}
    size = {key: float(np.sqrt(t.size)) for key, t in L.items()}
    two = {k: float(np.linalg.norm(L[k, k], 2)) for k in range(nt)}
    kap = {k: float(np.linalg.cond(np.tril(L[k, k]))) for k in range(nt)}

    def e_comm(key, p):
        return U_PREC[int(p)] * nrm[key] + (ABS16 * size[key] if int(p) == 2 else 0.0)

    def e_op(key, p):
        return OP_REL[int(p)] * nrm[key] + (ABS16 * size[key] if int(p) == 2 and not scaled_fp16 else 0.0)

    worst, tot2 = 0.0, 0.0
    for n_ in range(nt):
        for m in range(n_, nt):
            D = -torch.from_numpy(np.ascontiguousarray(A[m, n_])).to(dev)
            for k in range(n_ + 1):
                D = D + T[m, k] @ T[n_, k].T
            d = float(torch.linalg.norm(D))
            tot2 += d * d * (1 if m == n_ else 2)
            us = U_PREC[int(sm[m, n_])]
            p = int(km[m, n_]) if m != n_ else 0  # SYRK (m == n) is FP64
            sum_ll = sum(nrm[m, k] * nrm[n_, k] for k in range(n_))
            a = float(np.linalg.norm(A[m, n_]))
            b = (nt + 1) * us * (a + sum_ll)
            for k in range(n_):
                em = e_comm((m, k), cm[m, k]) + e_op((m, k), p)
                en = e_comm((n_, k), cm[n_, k]) + e_op((n_, k), p)
                b += em * nrm[n_, k] + nrm[m, k] * en + nb * ACC[p] * nrm[m, k] * nrm[n_, k]
            if m > n_:
                if lowp_trsm and km[m, n_] != 0:
                    t = us + nb * 2.0**-25 * kap[n_]
                else:
                    t = us + nb * 2.0**-52 * kap[n_]
                b += t * nrm[m, n_] * two[n_] + nrm[m, n_] * kap[n_] * e_comm((n_, n_), cm[n_, n_])
            else:
                b += nb * 2.0**-53 * a
            worst = max(worst, d / (c * b))
    return worst, float(np.sqrt(tot2))


def loglik_perturbation_bound(A_dense, z, dA_fro):
    """Bound on |l(A + dA) - l(A)| given ||dA||_F, valid whenever rho = ||A^-1||_2 ||dA||_F < 1:
    |log det(A + dA) - log det A| = |sum_i log(1 + mu_i)| <= sum |mu_i| / (1 - rho) <= ||A^-1||_F ||dA||_F / (1 - rho)
    (mu_i the eigenvalues of A^-1/2 dA A^-1/2) and |z^T (A + dA)^-1 z - z^T A^-1 z| <= ||A^-1 z||^2 ||dA|| / (1 - rho),
    so |dl| <= 1/2 (||A^-1||_F + ||A^-1 z||^2) ||dA||_F / (1 - rho).  Returns (bound, rho)."""
    import scipy.linalg
    c = scipy.linalg.cho_factor(A_dense, lower=True)
    Ainv = scipy.linalg.cho_solve(c, np.eye(A_dense.shape[0]))
    w = scipy.linalg.cho_solve(c, z)
    rho = float(np.linalg.norm(Ainv, 2)) * dA_fro
    bound = 0.5 * (np.linalg.norm(Ainv) + float(w @ w)) * dA_fro / (1.0 - rho) if rho < 1 else float("inf")
    return bound, rho


def residual_tiles(A, L, nt):
    """||A - L L^T||_F / ||A||_F over the whole symmetric matrix, tile by tile (torch FP64; the GPU when
    available) — the oracle's `residual` for sizes where a dense n x n copy is too large.  Pinned
    against oracle.cholesky.residual in tests/test_helpers_cpu.py."""
    import torch
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    T = {key: torch.from_numpy(np.ascontiguousarray(t)).to(dev) for key, t in L.items()}
    num, den = 0.0, 0.0
    for n_ in range(nt):
        for m in range(n_, nt):
            a = torch.from_numpy(np.ascontiguousarray(A[m, n_])).to(dev)
            D = -a
            for k in range(n_ + 1):
                Lm, Ln = T[m, k], T[n_, k]
                if m == k:
                    Lm = torch.tril(Lm)
                if n_ == k:
                    Ln = torch.tril(Ln)
                D = D + Lm @ Ln.T
            w = 1 if m == n_ else 2
            num += w * float(torch.sum(D * D))
            den += w * float(torch.sum(a * a))
    return float(np.sqrt(num / den))
