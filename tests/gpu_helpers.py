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
            for e in (eps[1], eps[2]):
                worst = min(worst, abs(r / (u_req / e) - 1.0))
    assert worst >= 1e-12, f"near tie in the precision rule (|r/thr - 1| = {worst:g}); change the seed"
    return worst
