"""Kernel-, storage- and communication-precision maps.  Oracle: test infrastructure only.

Three precision classes (reading C7): FP64 > FP32 > FP16, encoded 0/1/2 (smaller
= higher precision).  "FP16" is the paper's FP16_32 (FP16 operands, FP32
accumulation and storage).  Four-level maps ("we
incorporate FP64, FP32, FP16_32, and FP16") add FP16H = 3, the
paper's pure FP16 class (FP16 operands and accumulation), tried before FP16_32
with its own epsilon (eps = 4-tuple; reading C7' in DESIGN.md for FP16_32's).

kernel map  (§V; readings C6, C7):
    kernel(k, k) = FP64  ("computations ... on tiles ... along the diagonal ...
    invariably make use of FP64").
    Off-diagonal: the lowest precision p with ||A_mk|| * NT / ||A|| <= u_req / u_p
    (P:117), evaluated exactly as
        r = sqrt(s_mk) * NT / sqrt(S)          (FP64, this operation order)
        FP16 if r <= u_req / eps16, else FP32 if r <= u_req / eps32, else FP64
    with eps = machine epsilons (2^-52, 2^-23, 2^-10 by default) and ties going
    to the lower precision (the paper's "<=").
storage map: FP64 where the kernel is FP64, else FP32 (tiles whose
    kernel is FP16 are "stored directly in FP32 during the matrix generation").
comm map    (Algorithm 2; reading C10, C11):
    diagonal:  comm(k,k) = FP32, raised to FP64 if some kernel(m,k), m>k, is FP64
               (Alg. 2 lines 5-10; for k = NT-1 there are no consumers).
    off-diagonal (m > k; Alg. 2 lines 12-28 with m starting at k+1):
               comm(m,k) starts at kernel(m,k) (reading C10: SYRK(m,k) is a successor
               that receives the tile at the precision TRSM(m,k) produced it for),
               then is raised to the highest kernel precision of its GEMM successors,
               row broadcast kernel(m,n), k<n<m (lines 17-21) and column broadcast
               kernel(n,m), n>m (lines 23-27), stopping as soon as it is not lower
               than storage(m,k), in which case comm = storage (TTC).
    policy TTC: comm = storage everywhere, comm(k,k) = FP64 (the POTRF precision).
"""
from __future__ import annotations

import numpy as np

from . import FP16, FP16H, FP32, FP64
from .tiles import global_sqnorm

EPS_DEFAULT = (2.0**-52, 2.0**-23, 2.0**-10)  # reading C7: literal machine epsilons
COMM_TTC, COMM_AUTO = 0, 1


def tile_ratio(s_mk: float, nt: int, S: float) -> float:
    """||A_mk|| * NT / ||A||, in the fixed FP64 operation order of reading C6/O5."""
    return np.sqrt(s_mk) * float(nt) / np.sqrt(S)


def kernel_map(s: np.ndarray, u_req: float, eps=EPS_DEFAULT) -> np.ndarray:
    """kernel_precision[m, k] for m >= k (upper triangle left at 255 = unused). P:117.

    Three levels (len(eps) == 3; FP16 = FP16_32) or four (len(eps) == 4: eps = (FP64, FP32,
    FP16_32, FP16), P:113 / P:117 "FP64, FP32, FP16_32, and FP16"; the pure-FP16 class FP16H is
    tried first: FP16H if r <= u_req/eps[3], else FP16_32 if r <= u_req/eps[2], ...)."""
    nt = s.shape[0]
    S = global_sqnorm(s)
    four = len(eps) == 4
    thr16h = u_req / eps[FP16H] if four else -1.0
    thr16 = u_req / eps[FP16]
    thr32 = u_req / eps[FP32]
    kmap = np.full((nt, nt), 255, dtype=np.uint8)
    for k in range(nt):
        kmap[k, k] = FP64
        for m in range(k + 1, nt):
            r = tile_ratio(float(s[m, k]), nt, S)
            if r <= thr16h:
                kmap[m, k] = FP16H
            elif r <= thr16:
                kmap[m, k] = FP16
            elif r <= thr32:
                kmap[m, k] = FP32
            else:
                kmap[m, k] = FP64
    return kmap


def storage_precision(kernel_prec: int) -> int:
    """get_storage_precision of Alg. 2 line 16: FP64 stays FP64, FP32 and FP16 kernels (FP16_32 and
    pure FP16) store FP32."""
    return FP64 if kernel_prec == FP64 else FP32


def storage_map(kmap: np.ndarray) -> np.ndarray:
    nt = kmap.shape[0]
    smap = np.full((nt, nt), 255, dtype=np.uint8)
    for k in range(nt):
        for m in range(k, nt):
            smap[m, k] = storage_precision(int(kmap[m, k]))
    return smap


def higher(a: int, b: int) -> int:
    """get_higher_precision of Alg. 2 (smaller code = higher precision)."""
    return min(a, b)


def comm_map(kmap: np.ndarray, policy: int = COMM_AUTO) -> np.ndarray:
    """comm_precision per Algorithm 2 under readings C10/C11, or TTC."""
    nt = kmap.shape[0]
    smap = storage_map(kmap)
    cmap = np.full((nt, nt), 255, dtype=np.uint8)
    if policy == COMM_TTC:
        for k in range(nt):
            cmap[k, k] = FP64
            for m in range(k + 1, nt):
                cmap[m, k] = smap[m, k]
        return cmap
    # Diagonal tiles (k, k) operating POTRF(k, k): Alg. 2 lines 5-10.
    for k in range(nt):
        cmap[k, k] = FP32
        for m in range(k + 1, nt):
            if kmap[m, k] == FP64:
                cmap[k, k] = FP64
    # Off-diagonal tiles (m, k) operating TRSM(m, k): Alg. 2 lines 12-28.
    for k in range(nt - 1):
        for m in range(k + 1, nt):  # reading C10 (i): m starts at k+1
            st = int(smap[m, k])
            comm = FP16  # line 14: initialised to the lowest precision (FP16 data; an FP16H
            # consumer receives FP16 operands too, so higher() with it leaves FP16)
            comm = higher(comm, int(kmap[m, k]))  # reading C10 (ii): SYRK(m,k) successor
            done = False
            if comm <= st:
                comm, done = st, True
            # row broadcast: GEMM(m, n, k), k < n < m  (lines 17-21)
            n = k + 1
            while not done and n < m:
                comm = higher(comm, int(kmap[m, n]))
                if comm <= st:
                    comm, done = st, True
                n += 1
            # column broadcast: GEMM(n, m, k), n > m  (lines 23-27)
            n = m + 1
            while not done and n < nt:
                comm = higher(comm, int(kmap[n, m]))
                if comm <= st:
                    comm, done = st, True
                n += 1
            cmap[m, k] = comm
    return cmap


def precision_maps(s: np.ndarray, u_req: float, eps=EPS_DEFAULT, policy: int = COMM_AUTO):
    """(kernel, storage, comm) maps from the tile square norms."""
    kmap = kernel_map(s, u_req, eps)
    return kmap, storage_map(kmap), comm_map(kmap, policy)


def all_fp64_maps(nt: int):
    kmap = np.full((nt, nt), 255, dtype=np.uint8)
    for k in range(nt):
        for m in range(k, nt):
            kmap[m, k] = FP64
    return kmap, storage_map(kmap), comm_map(kmap, COMM_TTC)


def extreme_map(nt: int, off: int = FP16) -> np.ndarray:
    """The paper's extreme kernel map: FP64 diagonal, `off` elsewhere."""
    kmap = np.full((nt, nt), 255, dtype=np.uint8)
    for k in range(nt):
        kmap[k, k] = FP64
        for m in range(k + 1, nt):
            kmap[m, k] = off
    return kmap


def band_map(s: np.ndarray, u_req: float, eps=EPS_DEFAULT) -> np.ndarray:
    """Reading C21 (config 2, "band FP64/FP32"): the narrowest band b such that every tile
    the two-level (FP64/FP32) rule marks FP64 lies within |m-k| < b; FP64 inside, FP32 outside."""
    nt = s.shape[0]
    S = global_sqnorm(s)
    thr32 = u_req / eps[FP32]
    b = 1
    for k in range(nt):
        for m in range(k + 1, nt):
            if not tile_ratio(float(s[m, k]), nt, S) <= thr32:  # two-level rule marks FP64
                b = max(b, m - k + 1)
    kmap = np.full((nt, nt), 255, dtype=np.uint8)
    for k in range(nt):
        for m in range(k, nt):
            kmap[m, k] = FP64 if m - k < b else FP32
    return kmap
