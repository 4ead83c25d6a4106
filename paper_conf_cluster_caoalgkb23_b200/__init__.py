"""B200-native mixed-precision tile-Cholesky Matérn log-likelihood (Cao et al., CLUSTER 2023).

Thin Python layer over libmpgeo.so (C ABI in include/mpgeo.h).  PyTorch provides
device memory and streams only; every step of the path — Matérn generation,
precision maps (Alg. 2), the mixed-precision tile Cholesky (Alg. 1) and
Eq. (1) — runs in the library.

    from paper_conf_cluster_caoalgkb23_b200 import Evaluator
    ev = Evaluator(n, nb)                  # one handle + worst-case workspace
    rep = ev.eval(x, y, z, theta)          # numpy (host) or torch.cuda tensors
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from ._lib import (EvalReport, MpError, Profile, PROF_CLASSES, lib, MP_OK, MP_ERR_NOT_SPD, MP_FP64, MP_FP32, MP_FP16,  # noqa: F401
                   MP_COMM_TTC, MP_COMM_AUTO, MP_MAP_ADAPTIVE, MP_MAP_FP64, MP_MAP_BAND, MP_MAP_EXTREME,
                   MP_MAP_USER, MP_COV_MATERN, MP_COV_SQEXP)

__all__ = ["Handle", "Matrix", "Evaluator", "precision_map", "exchange_plan", "exact_sum", "MpError", "EvalReport"]

_u8p = C.POINTER(C.c_uint8)
_dp = C.POINTER(C.c_double)


def _u8(a: np.ndarray | None):
    if a is None:
        return None
    assert a.dtype == np.uint8 and a.flags.c_contiguous
    return a.ctypes.data_as(_u8p)


def _d(a: np.ndarray | None):
    if a is None:
        return None
    assert a.dtype == np.float64 and a.flags.c_contiguous
    return a.ctypes.data_as(_dp)


def _ptr(t) -> int:
    """Device or host address of a torch tensor / numpy array."""
    if isinstance(t, np.ndarray):
        return t.ctypes.data
    return t.data_ptr()


class Handle:
    """mp_init / mp_finalize.  One per process and GPU."""

    def __init__(self, device: int = 0, rank: int = 0, nranks: int = 1, P: int = 1, Q: int = 1,
                 nccl_id: bytes | None = None, stream=None):
        import torch

        torch.cuda.set_device(device)
        self.stream = stream if stream is not None else torch.cuda.current_stream(device)
        h = C.c_void_p()
        uid = None
        if nccl_id is not None:
            uid = (C.c_uint8 * 128).from_buffer_copy(nccl_id)
            uid = C.cast(uid, _u8p)
        st = lib.mp_init(device, rank, nranks, P, Q, uid, C.c_void_p(self.stream.cuda_stream), C.byref(h))
        if st != MP_OK:
            raise MpError(st, "mp_init failed")
        self.h = h
        self.device = device
        self.rank, self.nranks, self.P, self.Q = rank, nranks, P, Q

    def check(self, st: int):
        if st != MP_OK:
            raise MpError(st, lib.mp_last_error(self.h).decode())

    def set_profiling(self, enable: bool):
        self.check(lib.mp_set_profiling(self.h, int(enable)))

    def profile(self) -> Profile:
        p = Profile()
        self.check(lib.mp_get_profile(self.h, C.byref(p)))
        return p

    def config(self) -> dict:
        tc, la, oz = C.c_int(), C.c_int(), C.c_int()
        self.check(lib.mp_handle_config(self.h, C.byref(tc), C.byref(la), C.byref(oz)))
        return {"tc": tc.value, "lookahead": la.value, "ozaki": oz.value}

    @property
    def launches(self) -> int:
        return int(lib.mp_launch_count(self.h))

    def close(self):
        if getattr(self, "h", None):
            lib.mp_finalize(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Matrix:
    """mp_matrix_*: geometry + a caller-owned (torch) workspace."""

    def __init__(self, handle: Handle, n: int, nb: int, storage_prec: np.ndarray | None = None, group=None):
        import torch

        self.handle = handle
        A = C.c_void_p()
        handle.check(lib.mp_matrix_create(handle.h, n, nb, C.byref(A)))
        self.A = A
        self.n, self.nb = n, nb
        self.nt = lib.mp_matrix_nt(A)
        if handle.nranks > 1:
            self._connect(group)
        nbytes = C.c_size_t()
        handle.check(lib.mp_matrix_bytes(A, _u8(storage_prec), C.byref(nbytes)))
        self.nbytes = nbytes.value
        self.ws = torch.empty(self.nbytes, dtype=torch.uint8, device=f"cuda:{handle.device}")
        self.bind(storage_prec)

    def _connect(self, group):
        """Exchange the CUDA IPC handles of every rank's exchange area (torch.distributed all-gather)."""
        import torch.distributed as dist

        buf = (C.c_uint8 * 64)()
        self.handle.check(lib.mp_matrix_comm_export(self.A, buf))
        allh = [None] * self.handle.nranks
        dist.all_gather_object(allh, bytes(buf), group=group)
        joined = b"".join(allh)
        self.handle.check(lib.mp_matrix_comm_connect(self.A, joined))

    def owner(self, m: int, k: int) -> int:
        return int(lib.mp_matrix_owner(self.A, m, k))

    def bind(self, storage_prec: np.ndarray | None):
        self.handle.check(lib.mp_matrix_bind(self.A, _u8(storage_prec), C.c_void_p(self.ws.data_ptr()), self.nbytes))

    def tile(self, m: int, k: int) -> np.ndarray:
        out = np.empty((self.nb, self.nb), dtype=np.float64)
        self.handle.check(lib.mp_matrix_get_tile(self.handle.h, self.A, m, k, _d(out)))
        return out

    def set_covariance(self, kind: int):
        """MP_COV_MATERN (default) or MP_COV_SQEXP."""
        self.handle.check(lib.mp_matrix_set_covariance(self.A, kind))

    def set_tile(self, m: int, k: int, t: np.ndarray):
        t = np.ascontiguousarray(t, dtype=np.float64)
        assert t.shape == (self.nb, self.nb)
        self.handle.check(lib.mp_matrix_set_tile(self.handle.h, self.A, m, k, _d(t)))

    def maps(self):
        nn = self.nt * self.nt
        km, sm, cm = (np.full(nn, 255, np.uint8) for _ in range(3))
        self.handle.check(lib.mp_matrix_maps(self.A, _u8(km), _u8(sm), _u8(cm)))
        return km.reshape(self.nt, self.nt), sm.reshape(self.nt, self.nt), cm.reshape(self.nt, self.nt)

    # ---- the four calls of the path
    def matern_gen(self, x, y, theta, storage_prec: np.ndarray | None = None) -> np.ndarray | None:
        th = np.ascontiguousarray(theta, dtype=np.float64)
        if storage_prec is None:
            s = np.zeros((self.nt, self.nt), dtype=np.float64)
            self.handle.check(lib.mp_matern_gen(self.handle.h, self.A, C.c_void_p(_ptr(x)), C.c_void_p(_ptr(y)),
                                                _d(th), None, _d(s)))
            return s
        sp = np.ascontiguousarray(storage_prec, dtype=np.uint8)
        self.handle.check(lib.mp_matern_gen(self.handle.h, self.A, C.c_void_p(_ptr(x)), C.c_void_p(_ptr(y)),
                                            _d(th), _u8(sp), None))
        return None

    def potrf(self, kernel_prec: np.ndarray, comm_prec: np.ndarray) -> int:
        info = C.c_int64(0)
        st = lib.mp_tile_potrf(self.handle.h, self.A, _u8(np.ascontiguousarray(kernel_prec, np.uint8)),
                               _u8(np.ascontiguousarray(comm_prec, np.uint8)), C.byref(info))
        if st == MP_ERR_NOT_SPD:
            return int(info.value)
        self.handle.check(st)
        return 0

    def gp_sample(self, e, z):
        """z = L e with the factor in this matrix (device tensors, FP64 [n])."""
        self.handle.check(lib.mp_gp_sample(self.handle.h, self.A, C.c_void_p(_ptr(e)), C.c_void_p(_ptr(z))))

    def loglik(self, z) -> tuple[float, float, float]:
        ll, ld, q = C.c_double(), C.c_double(), C.c_double()
        self.handle.check(lib.mp_loglik(self.handle.h, self.A, C.c_void_p(_ptr(z)), C.byref(ll), C.byref(ld),
                                        C.byref(q)))
        return ll.value, ld.value, q.value

    def close(self):
        if getattr(self, "A", None):
            lib.mp_matrix_destroy(self.A)
            self.A = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def precision_map(tile_sqnorm: np.ndarray | None, u_req: float = 1e-9, eps=None, policy: int = MP_COMM_AUTO,
                  kernel_prec: np.ndarray | None = None):
    """mp_precision_map (host only).  Returns (kernel, storage, comm) NT x NT uint8 maps."""
    if tile_sqnorm is not None:
        s = np.ascontiguousarray(tile_sqnorm, dtype=np.float64)
        nt = s.shape[0]
        km = np.full((nt, nt), 255, np.uint8)
    else:
        km = np.ascontiguousarray(kernel_prec, dtype=np.uint8).copy()
        nt = km.shape[0]
        s = None
    sm = np.full((nt, nt), 255, np.uint8)
    cm = np.full((nt, nt), 255, np.uint8)
    e = None if eps is None else np.ascontiguousarray(eps, dtype=np.float64)
    st = lib.mp_precision_map(nt, _d(s), float(u_req), _d(e), policy, _u8(km), _u8(sm), _u8(cm))
    if st != MP_OK:
        raise MpError(st, "mp_precision_map failed")
    return km, sm, cm


def exchange_plan(nt: int, P: int, Q: int, rank: int, comm_prec: np.ndarray) -> list[tuple]:
    """mp_exchange_plan: [(k, m, peer, prec, dir)] for `rank` (dir 0 = publish, 1 = pull)."""
    from ._lib import Xfer

    cm = np.ascontiguousarray(comm_prec, dtype=np.uint8)
    cnt = C.c_int64(0)
    st = lib.mp_exchange_plan(nt, P, Q, rank, _u8(cm), None, 0, C.byref(cnt))
    if st != MP_OK:
        raise MpError(st, "mp_exchange_plan failed")
    arr = (Xfer * max(1, cnt.value))()
    st = lib.mp_exchange_plan(nt, P, Q, rank, _u8(cm), arr, cnt.value, C.byref(cnt))
    if st != MP_OK:
        raise MpError(st, "mp_exchange_plan failed")
    return [(x.k, x.m, x.peer, x.prec, x.dir) for x in arr[: cnt.value]]


def exact_sum(v: np.ndarray) -> float:
    v = np.ascontiguousarray(v, dtype=np.float64)
    return float(lib.mpgeo_exact_sum(_d(v), v.size))


class Evaluator:
    """One log-likelihood evaluation per call (mp_eval) on a worst-case (all-FP64) workspace."""

    def __init__(self, n: int, nb: int, device: int = 0, handle: Handle | None = None, group=None,
                 covariance: int = MP_COV_MATERN):
        self.handle = handle or Handle(device)
        self.M = Matrix(self.handle, n, nb, None, group=group)
        if covariance != MP_COV_MATERN:
            self.M.set_covariance(covariance)
        self.n, self.nb, self.nt = n, nb, self.M.nt

    def eval(self, x, y, z, theta, u_req: float = 1e-9, mode: int = MP_MAP_ADAPTIVE, policy: int = MP_COMM_AUTO,
             eps=None, kernel_prec: np.ndarray | None = None) -> EvalReport:
        on_host = isinstance(x, np.ndarray)
        if on_host:
            for a in (x, y, z):
                assert a.dtype == np.float64 and a.flags.c_contiguous and a.shape == (self.n,)
        th = np.ascontiguousarray(theta, dtype=np.float64)
        e = None if eps is None else np.ascontiguousarray(eps, dtype=np.float64)
        rep = EvalReport()
        st = lib.mp_eval(self.handle.h, self.M.A, C.c_void_p(_ptr(x)), C.c_void_p(_ptr(y)), C.c_void_p(_ptr(z)),
                         int(on_host), _d(th), float(u_req), _d(e), policy, mode,
                         _u8(None if kernel_prec is None else np.ascontiguousarray(kernel_prec, np.uint8)),
                         C.byref(rep))
        if st not in (MP_OK, MP_ERR_NOT_SPD):
            self.handle.check(st)
        return rep
