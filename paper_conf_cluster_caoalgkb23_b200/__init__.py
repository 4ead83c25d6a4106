"""B200-native mixed-precision tile-Cholesky Matérn log-likelihood (Cao et al., CLUSTER 2023).

Thin Python layer over libmpgeo.so (C ABI in include/mpgeo.h).  PyTorch provides
device memory and streams only; every step of the path — Matérn generation,
precision maps (Alg. 2), the mixed-precision tile Cholesky (Alg. 1) and
Eq. (1) — runs in the library.

    from paper_conf_cluster_caoalgkb23_b200 import Evaluator
    ev = Evaluator(n, nb)                  # one handle; the workspace grows to what each map needs
    rep = ev.eval(x, y, z, theta)          # numpy (host) or torch.cuda tensors

Engines and schedule switches are an mp_config (Handle(config={...})): fp64_engine MP_F64_CRT16
(default) / MP_F64_DMMA, fp32_engine MP_F32_3XFP16 (default) / MP_F32_3XTF32 / MP_F32_DMMA,
fp16_tensor, lookahead, reserve_pairs, lowp_trsm_product, matern_table, f16x3_persistent,
crt_phase_lock (include/mpgeo.h).
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from ._lib import (Config, EvalReport, MpError, Profile, PROF_CLASSES, lib, MP_OK, MP_ERR_NOT_SPD,  # noqa: F401
                   MP_ERR_NOMEM, MP_FP64, MP_FP32, MP_FP16, MP_COMM_TTC, MP_COMM_AUTO, MP_MAP_ADAPTIVE, MP_MAP_FP64,
                   MP_MAP_BAND, MP_MAP_EXTREME, MP_MAP_USER, MP_COV_MATERN, MP_COV_SQEXP, MP_F64_CRT16, MP_F64_DMMA,
                   MP_F32_3XFP16, MP_F32_3XTF32, MP_F32_DMMA, MP_FP16H, MP_MAP_ADAPTIVE4, MP_EPS_FP16_32)

__all__ = ["Handle", "Matrix", "Evaluator", "precision_map", "exchange_plan", "exact_sum", "unique_id", "MpError",
           "EvalReport", "default_config", "shared_unique_id"]

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


def unique_id() -> bytes:
    """mp_get_unique_id: the 128-byte communicator id rank 0 creates and broadcasts."""
    buf = (C.c_uint8 * 128)()
    st = lib.mp_get_unique_id(C.cast(buf, _u8p))
    if st != MP_OK:
        raise MpError(st, "mp_get_unique_id failed")
    return bytes(buf)


def shared_unique_id(group=None) -> bytes:
    """unique_id() on rank 0, broadcast to every rank of the torch.distributed group."""
    import torch.distributed as dist

    obj = [unique_id() if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def default_config() -> dict:
    """mp_config_default as a dict."""
    c = Config()
    lib.mp_config_default(C.byref(c))
    return c.as_dict()


class Handle:
    """mp_init_config / mp_finalize.  One per process and GPU.  `config`: dict of mp_config fields
    overriding the defaults; `uid`: the communicator id (unique_id()) shared by all ranks."""

    def __init__(self, device: int = 0, rank: int = 0, nranks: int = 1, P: int = 1, Q: int = 1,
                 uid: bytes | None = None, stream=None, config: dict | None = None):
        import torch

        torch.cuda.set_device(device)
        self.stream = stream if stream is not None else torch.cuda.current_stream(device)
        h = C.c_void_p()
        cid = None
        if uid is not None:
            cid = C.cast((C.c_uint8 * 128).from_buffer_copy(uid), _u8p)
        cfg = Config()
        lib.mp_config_default(C.byref(cfg))
        for k, v in (config or {}).items():
            if not hasattr(cfg, k):
                raise ValueError(f"unknown mp_config field {k}")
            setattr(cfg, k, int(v))
        st = lib.mp_init_config(device, rank, nranks, P, Q, cid, C.c_void_p(self.stream.cuda_stream), C.byref(cfg),
                                C.byref(h))
        if st != MP_OK:
            raise MpError(st, "mp_init_config failed")
        self.h = h
        self.device = device
        self.rank, self.nranks, self.P, self.Q = rank, nranks, P, Q

    def check(self, st: int):
        if st != MP_OK:
            raise MpError(st, lib.mp_last_error(self.h).decode())

    def set_profiling(self, enable: bool, classes=None):
        """All classes, or only `classes` (names of PROF_CLASSES or indices)."""
        if classes is None:
            self.check(lib.mp_set_profiling(self.h, int(enable)))
            return
        mask = 0
        for c in classes:
            mask |= 1 << (PROF_CLASSES.index(c) if isinstance(c, str) else int(c))
        self.check(lib.mp_set_profiling_mask(self.h, mask if enable else 0))

    def profile(self) -> Profile:
        p = Profile()
        self.check(lib.mp_get_profile(self.h, C.byref(p)))
        return p

    def config(self) -> dict:
        c = Config()
        self.check(lib.mp_handle_get_config(self.h, C.byref(c)))
        return c.as_dict()

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
    """mp_matrix_*: geometry + a caller-owned (torch) workspace.

    attach=False: the workspace is sized for `storage_prec` (None = all FP64) and bound to it.
    attach=True: a workspace for mp_eval only (mp_matrix_attach), sized for the smallest map and grown
    by Evaluator when an evaluation's map needs more (no all-FP64 worst case)."""

    def __init__(self, handle: Handle, n: int, nb: int, storage_prec: np.ndarray | None = None, group=None,
                 attach: bool = False):
        self.handle = handle
        A = C.c_void_p()
        handle.check(lib.mp_matrix_create(handle.h, n, nb, C.byref(A)))
        self.A = A
        self.n, self.nb = n, nb
        self.nt = lib.mp_matrix_nt(A)
        self.ws = None
        if handle.nranks > 1:
            self._connect(group)
        if attach:
            nt = self.nt
            smallest = np.full((nt, nt), 255, np.uint8)  # FP64 diagonal, FP32 elsewhere
            smallest[np.tril_indices(nt, -1)] = MP_FP32
            np.fill_diagonal(smallest, MP_FP64)
            self.attach(self.bytes_for(smallest))
        else:
            self._alloc(self.bytes_for(storage_prec))
            self.bind(storage_prec)

    def bytes_for(self, storage_prec: np.ndarray | None) -> int:
        nbytes = C.c_size_t()
        self.handle.check(lib.mp_matrix_bytes(self.A, _u8(storage_prec), C.byref(nbytes)))
        return nbytes.value

    def _alloc(self, nbytes: int):
        import torch

        self.ws = None  # release the old workspace before the new one is allocated
        torch.cuda.empty_cache()
        self.nbytes = int(nbytes)
        self.ws = torch.empty(self.nbytes, dtype=torch.uint8, device=f"cuda:{self.handle.device}")

    def attach(self, nbytes: int):
        """(Re)allocate a workspace of nbytes and attach it for mp_eval (mp_matrix_attach)."""
        self._alloc(nbytes)
        self.handle.check(lib.mp_matrix_attach(self.A, C.c_void_p(self.ws.data_ptr()), self.nbytes))

    def engines(self) -> dict:
        """mp_matrix_engines: the engines this matrix runs with (handle config + nb)."""
        f64, f32, f16, tr = C.c_int(), C.c_int(), C.c_int(), C.c_int()
        self.handle.check(lib.mp_matrix_engines(self.A, C.byref(f64), C.byref(f32), C.byref(f16), C.byref(tr)))
        return {"fp64": f64.value, "fp32": f32.value, "fp16_tensor": f16.value, "lowp_trsm_product": tr.value}

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
                  kernel_prec: np.ndarray | None = None, levels: int = 3):
    """mp_precision_map (levels = 3) or mp_precision_map4 (levels = 4; host only).  Returns (kernel,
    storage, comm) NT x NT uint8 maps."""
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
    fn = lib.mp_precision_map4 if levels == 4 else lib.mp_precision_map
    st = fn(nt, _d(s), float(u_req), _d(e), policy, _u8(km), _u8(sm), _u8(cm))
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
    """One log-likelihood evaluation per call (mp_eval).  One rank: the workspace is sized by the
    evaluation's storage map and grows when a later map needs more (mp_matrix_attach, MP_ERR_NOMEM);
    several ranks: each binds its all-FP64 worst case once (the ranks must not disagree mid-call)."""

    def __init__(self, n: int, nb: int, device: int = 0, handle: Handle | None = None, group=None,
                 covariance: int = MP_COV_MATERN, config: dict | None = None):
        self.handle = handle or Handle(device, config=config)
        self.M = Matrix(self.handle, n, nb, None, group=group, attach=self.handle.nranks == 1)
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
        km = None if kernel_prec is None else np.ascontiguousarray(kernel_prec, np.uint8)
        for _ in range(2):
            rep = EvalReport()
            st = lib.mp_eval(self.handle.h, self.M.A, C.c_void_p(_ptr(x)), C.c_void_p(_ptr(y)), C.c_void_p(_ptr(z)),
                             int(on_host), _d(th), float(u_req), _d(e), policy, mode, _u8(km), C.byref(rep))
            if st == MP_ERR_NOMEM and self.handle.nranks == 1 and rep.workspace_bytes > self.M.nbytes:
                self.M.attach(rep.workspace_bytes)  # this map needs a larger workspace: grow, repeat
                continue
            break
        if st not in (MP_OK, MP_ERR_NOT_SPD):
            self.handle.check(st)
        return rep
