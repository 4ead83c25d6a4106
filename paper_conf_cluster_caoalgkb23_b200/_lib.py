"""ctypes binding of libmpgeo.so (include/mpgeo.h): argument marshalling only.

Every step of the path runs in the library's CUDA kernels; nothing here computes.
If the shared library is missing this module raises at import — there is no CPU
fallback (the CPU oracle under oracle/ is test infrastructure, never imported here).
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmpgeo.so")

MP_OK, MP_ERR_ARG, MP_ERR_NOT_SPD, MP_ERR_CUDA, MP_ERR_COMM, MP_ERR_NOMEM, MP_ERR_UNSUPPORTED, MP_ERR_STATE = range(8)
STATUS_NAMES = ["MP_OK", "MP_ERR_ARG", "MP_ERR_NOT_SPD", "MP_ERR_CUDA", "MP_ERR_COMM", "MP_ERR_NOMEM",
                "MP_ERR_UNSUPPORTED", "MP_ERR_STATE"]
MP_FP64, MP_FP32, MP_FP16, MP_FP16H = 0, 1, 2, 3  # MP_FP16 = FP16_32; MP_FP16H = pure FP16 (four-level maps)
MP_COMM_TTC, MP_COMM_AUTO = 0, 1
MP_MAP_ADAPTIVE, MP_MAP_FP64, MP_MAP_BAND, MP_MAP_EXTREME, MP_MAP_USER, MP_MAP_ADAPTIVE4 = range(6)
MP_EPS_FP16_32 = 1.0 / 16384.0  # include/mpgeo.h (reading C7')
MP_COV_MATERN, MP_COV_SQEXP = 0, 1
MP_F64_CRT16, MP_F64_DMMA = 0, 1
MP_F32_3XFP16, MP_F32_3XTF32, MP_F32_DMMA = 0, 1, 2


class EvalReport(C.Structure):
    _fields_ = [
        ("loglik", C.c_double), ("logdet", C.c_double), ("quad", C.c_double),
        ("info", C.c_int64),
        ("t_gen_ms", C.c_double), ("t_map_ms", C.c_double), ("t_potrf_ms", C.c_double),
        ("t_solve_ms", C.c_double), ("t_total_ms", C.c_double),
        ("flops_potrf", C.c_double), ("flops_update", C.c_double * 3),
        ("tiles", C.c_int64 * 3), ("stc_tiles", C.c_int64), ("gpu_launches", C.c_int64),
        ("workspace_bytes", C.c_uint64),
        ("tiles_fp16h", C.c_int64), ("flops_update_fp16h", C.c_double),
    ]


class Config(C.Structure):
    """mp_config (include/mpgeo.h): engines and schedule switches of a handle."""
    _fields_ = [("fp64_engine", C.c_int), ("fp32_engine", C.c_int), ("fp16_tensor", C.c_int), ("lookahead", C.c_int),
                ("reserve_pairs", C.c_int), ("lowp_trsm_product", C.c_int), ("matern_table", C.c_int),
                ("f16x3_persistent", C.c_int), ("crt_phase_lock", C.c_int), ("fp16_storage", C.c_int)]

    def as_dict(self):
        return {name: getattr(self, name) for name, _ in self._fields_}


PROF_CLASSES = ["upd_fp64", "upd_fp32", "upd_fp16", "potrf", "trsm", "convert", "generate", "solve"]


class Profile(C.Structure):
    _fields_ = [("ms", C.c_double * 8), ("flops", C.c_double * 8), ("launches", C.c_int64 * 8)]

    def as_dict(self):
        return {name: {"ms": self.ms[i], "flops": self.flops[i], "launches": int(self.launches[i])}
                for i, name in enumerate(PROF_CLASSES)}


class Xfer(C.Structure):
    _fields_ = [("k", C.c_int32), ("m", C.c_int32), ("peer", C.c_int32), ("prec", C.c_int32), ("dir", C.c_int32)]


class MpError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES[status] if 0 <= status < len(STATUS_NAMES) else status}: {msg}")
        self.status = status


def _load() -> C.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() (make -C {_HERE}); "
                          "there is no CPU fallback")
    lib = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
    vp, i32, i64, dbl, u8p, dp = C.c_void_p, C.c_int, C.c_int64, C.c_double, C.POINTER(C.c_uint8), C.POINTER(C.c_double)
    sig = {
        "mp_init": (i32, [i32, i32, i32, i32, i32, u8p, vp, C.POINTER(vp)]),
        "mp_init_config": (i32, [i32, i32, i32, i32, i32, u8p, vp, C.POINTER(Config), C.POINTER(vp)]),
        "mp_config_default": (None, [C.POINTER(Config)]),
        "mp_handle_get_config": (i32, [vp, C.POINTER(Config)]),
        "mp_get_unique_id": (i32, [u8p]),
        "mp_matrix_attach": (i32, [vp, vp, C.c_size_t]),
        "mp_matrix_engines": (i32, [vp, C.POINTER(i32), C.POINTER(i32), C.POINTER(i32), C.POINTER(i32)]),
        "mp_finalize": (i32, [vp]),
        "mp_last_error": (C.c_char_p, [vp]),
        "mp_matrix_create": (i32, [vp, i64, i32, C.POINTER(vp)]),
        "mp_matrix_destroy": (i32, [vp]),
        "mp_matrix_bytes": (i32, [vp, u8p, C.POINTER(C.c_size_t)]),
        "mp_matrix_bind": (i32, [vp, u8p, vp, C.c_size_t]),
        "mp_matern_gen": (i32, [vp, vp, vp, vp, dp, u8p, dp]),
        "mp_precision_map": (i32, [i32, dp, dbl, dp, i32, u8p, u8p, u8p]),
        "mp_precision_map4": (i32, [i32, dp, dbl, dp, i32, u8p, u8p, u8p]),
        "mp_tile_potrf": (i32, [vp, vp, u8p, u8p, C.POINTER(i64)]),
        "mp_loglik": (i32, [vp, vp, vp, dp, dp, dp]),
        "mp_gp_sample": (i32, [vp, vp, vp, vp]),
        "mp_eval": (i32, [vp, vp, vp, vp, vp, i32, dp, dbl, dp, i32, i32, u8p, C.POINTER(EvalReport)]),
        "mp_matrix_maps": (i32, [vp, u8p, u8p, u8p]),
        "mp_matrix_get_tile": (i32, [vp, vp, i32, i32, dp]),
        "mp_matrix_set_tile": (i32, [vp, vp, i32, i32, dp]),
        "mp_matrix_set_covariance": (i32, [vp, i32]),
        "mp_matrix_comm_export": (i32, [vp, vp]),
        "mp_matrix_comm_connect": (i32, [vp, vp]),
        "mp_exchange_plan": (i32, [i32, i32, i32, i32, u8p, C.POINTER(Xfer), i64, C.POINTER(i64)]),
        "mp_matrix_nt": (i32, [vp]),
        "mp_matrix_owner": (i32, [vp, i32, i32]),
        "mp_launch_count": (i64, [vp]),
        "mp_set_profiling": (i32, [vp, i32]),
        "mp_set_profiling_mask": (i32, [vp, C.c_uint]),
        "mp_get_profile": (i32, [vp, C.POINTER(Profile)]),
        "mp_version": (C.c_char_p, []),
        "mpgeo_exact_sum": (dbl, [dp, i64]),
        "mp_test_bessel_k": (i32, [dbl, vp, vp, i32]),
        "mp_test_dgemm": (i32, [vp, vp, vp, i32, i32, i32, i32, i32, i32, i32, dbl, dbl, i32, i32]),
        "mp_test_tc_gemm": (i32, [i32, vp, vp, vp, i32, i32, i32, i32]),
        "mp_test_tc_gemm_split": (i32, [i32, vp, vp, i32, i32, i32, i32, i32]),
        "mp_tc_available": (i32, []),
        "mp_test_crt_gemm": (i32, [vp, vp, i32, i32, i32, i32, i32, i32, i32]),
        "mp_bench_fp64_engine": (i32, [i32, i32, i32, i32, i32, C.POINTER(C.c_float)]),
        "mp_test_crt_constants": (i32, [i32, i32, C.POINTER(i32), C.POINTER(i32), dp, dp, dp]),
        "mp_test_crt_recon": (i32, [i32, i32, C.POINTER(C.c_uint32), C.POINTER(i32), i32, i32, dp]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


lib = _load()
