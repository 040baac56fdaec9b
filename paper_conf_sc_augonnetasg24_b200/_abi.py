"""ctypes binding of include/stf_cholesky.h -- argument marshalling only.

Every function here has the C name and forwards to libstf_cholesky.so; no step
of the factorisation runs in Python.  Importing this module raises if the
library is missing (there is no CPU fallback).
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("STF_LIB_PATH") or os.path.join(_HERE, "libstf_cholesky.so")  # override: A/B experiments only

STF_DESC_TILED_2DBC = 0
STF_DESC_DEVICE_COLMAJOR = 1
STF_DESC_HOST_COLMAJOR = 2

KIND_NAMES = {0: "POTRF", 1: "TRSM", 2: "SYRK", 3: "GEMM", 4: "COPY", 5: "LOAD", 6: "STORE", 7: "FENCE"}


class stf_matrix_desc(ctypes.Structure):
    _fields_ = [
        ("kind", ctypes.c_int32),
        ("device", ctypes.c_int32),
        ("ld", ctypes.c_int64),
        ("ptr", ctypes.c_void_p),
        ("p", ctypes.c_int32),
        ("q", ctypes.c_int32),
        ("tiles", ctypes.POINTER(ctypes.c_void_p)),
    ]


class stf_plan_stats(ctypes.Structure):
    _fields_ = [
        ("tasks", ctypes.c_int64),
        ("transfers", ctypes.c_int64),
        ("edges", ctypes.c_int64),
        ("transfer_bytes", ctypes.c_int64),
        ("critical_path", ctypes.c_int64),
        ("graph_nodes", ctypes.c_int64),
        ("kernel_launches", ctypes.c_int64),
        ("build_ms", ctypes.c_double),
        ("device_ms", ctypes.c_double),
        ("graph_reuse", ctypes.c_int64),
        ("dag_tasks", ctypes.c_int64),
        ("host_loads", ctypes.c_int64),
        ("host_stores", ctypes.c_int64),
        ("frames", ctypes.c_int64),
        ("pushed", ctypes.c_int64),
        ("replicas_max", ctypes.c_int64),
        ("data_plane", ctypes.c_int64),
        ("graph_fallback", ctypes.c_int64),
        ("graph", ctypes.c_int64),
        ("devices", ctypes.c_int64),
        ("slots", ctypes.c_int64),
        ("peer_transfers", ctypes.c_int64),
        ("merged_gemms", ctypes.c_int64),
        ("pdl_edges", ctypes.c_int64),
    ]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


# Every symbol include/stf_cholesky.h declares (checked by tests/test_abi.py) ...
EXPORTS = [
    "stf_cholesky_init", "stf_potrf", "stf_finalize", "stf_last_error",
    "stf_set_option", "stf_get_option", "stf_last_stats", "stf_dag_build", "stf_dag_build_call", "stf_infer_edges",
    "stf_dag_tasks_io", "stf_dag_tasks_io2", "stf_dag_tasks_mirrors", "stf_mp_init", "stf_mp_blob_size", "stf_mp_prepare", "stf_mp_import", "stf_mp_potrf",
]
# ... and every symbol include/stf_harness.h declares (test / benchmark entry points).
HARNESS_EXPORTS = [
    "stf_fill_spd_tiles", "stf_fill_spd_block",
    "stf_kernel_gemm_nt", "stf_kernel_trsm", "stf_kernel_potrf", "stf_bench_kernel", "stf_debug_potrf_trace",
    "stf_debug_last_trace", "stf_debug_trsm_trace",
]

if not os.path.exists(LIB_PATH):
    raise ImportError(
        "libstf_cholesky.so not built (%s); run `python -m paper_conf_sc_augonnetasg24_b200.build` "
        "or __graft_entry__.build() -- there is no CPU fallback" % LIB_PATH)

lib = ctypes.CDLL(LIB_PATH)

_i64, _i32, _int, _vp, _dbl = ctypes.c_int64, ctypes.c_int32, ctypes.c_int, ctypes.c_void_p, ctypes.c_double
_P = ctypes.POINTER


def _decl(name, restype, argtypes):
    f = getattr(lib, name)
    f.restype = restype
    f.argtypes = argtypes
    return f


stf_cholesky_init = _decl("stf_cholesky_init", _int, [_int, _P(_int)])
stf_potrf = _decl("stf_potrf", _int, [_i64, _i64, ctypes.c_char, _P(stf_matrix_desc), _int])
stf_finalize = _decl("stf_finalize", _int, [])
stf_last_error = _decl("stf_last_error", ctypes.c_char_p, [])
stf_set_option = _decl("stf_set_option", _int, [ctypes.c_char_p, _i64])
stf_get_option = _decl("stf_get_option", _int, [ctypes.c_char_p, _P(_i64)])
stf_last_stats = _decl("stf_last_stats", _int, [_P(stf_plan_stats)])
stf_dag_build = _decl("stf_dag_build", _int, [_i64, _int, _int, _i64, _P(_i64), _i64, _P(_i32), _P(_i64),
                                              _P(stf_plan_stats)])
stf_dag_build_call = _decl("stf_dag_build_call", _int, [_i64, _i64, _int, _int, _int, _int, _int, _i64, _P(_i64), _i64,
                                                        _P(_i32), _P(_i64), _P(stf_plan_stats)])
stf_infer_edges = _decl("stf_infer_edges", _i64, [_i64, _P(_i32), _P(_i64), _P(_i32), _i64, _P(_i64)])
stf_fill_spd_tiles = _decl("stf_fill_spd_tiles", _int, [_i64, _i64, _P(stf_matrix_desc), _int, ctypes.c_uint64])
stf_fill_spd_block = _decl("stf_fill_spd_block", _int, [_vp, _i64, _i64, _i64, _i64, _i64, _i64, ctypes.c_uint64])
stf_kernel_gemm_nt = _decl("stf_kernel_gemm_nt", _int, [_i64, _i64, _i64, _vp, _i64, _vp, _i64, _vp, _i64, _int])
stf_kernel_trsm = _decl("stf_kernel_trsm", _int, [_i64, _i64, _vp, _i64, _vp, _i64])
stf_kernel_potrf = _decl("stf_kernel_potrf", _int, [_i64, _vp, _i64, _P(_i64)])
stf_bench_kernel = _decl("stf_bench_kernel", _int, [_int, _i64, _i64, _i64, _int, _P(_dbl)])
stf_dag_tasks_io = _decl("stf_dag_tasks_io", _int, [_i64, _P(_i64)])
stf_dag_tasks_mirrors = _decl("stf_dag_tasks_mirrors", _i64, [_i64, _P(_i64)])
stf_dag_tasks_io2 = _decl("stf_dag_tasks_io2", _i64, [_i64, _P(_i64)])
stf_mp_init = _decl("stf_mp_init", _int, [_int, _int, _int])
stf_mp_blob_size = _decl("stf_mp_blob_size", _i64, [])
stf_mp_prepare = _decl("stf_mp_prepare", _int, [_i64, _i64, _P(stf_matrix_desc), _vp])
stf_mp_import = _decl("stf_mp_import", _int, [_vp])
stf_mp_potrf = _decl("stf_mp_potrf", _int, [])
stf_debug_last_trace = _decl("stf_debug_last_trace", _i64, [_P(_i64), _i64])
stf_debug_potrf_trace = _decl("stf_debug_potrf_trace", _i64, [_i64, _vp, _i64, _int, _P(_i64), _i64])
stf_debug_trsm_trace = _decl("stf_debug_trsm_trace", _i64, [_i64, _i64, _vp, _i64, _vp, _i64, _P(_i64), _i64])


class StfError(RuntimeError):
    def __init__(self, code: int, where: str):
        msg = stf_last_error().decode(errors="replace")
        super().__init__("%s returned %d: %s" % (where, code, msg))
        self.code = code


def check(code: int, where: str) -> int:
    if code < 0:
        raise StfError(code, where)
    return code
