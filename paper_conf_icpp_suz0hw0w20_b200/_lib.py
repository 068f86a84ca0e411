"""ctypes binding of libsptrsv.so (include/sptrsv.h) -- argument marshalling only.

Every step of the solve runs in the CUDA kernels of libsptrsv.so.  There is no
CPU fallback: if the library is missing this module raises at import time.
"""
from __future__ import annotations

import ctypes
import os

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG, "libsptrsv.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python -m paper_conf_icpp_suz0hw0w20_b200.build` "
        "(or __graft_entry__.build()); there is no CPU fallback")

lib = ctypes.CDLL(LIB_PATH)

# status codes (include/sptrsv.h)
OK = 0
ERR_INVALID_ARG = -1
ERR_NOT_LOWER = -2
ERR_MISSING_DIAG = -3
ERR_ZERO_DIAG = -4
ERR_UNSORTED = -5
ERR_BAD_ROWPTR = -6
ERR_BAD_COL = -7
ERR_TOO_LARGE = -8

# triangular forms of sptrsv_analyse_csr_ex
TRI_UPPER = 1
TRI_UNIT_DIAG = 2
ERR_CUDA = -9
ERR_ALLOC = -10
ERR_TIMEOUT = -11
ERR_STALE_LAUNCH = -12
ERR_INEXACT = -13

# options
OPT_MODE = 1
OPT_WARP_THRESHOLD = 2
OPT_CTA_THREADS = 3
OPT_BACKOFF_MIN_NS = 4
OPT_BACKOFF_MAX_NS = 5
OPT_SPIN_LIMIT = 6
OPT_L2_WINDOW = 7
OPT_STAGE_SMEM = 8
OPT_PROTOCOL = 9
OPT_LOCAL = 10
OPT_ENGINE = 11
OPT_ROWS_PER_LANE = 15
OPT_VARIANT = 16
OPT_LEAN_OCCUPANCY = 17
OPT_POLL_GAP_NS = 19
OPT_POLL_ONE = 20
OPT_WARP_SPLIT_LAST = 22
OPT_HOST_IO = 23
OPT_SUBWARP = 24
OPT_CHAIN_DIV = 25
(ENGINE_ONESHOT, ENGINE_LEAN, ENGINE_AUTO, ENGINE_HYBRID, ENGINE_CHAIN, ENGINE_SMALL, ENGINE_LEANP,
 ENGINE_GRID) = 0, 3, 5, 6, 7, 8, 9, 10
PROTO_FLAGS, PROTO_FUSED = 0, 1
MODE_AUTO, MODE_THREAD, MODE_WARP, MODE_SUBWARP = 0, 1, 2, 3


class sptrsv_info(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_int32),
        ("n_thread_groups", ctypes.c_int32),
        ("nnz", ctypes.c_int64),
        ("n_warp_rows", ctypes.c_int32),
        ("n_tasks", ctypes.c_int32),
        ("max_row_nnz", ctypes.c_int32),
        ("device", ctypes.c_int32),
        ("analyse_ms", ctypes.c_float),
        ("solves", ctypes.c_uint32),
        ("near_deps", ctypes.c_int64),
        ("warp_deps", ctypes.c_int64),
        ("engine", ctypes.c_int32),
        ("cta_threads", ctypes.c_int32),
        ("rows_per_lane", ctypes.c_int32),
        ("prev_deps", ctypes.c_int64),
        ("n_sub_tasks", ctypes.c_int32),
        ("pad_", ctypes.c_int32),
        ("near_rows", ctypes.c_int64),
    ]


_h = ctypes.c_void_p
_p = ctypes.c_void_p
_i32, _i64 = ctypes.c_int32, ctypes.c_int64

EXPORTS = {
    "sptrsv_analyse_csr": (ctypes.c_int, [_i32, _p, _p, _p, ctypes.POINTER(_h)]),
    "sptrsv_analyse_csr_ex": (ctypes.c_int, [_i32, _p, _p, _p, _i32, ctypes.POINTER(_h)]),
    "sptrsv_analyse_csr_batch": (ctypes.c_int, [_i32, _p, _p, _p, _p, _i32, ctypes.POINTER(_h)]),
    "sptrsv_solve": (ctypes.c_int, [_h, _p, _p, _p]),
    "sptrsv_solve_host": (ctypes.c_int, [_h, _p, _p, _p]),
    "sptrsv_solve_multi": (ctypes.c_int, [_h, _p, _p, _i32, _i64, _i64, _p]),
    "sptrsv_destroy": (ctypes.c_int, [_h]),
    "sptrsv_set_option": (ctypes.c_int, [_h, ctypes.c_int, _i64]),
    "sptrsv_get_option": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(_i64)]),
    "sptrsv_get_info": (ctypes.c_int, [_h, ctypes.POINTER(sptrsv_info)]),
    "sptrsv_get_indegree": (ctypes.c_int, [_h, _p, _p]),
    "sptrsv_levels": (ctypes.c_int, [_h, _p, _p, ctypes.POINTER(_i32), _p]),
    "sptrsv_check": (ctypes.c_int, [_h, _p]),
    "sptrsv_set_trace": (ctypes.c_int, [_h, _p]),
    "sptrsv_flag_latency": (ctypes.c_int, [_i32, _i32, ctypes.POINTER(ctypes.c_double),
                                           ctypes.POINTER(ctypes.c_double)]),
    "sptrsv_hop_scan": (ctypes.c_int, [_i32, _i32, _i32, ctypes.POINTER(_i32), _p, _p, ctypes.POINTER(_i32)]),
    "sptrsv_strerror": (ctypes.c_char_p, [ctypes.c_int]),
    "sptrsv_abi_version": (ctypes.c_int, []),
}

for _name, (_res, _args) in EXPORTS.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args


class SptrsvError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        self.status = status
        msg = lib.sptrsv_strerror(status).decode()
        super().__init__(f"{what}: {msg} (status {status})" if what else f"{msg} (status {status})")


def check(status: int, what: str = "") -> None:
    if status != OK:
        raise SptrsvError(status, what)
