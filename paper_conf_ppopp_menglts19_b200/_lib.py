"""ctypes declarations of the C ABI in include/gsw.h (argument marshalling only).

The CUDA library ``libgsw.so`` must exist next to this file; there is no fallback of any kind:
importing this module without it raises ImportError.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GSW_LIB_PATH") or os.path.join(_HERE, "libgsw.so")   # override: A/B builds

# ---- enums (include/gsw.h) ----------------------------------------------------------------
GSW_OK, GSW_EINVAL, GSW_ENOMEM, GSW_ECUDA, GSW_ENCCL, GSW_EUNSUPPORTED, GSW_EOVERFLOW = range(7)
STATUS_NAMES = ["GSW_OK", "GSW_EINVAL", "GSW_ENOMEM", "GSW_ECUDA", "GSW_ENCCL", "GSW_EUNSUPPORTED",
                "GSW_EOVERFLOW"]
AUTO = 0
PUSH, PULL = 1, 2
BITMAP, QUEUE, SORTED_QUEUE = 1, 2, 3
LB_THREAD, LB_TWC, LB_WM, LB_CM, LB_STRICT = 1, 2, 3, 4, 5
STEP_INCREASE, STEP_DECREASE, STEP_REMAIN, STEP_STATIC, STEP_UNORDERED = 1, 2, 3, 4, 5
STANDALONE, FUSED = 1, 2

DIRECTIONS = {"push": PUSH, "pull": PULL}
FORMATS = {"bitmap": BITMAP, "queue": QUEUE, "sorted_queue": SORTED_QUEUE}
LOAD_BALANCES = {"thread": LB_THREAD, "twc": LB_TWC, "wm": LB_WM, "cm": LB_CM, "strict": LB_STRICT}
STEPPINGS = {"increase": STEP_INCREASE, "decrease": STEP_DECREASE, "remain": STEP_REMAIN,
             "static": STEP_STATIC, "unordered": STEP_UNORDERED}
FUSIONS = {"standalone": STANDALONE, "fused": FUSED}


class gsw_csr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("row_offsets", ctypes.c_void_p),
                ("col_indices", ctypes.c_void_p), ("weights", ctypes.c_void_p)]


class gsw_config(ctypes.Structure):
    _fields_ = [("direction", ctypes.c_int32), ("format", ctypes.c_int32),
                ("load_balance", ctypes.c_int32), ("stepping", ctypes.c_int32),
                ("fusion", ctypes.c_int32), ("delta0", ctypes.c_uint32)]


class gsw_iter_record(ctypes.Structure):
    _fields_ = [("iteration", ctypes.c_int32), ("direction", ctypes.c_int32), ("format", ctypes.c_int32),
                ("load_balance", ctypes.c_int32), ("stepping", ctypes.c_int32), ("fusion", ctypes.c_int32),
                ("Va", ctypes.c_int64), ("Ea", ctypes.c_int64), ("Via", ctypes.c_int64),
                ("Eia", ctypes.c_int64), ("edges", ctypes.c_int64), ("theta", ctypes.c_uint32),
                ("filter_us", ctypes.c_float), ("expand_us", ctypes.c_float), ("ctas", ctypes.c_int32)]


class gsw_run_stats(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_int32), ("gpu_ms", ctypes.c_float),
                ("edges_touched", ctypes.c_int64), ("bytes_alg", ctypes.c_int64),
                ("records", ctypes.POINTER(gsw_iter_record)), ("max_records", ctypes.c_int32)]


# every symbol include/gsw.h declares: name -> (restype, argtypes)
_P = ctypes.c_void_p
# host-staged exchange callbacks (include/gsw.h gsw_exchange)
ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, _P, _P, _P, ctypes.c_size_t)
ALLREDUCE_U64_FN = ctypes.CFUNCTYPE(ctypes.c_int, _P, ctypes.POINTER(ctypes.c_uint64), ctypes.c_size_t)
ALLREDUCE_F64_FN = ctypes.CFUNCTYPE(ctypes.c_int, _P, ctypes.POINTER(ctypes.c_double), ctypes.c_size_t)


class gsw_exchange(ctypes.Structure):
    _fields_ = [("user", _P), ("allgather", ALLGATHER_FN), ("allreduce_u64", ALLREDUCE_U64_FN),
                ("allreduce_f64", ALLREDUCE_F64_FN)]


SIGNATURES = {
    "gsw_workspace_size": (ctypes.c_int, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                          ctypes.POINTER(ctypes.c_size_t)]),
    "gsw_graph_create": (ctypes.c_int, [ctypes.POINTER(gsw_csr), ctypes.POINTER(gsw_csr), _P, ctypes.c_size_t,
                                        _P, ctypes.POINTER(_P)]),
    "gsw_graph_destroy": (ctypes.c_int, [_P]),
    "gsw_graph_validate": (ctypes.c_int, [_P]),
    "gsw_graph_attributes": (ctypes.c_int, [_P, ctypes.POINTER(ctypes.c_double)]),
    "gsw_force_config": (ctypes.c_int, [_P, ctypes.POINTER(gsw_config)]),
    "gsw_bfs": (ctypes.c_int, [_P, ctypes.c_int32, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_sssp": (ctypes.c_int, [_P, ctypes.c_int32, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_cc": (ctypes.c_int, [_P, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_cc_hook": (ctypes.c_int, [_P, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_pr": (ctypes.c_int, [_P, ctypes.c_double, ctypes.c_int32, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_dpr": (ctypes.c_int, [_P, ctypes.c_double, ctypes.c_double, ctypes.c_int32, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_bc": (ctypes.c_int, [_P, _P, ctypes.c_int32, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_app_bfs": (ctypes.c_int, [_P, ctypes.c_int32, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_app_sssp": (ctypes.c_int, [_P, ctypes.c_int32, _P, ctypes.POINTER(gsw_run_stats)]),
    "gsw_dist_slice": (ctypes.c_int64, [ctypes.c_int64, ctypes.c_int32]),
    "gsw_dist_unique_id": (ctypes.c_int, [_P]),
    "gsw_dist_workspace_size": (ctypes.c_int, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int32,
                                               ctypes.POINTER(ctypes.c_size_t)]),
    "gsw_graph_create_dist": (ctypes.c_int, [ctypes.POINTER(gsw_csr), ctypes.c_int64, _P, ctypes.c_int32,
                                             ctypes.c_int32, _P, ctypes.c_size_t, _P, ctypes.POINTER(_P)]),
    "gsw_dist_workspace_size_weighted": (ctypes.c_int, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                                        ctypes.c_int32, ctypes.POINTER(ctypes.c_size_t)]),
    "gsw_graph_create_dist_host": (ctypes.c_int, [ctypes.POINTER(gsw_csr), ctypes.c_int64,
                                                  ctypes.POINTER(gsw_exchange), ctypes.c_int32, ctypes.c_int32, _P,
                                                  ctypes.c_size_t, _P, ctypes.POINTER(_P)]),
    "gsw_dist_loopback_workspace_size": (ctypes.c_int, [ctypes.c_int64, ctypes.c_int64, ctypes.c_int32,
                                                        ctypes.POINTER(ctypes.c_size_t)]),
    "gsw_graph_create_partitioned": (ctypes.c_int, [ctypes.POINTER(gsw_csr), ctypes.c_int32, _P, ctypes.c_size_t,
                                                    _P, ctypes.POINTER(_P)]),
    "gsw_last_error": (ctypes.c_char_p, []),
    "gsw_version": (ctypes.c_char_p, []),
}

_lib = None


def load() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build the CUDA library first "
                              "(python -c 'import __graft_entry__ as g; g.build()'); there is no fallback")
        lib = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(lib, name)
            fn.restype = res
            fn.argtypes = args
        _lib = lib
    return _lib


class GswError(RuntimeError):
    def __init__(self, status: int, where: str):
        msg = load().gsw_last_error().decode(errors="replace")
        name = STATUS_NAMES[status] if 0 <= status < len(STATUS_NAMES) else str(status)
        super().__init__(f"{where}: {name}: {msg}")
        self.status = status


def check(status: int, where: str) -> None:
    if status != GSW_OK:
        raise GswError(status, where)
