"""ctypes declarations of libasgd.so (include/asgd.h).  Marshalling only.

The library is loaded from this package directory (built in-tree by
build.py).  There is no fallback: if the shared object is missing the import
of anything that needs it raises.
"""
from __future__ import annotations

import ctypes as C
import os
import re

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libasgd.so")
HEADER = os.path.join(_HERE, "..", "include", "asgd.h")

OK, E_ARG, E_SHAPE, E_CUDA, E_STATE, E_UNSUPPORTED = 0, 1, 2, 3, 4, 5
PREC_FP32, PREC_BF16 = 0, 1
LOSS_SOFTMAX, LOSS_SIGMOID = 0, 1
PEER_HANDLE_BYTES = 160   # ASGD_PEER_HANDLE_BYTES
PROF_NAMES = ["touched", "spmm", "g1", "softmax", "g2", "dh_b1", "b2", "g3", "scatter", "merge"]


class ModelDesc(C.Structure):
    _fields_ = [("F", C.c_int64), ("L", C.c_int64), ("H", C.c_int64), ("precision", C.c_int32),
                ("b_max", C.c_int32), ("max_step_nnz", C.c_int64), ("max_step_labels", C.c_int64),
                ("loss", C.c_int32), ("reserved", C.c_int32)]


class Csr(C.Structure):
    _fields_ = [("row_ptr", C.c_void_p), ("col", C.c_void_p), ("val", C.c_void_p),
                ("lab_ptr", C.c_void_p), ("lab", C.c_void_p), ("n_rows", C.c_int64),
                ("nnz", C.c_int64), ("n_lab", C.c_int64)]


class AsgdError(RuntimeError):
    def __init__(self, fn, code, msg):
        super().__init__(f"{fn} failed ({code}): {msg}")
        self.code = code


_P = C.c_void_p
_i32, _i64, _f32, _f64 = C.c_int32, C.c_int64, C.c_float, C.c_double
_SIGS = {
    "asgd_workspace_bytes": (C.c_size_t, [C.POINTER(ModelDesc)]),
    "asgd_replica_init": (C.c_int, [C.POINTER(_P), C.POINTER(ModelDesc), C.c_int, _P, _P, _P, _P, _P, C.c_size_t]),
    "asgd_replica_destroy": (C.c_int, [_P]),
    "asgd_set_stream": (C.c_int, [_P, _P]),
    "asgd_params_changed": (C.c_int, [_P]),
    "asgd_data_register": (C.c_int, [_P, C.POINTER(Csr)]),
    "asgd_data_upload": (C.c_int, [_P, C.POINTER(Csr), C.POINTER(Csr)]),
    "asgd_data_stage": (C.c_int, [_P, C.POINTER(Csr), C.POINTER(Csr), _P]),
    "asgd_data_use": (C.c_int, [_P, C.POINTER(Csr)]),
    "asgd_local_step": (C.c_int, [_P, _P, _i32, _f32, _P]),
    "asgd_updates": (C.c_int, [_P, C.POINTER(_i64)]),
    "asgd_set_debug_grads": (C.c_int, [_P, _P]),
    "asgd_last_touched": (C.c_int, [_P, _P, _i64, C.POINTER(_i64)]),
    "asgd_replica_sqnorm": (C.c_int, [_P, _P]),
    "asgd_merge_weights": (C.c_int, [_i32, _P, _P, _P, _f64, _f64, _i32, _P, C.POINTER(_i32),
                                     C.POINTER(_i32), C.POINTER(_i32)]),
    "asgd_merge_prescale": (C.c_int, [_P, _f64]),
    "asgd_merge_finish": (C.c_int, [_P, _f32]),
    "asgd_peer_export": (C.c_int, [_P, _P]),
    "asgd_peer_open": (C.c_int, [_P, _i32, _i32, _P]),
    "asgd_merge_fused": (C.c_int, [_P, _P, _f32]),
    "asgd_replicas_weighted_sum": (C.c_int, [_P, _P, _P, _i32, _P]),
    "asgd_scale_batches": (C.c_int, [_i32, _P, _P, _P, _i64, _i64, _i64, _f64]),
    "asgd_sched_open": (C.c_int, [C.c_char_p, _i32, _i64, _i32, C.POINTER(_P)]),
    "asgd_sched_next": (C.c_int, [_P, _i32, _i64, C.POINTER(_i64), C.POINTER(_i64)]),
    "asgd_run_tickets": (C.c_int, [_P, _P, _i32, _i64, _P, _f32, _P, _i64, _i32, C.POINTER(_i64)]),
    "asgd_run_static": (C.c_int, [_P, _i32, _i32, _i64, _P, _i64, _f32, _P, _i64, _i32, C.POINTER(_i64)]),
    "asgd_sched_log": (C.c_int, [_P, _P, _i64, C.POINTER(_i64)]),
    "asgd_sched_reset": (C.c_int, [_P, _i64]),
    "asgd_sched_wait": (C.c_int, [_P, _i64, _i64]),
    "asgd_sched_close": (C.c_int, [_P, _i32]),
    "asgd_route_replay": (C.c_int, [_i32, _i32, _P, _P, _i64, _P, _i64, C.POINTER(_i64)]),
    "asgd_norm_per_param": (C.c_int, [_i32, _P, _i64, _P]),
    "asgd_scale_frequency": (C.c_int, [_i32, _P, _P, _P, _i32, _i32, C.POINTER(_i32)]),
    "asgd_route_static": (C.c_int, [_i32, _i64, _i64, _P, _i64, C.POINTER(_i64)]),
    "asgd_elastic_weights": (C.c_int, [_i32, _P]),
    "asgd_peer_close": (C.c_int, [_P]),
    "asgd_trace_enable": (C.c_int, [_P, _i32]),
    "asgd_trace_read": (C.c_int, [_P, _P, _i64, C.POINTER(_i64)]),
    "asgd_timeline_set": (C.c_int, [_P]),
    "asgd_route_simulate": (C.c_int, [_i32, _P, _i64, _P, _f64, _P, _P, _i64, C.POINTER(_i64)]),
    "asgd_eval_topk": (C.c_int, [_P, C.POINTER(Csr), _P, _i32, _i32, _P]),
    "asgd_precision_at_k": (C.c_int, [_P, _P, _P, _i32, _i32, C.POINTER(_i64)]),
    "asgd_sync": (C.c_int, [_P]),
    "asgd_kernel_launches": (C.c_int, [_P, C.POINTER(_i64)]),
    "asgd_profile": (C.c_int, [_P, _i32]),
    "asgd_profile_read": (C.c_int, [_P, _P, _P]),
    "asgd_copy_to_host": (C.c_int, [_P, _P, _P, C.c_size_t]),
    "asgd_last_error": (C.c_char_p, []),
    "asgd_version": (C.c_char_p, []),
}

_lib = None


def lib():
    """Load libasgd.so (raises if it was not built -- no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_ipps_marws22_b200.build`")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in _SIGS.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def check(fn_name: str, rc: int):
    if rc != OK:
        msg = lib().asgd_last_error().decode(errors="replace")
        raise AsgdError(fn_name, rc, msg)


def call(name: str, *args):
    rc = getattr(lib(), name)(*args)
    check(name, rc)
    return rc


def header_symbols():
    """Function names the public header declares."""
    with open(HEADER) as f:
        src = f.read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(asgd_[a-z0-9_]+)\s*\(", src)))
