"""ctypes mirror of include/pepp_spmv.h (argument marshalling only).

Loads the in-tree ``libpepp_spmv.so``; raises if it is missing — there is no
CPU fallback anywhere on the product path.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libpepp_spmv.so")

PEPP_OK, PEPP_E_INVALID, PEPP_E_CUDA, PEPP_E_NCCL, PEPP_E_NOMEM, PEPP_E_UNSUPPORTED, PEPP_E_STATE = 0, -1, -2, -3, -4, -5, -6
V_AUTO, V_CSR_VECTOR, V_MERGE_PATH, V_SELL, V_CSR_STREAM, V_PANEL, V_COUNT = -1, 0, 1, 2, 3, 4, 5
X_AUTO, X_NONE, X_ALLGATHER, X_HALO, X_P2P = -1, 0, 1, 2, 3
Y_LOCAL, Y_NEXT_INPUT, Y_REPLICATED, EXEC_NO_TIMING = 0x0, 0x1, 0x2, 0x10
ACCESS_READ, ACCESS_WRITE, ACCESS_READWRITE = 1, 2, 3
VALUE_F64, VALUE_F32 = 0, 1
DEVICE_SIMULATED = -2
KEY_F32, KEY_COMPRESS, KEY_DIST = 0x1, 0x2, 0x4
VARIANT_NAMES = {V_CSR_VECTOR: "csr_vector", V_MERGE_PATH: "merge_path", V_SELL: "sell", V_CSR_STREAM: "csr_stream",
                 V_PANEL: "panel"}
EXCHANGE_NAMES = {X_NONE: "none", X_ALLGATHER: "allgather", X_HALO: "halo", X_P2P: "p2p", X_AUTO: "auto"}

c_i32, c_i64, c_u32, c_u64, c_f64, c_vp = (ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_uint64,
                                          ctypes.c_double, ctypes.c_void_p)


class CSR_T(ctypes.Structure):
    _fields_ = [("nrows", c_i64), ("ncols", c_i64), ("nnz", c_i64), ("first", c_i64),
                ("row_ptr", c_vp), ("col_idx", c_vp), ("values", c_vp), ("on_device", c_i32), ("value_type", c_i32)]


class INFO_T(ctypes.Structure):
    _fields_ = [("nrows", c_i64), ("ncols", c_i64), ("nnz", c_i64), ("mean_row", c_f64), ("cv_row", c_f64),
                ("max_row", c_i64), ("empty_rows", c_i64), ("nranks", c_i32), ("rank", c_i32),
                ("row_offset", c_i64), ("key", c_u64), ("ncandidates", c_i32), ("sell_sigma", c_i32),
                ("sell_fill", c_f64), ("device_bytes", c_i64), ("algorithmic_bytes", c_i64),
                ("exchange", c_i32), ("halo_recv", c_i64), ("halo_send", c_i64), ("sell_col16_frac", c_f64),
                ("prior_key", c_u64), ("sell_stencil_frac", c_f64),
                ("overlap", c_i32), ("overlap_head", c_i64), ("overlap_tail", c_i64), ("predicted", c_i32),
                ("sell_constval_frac", c_f64), ("p2p_buffers", c_i32),
                ("sell_long_rows", c_i64), ("sell_cap", c_i64), ("dist_candidates", c_i32),
                ("dist_nparts", c_i32), ("dist_exchange", c_i32), ("dist_repl_nparts", c_i32),
                ("dist_probe_ms", c_f64), ("sell_ptile_frac", c_f64),
                ("sell_tile_multiline", c_i64)]

    def as_dict(self) -> dict:
        return {f: getattr(self, f) for f, _ in self._fields_}


# pepp_predict_fn: double (*)(const pepp_plan_info_t*, int32_t variant, int32_t param, void* user)
PREDICT_FN = ctypes.CFUNCTYPE(c_f64, ctypes.POINTER(INFO_T), c_i32, c_i32, c_vp)


class OPTS_T(ctypes.Structure):
    _fields_ = [("variant_mask", c_u32), ("use_history", c_i32), ("validate", c_i32), ("sell_sigma", c_i32),
                ("device", c_i32), ("min_samples", c_i32), ("sample_period", c_i32), ("nranks", c_i32),
                ("rank", c_i32), ("row_bounds", c_vp), ("nccl_comm", c_vp), ("nccl_unique_id", c_vp),
                ("exchange", c_i32), ("history_path", ctypes.c_char_p), ("prune", c_i32),
                ("overlap", c_i32), ("predict", PREDICT_FN), ("predict_user", c_vp),
                ("compress_values", c_i32), ("dist_select", c_i32)]


class CHOICE_T(ctypes.Structure):
    _fields_ = [("variant", c_i32), ("param", c_i32), ("nparts", c_i32), ("exchange", c_i32),
                ("calibrating", c_i32), ("candidate", c_i32), ("predicted_us", c_f64),
                ("launches", c_i32), ("reserved", c_i32), ("layout_bytes", c_i64)]

    def as_dict(self) -> dict:
        return {"variant": VARIANT_NAMES.get(self.variant, str(self.variant)), "variant_id": self.variant,
                "param": self.param, "nparts": self.nparts, "exchange": EXCHANGE_NAMES.get(self.exchange, "?"),
                "calibrating": bool(self.calibrating), "candidate": self.candidate,
                "predicted_us": self.predicted_us, "launches": self.launches, "layout_bytes": self.layout_bytes}


# (name, restype, argtypes) for every entry point of include/pepp_spmv.h
SIGNATURES = {
    "pepp_status_str": (ctypes.c_char_p, [c_i32]),
    "pepp_spmv_opts_default": (None, [ctypes.POINTER(OPTS_T)]),
    "pepp_spmv_plan": (c_i32, [ctypes.POINTER(CSR_T), ctypes.POINTER(OPTS_T), ctypes.POINTER(c_vp)]),
    "pepp_spmv_select": (c_i32, [c_vp, ctypes.POINTER(CHOICE_T)]),
    "pepp_spmv_exec": (c_i32, [c_vp, c_vp, c_vp, ctypes.c_int, c_vp, ctypes.POINTER(CHOICE_T), ctypes.POINTER(CHOICE_T)]),
    "pepp_spmv_exec_host": (c_i32, [c_vp, c_vp, c_vp, c_i32, ctypes.c_int, c_vp]),
    "pepp_spmv_exec_host_batch": (c_i32, [c_vp, c_i32, c_vp, c_vp, c_i32, ctypes.c_int, c_vp]),
    "pepp_spmv_exchange": (c_i32, [c_vp, c_vp, ctypes.c_int, c_vp]),
    "pepp_spmv_p2p_buffers": (c_i32, [c_vp, c_i32, ctypes.POINTER(c_vp)]),
    "pepp_spmv_destroy": (c_i32, [c_vp]),
    "pepp_spmv_plan_info": (c_i32, [c_vp, ctypes.POINTER(INFO_T)]),
    "pepp_spmv_candidates": (c_i32, [c_vp, ctypes.POINTER(CHOICE_T), c_i32, ctypes.POINTER(c_i32)]),
    "pepp_spmv_flush_history": (c_i32, [c_vp]),
    "pepp_spmv_dist_stats": (c_i32, [c_vp, c_i32, c_vp, c_vp, c_vp, ctypes.POINTER(c_i32)]),
    "pepp_dist_choose": (c_i32, [c_i32, c_i32, c_vp, c_vp, ctypes.POINTER(c_i32), c_vp]),
    "pepp_spmv_history_stats": (c_i32, [c_vp, c_i32, ctypes.POINTER(c_i64), ctypes.POINTER(c_f64), ctypes.POINTER(c_f64)]),
    "pepp_spmv_graph_create": (c_i32, [c_vp, c_vp, c_vp, c_vp, c_i32, c_i32, ctypes.c_int, c_vp, ctypes.POINTER(c_vp)]),
    "pepp_spmv_graph_launch": (c_i32, [c_vp, c_vp]),
    "pepp_spmv_graph_destroy": (c_i32, [c_vp]),
    "pepp_vector_create": (c_i32, [c_i64, c_vp, c_i32, ctypes.POINTER(c_vp)]),
    "pepp_vector_destroy": (c_i32, [c_vp]),
    "pepp_vector_acquire_host": (c_i32, [c_vp, c_i32, ctypes.POINTER(c_vp)]),
    "pepp_vector_acquire_device": (c_i32, [c_vp, c_i32, c_vp, ctypes.POINTER(c_vp)]),
    "pepp_vector_release_device": (c_i32, [c_vp, c_vp]),
    "pepp_vector_counters": (c_i32, [c_vp, ctypes.POINTER(c_i64), ctypes.POINTER(c_i64), ctypes.POINTER(c_i64)]),
    "pepp_vector_state": (c_i32, [c_vp, ctypes.POINTER(c_i32), ctypes.POINTER(c_i32)]),
    "pepp_vector_scale": (c_i32, [c_vp, c_f64, c_vp]),
    "pepp_spmv_exec_vec": (c_i32, [c_vp, c_vp, c_vp, ctypes.c_int, c_vp, ctypes.POINTER(CHOICE_T), ctypes.POINTER(CHOICE_T)]),
    "pepp_partition_rows": (c_i32, [c_vp, c_i64, c_i64, c_i32, c_vp]),
    "pepp_halo_ghosts": (c_i32, [c_vp, c_i64, c_i32, c_i32, c_vp, c_vp, c_vp, c_i64, ctypes.POINTER(c_i64)]),
    "pepp_history_create": (c_i32, [ctypes.POINTER(c_vp)]),
    "pepp_history_destroy": (c_i32, [c_vp]),
    "pepp_history_record": (c_i32, [c_vp, c_u64, c_i32, c_f64]),
    "pepp_history_stats": (c_i32, [c_vp, c_u64, c_i32, ctypes.POINTER(c_i64), ctypes.POINTER(c_f64), ctypes.POINTER(c_f64)]),
    "pepp_history_select": (c_i32, [c_vp, c_u64, c_i32, c_vp, c_i32, ctypes.POINTER(c_i32), ctypes.POINTER(c_i32), ctypes.POINTER(c_f64)]),
    "pepp_history_prior": (c_i32, [c_vp, c_u64, c_i32, c_vp, c_vp, ctypes.POINTER(c_u64)]),
    "pepp_history_save": (c_i32, [c_vp, ctypes.c_char_p]),
    "pepp_history_load": (c_i32, [c_vp, ctypes.c_char_p]),
    "pepp_context_key": (c_u64, [c_i64, c_i64, c_i64, c_f64, c_i32, c_i32]),
    "pepp_nccl_unique_id": (c_i32, [c_vp]),
    "pepp_nccl_selftest": (c_i32, [c_i32]),
    "pepp_abi_version": (c_i32, []),
    "pepp_last_error": (ctypes.c_char_p, []),
}

_lib = None


class PeppError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        detail = ""
        if status == PEPP_E_CUDA:
            try:
                detail = lib().pepp_last_error().decode()
            except Exception:
                pass
        super().__init__(f"{where}: {status_str(status)} ({status})" + (f": {detail}" if detail else ""))


ABI_VERSION = 10   # PEPP_ABI_VERSION of include/pepp_spmv.h


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python build.py` (no CPU fallback exists)")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        if L.pepp_abi_version() != ABI_VERSION:   # the structs below mirror one header version
            raise ImportError(f"{LIB_PATH} has ABI {L.pepp_abi_version()}, the binding expects {ABI_VERSION}: "
                              "rebuild with `python build.py`")
        _lib = L
    return _lib


def status_str(s: int) -> str:
    return lib().pepp_status_str(s).decode()


def check(status: int, where: str) -> None:
    if status != PEPP_OK:
        raise PeppError(status, where)
