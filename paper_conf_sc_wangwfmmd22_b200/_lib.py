"""ctypes declarations of include/ttemb.h and the loader of the in-tree libttemb.so.

There is no fallback: if the library is missing or fails to load, importing the
binding raises.  Every step of the hot path runs in the CUDA kernels behind
this ABI; Python only marshals arguments.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libttemb.so")

TTEMB_OK = 0
TTEMB_ERR_INVALID_ARG = -1
TTEMB_ERR_UNSUPPORTED = -2
TTEMB_ERR_INDEX_RANGE = -3
TTEMB_ERR_STATE = -4
TTEMB_ERR_CUDA = -5
TTEMB_ERR_CAPACITY = -6
TTEMB_SGD = 0
TTEMB_ADAGRAD = 1
TTEMB_FUSED_UPDATE = 1
TTEMB_FP32_CORES = 2
TTEMB_NO_PREFIX_REUSE = 4
TTEMB_NO_AGGREGATION = 8
TTEMB_MEAN_POOLING = 16

SYMBOLS = ["ttemb_query_sizes", "ttemb_create", "ttemb_destroy", "ttemb_core_layout",
           "ttemb_forward", "ttemb_backward", "ttemb_update", "ttemb_forward_host",
           "ttemb_backward_host", "ttemb_check", "ttemb_get_plan", "ttemb_read_counts",
           "ttemb_set_timing", "ttemb_stage_times", "ttemb_stage_name", "ttemb_status_string",
           "ttemb_set_bijection", "ttemb_total_rows", "ttemb_forward_weighted", "ttemb_plan_batch",
           "ttemb_forward_planned", "ttemb_update_range", "ttemb_grad_buckets", "ttemb_set_bucket_events", "ttemb_louvain",
           "ttemb_ht_cache_init", "ttemb_ht_sync", "ttemb_ht_pool", "ttemb_ht_grad", "ttemb_ht_tick",
           "ttemb_ht_update_push", "ttemb_ht_cache_stats", "ttemb_ht_host_gather", "ttemb_ht_host_sgd"]


class ttemb_ht_cache(C.Structure):
    _fields_ = [("index", C.c_void_p), ("rows", C.c_void_p), ("lc", C.c_void_p), ("owner", C.c_void_p),
                ("free_list", C.c_void_p), ("top", C.c_void_p), ("n_rows", C.c_int64),
                ("capacity", C.c_int32), ("dim", C.c_int32)]


class ttemb_table(C.Structure):
    _fields_ = [("num_rows", C.c_int64), ("row_factors", C.c_int32 * 3), ("dense", C.c_int32)]


class ttemb_config(C.Structure):
    _fields_ = [("num_tables", C.c_int32), ("tables", C.POINTER(ttemb_table)),
                ("num_cores", C.c_int32), ("dim", C.c_int32), ("col_factors", C.c_int32 * 3),
                ("rank", C.c_int32), ("index_bits", C.c_int32), ("max_batch", C.c_int32),
                ("max_nnz", C.c_int64), ("optimizer", C.c_int32), ("adagrad_eps", C.c_float),
                ("flags", C.c_uint32)]


_u32p = C.POINTER(C.c_uint32)


class ttemb_plan(C.Structure):
    _fields_ = [("nnz", C.c_int64), ("batch", C.c_int32)] + [
        (n, C.c_void_p) for n in ["counts", "skey", "spos", "bag_of", "ukey", "seg_off", "inverse",
                                  "row_pfx", "row_i3", "pfx_t", "pfx_i1", "pfx_i2", "row_seg",
                                  "grp_pfx", "grp_off", "grp_t", "grp_i2", "rows"]]


class TTEmbError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        self.code = code
        msg = status_string(code) if _lib is not None else str(code)
        super().__init__(f"{what}: {msg} ({code})" if what else f"{msg} ({code})")


_lib = None


def load(path: str = LIB_PATH):
    """Load libttemb.so (raises if it is missing: no CPU fallback exists)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"libttemb.so not built at {path}; run __graft_entry__.build() "
                          "or python -m paper_conf_sc_wangwfmmd22_b200.build")
    lib = C.CDLL(path)
    vp, i64, i32, f32 = C.c_void_p, C.c_int64, C.c_int32, C.c_float
    sz = C.POINTER(C.c_size_t)
    lib.ttemb_query_sizes.argtypes = [C.POINTER(ttemb_config), sz, sz, sz, sz]
    lib.ttemb_create.argtypes = [C.POINTER(ttemb_config), C.c_int, vp, vp, vp, vp, C.POINTER(vp)]
    lib.ttemb_destroy.argtypes = [vp]
    lib.ttemb_core_layout.argtypes = [vp, C.c_int, C.c_int, C.POINTER(i64), C.POINTER(i32)]
    lib.ttemb_forward.argtypes = [vp, vp, vp, i64, i32, vp, vp]
    lib.ttemb_backward.argtypes = [vp, vp, f32, vp]
    lib.ttemb_update.argtypes = [vp, f32, vp]
    lib.ttemb_forward_host.argtypes = [vp, vp, vp, i64, i32, vp, vp]
    lib.ttemb_backward_host.argtypes = [vp, vp, f32, vp]
    lib.ttemb_check.argtypes = [vp, vp]
    lib.ttemb_get_plan.argtypes = [vp, C.POINTER(ttemb_plan)]
    lib.ttemb_read_counts.argtypes = [vp, C.POINTER(i64), vp]
    lib.ttemb_set_timing.argtypes = [vp, C.c_int]
    lib.ttemb_stage_times.argtypes = [vp, C.POINTER(C.c_double), C.POINTER(i64), C.c_int]
    lib.ttemb_stage_name.argtypes = [C.c_int]
    lib.ttemb_stage_name.restype = C.c_char_p
    lib.ttemb_status_string.argtypes = [C.c_int]
    lib.ttemb_status_string.restype = C.c_char_p
    lib.ttemb_set_bijection.argtypes = [vp, vp]
    lib.ttemb_forward_weighted.argtypes = [vp, vp, vp, vp, i64, i32, vp, vp]
    lib.ttemb_plan_batch.argtypes = [vp, vp, vp, vp, i64, i32, vp]
    lib.ttemb_forward_planned.argtypes = [vp, vp, vp]
    lib.ttemb_total_rows.argtypes = [vp]
    lib.ttemb_update_range.argtypes = [vp, f32, i64, i64, vp]
    lib.ttemb_grad_buckets.argtypes = [vp, C.POINTER(i64), C.POINTER(i64), C.c_int]
    lib.ttemb_set_bucket_events.argtypes = [vp, C.POINTER(vp), C.c_int]
    lib.ttemb_louvain.argtypes = [i64, i64, C.POINTER(i64), C.POINTER(i64), C.POINTER(C.c_double), C.POINTER(i64)]
    hc = C.POINTER(ttemb_ht_cache)
    lib.ttemb_ht_cache_init.argtypes = [hc, vp]
    lib.ttemb_ht_sync.argtypes = [hc, vp, i64, vp, vp]
    lib.ttemb_ht_pool.argtypes = [vp, vp, vp, i32, i32, i32, vp, vp]
    lib.ttemb_ht_grad.argtypes = [vp, vp, vp, i64, i32, i32, i32, vp, vp]
    lib.ttemb_ht_tick.argtypes = [hc, vp]
    lib.ttemb_ht_update_push.argtypes = [hc, vp, vp, vp, i64, f32, i32, vp]
    lib.ttemb_ht_cache_stats.argtypes = [hc, C.POINTER(i32), C.POINTER(i32), vp]
    lib.ttemb_ht_host_gather.argtypes = [vp, i64, i32, vp, i64, vp, i32]
    lib.ttemb_ht_host_sgd.argtypes = [vp, i64, i32, vp, i64, vp, f32, i32]
    for s in SYMBOLS:
        f = getattr(lib, s)
        if s not in ("ttemb_stage_name", "ttemb_status_string", "ttemb_total_rows"):
            f.restype = C.c_int
    lib.ttemb_total_rows.restype = C.c_uint64
    _lib = lib
    return lib


def status_string(code: int) -> str:
    return load().ttemb_status_string(int(code)).decode()


def check(rc: int, what: str = "") -> None:
    if rc != TTEMB_OK:
        raise TTEmbError(rc, what)
