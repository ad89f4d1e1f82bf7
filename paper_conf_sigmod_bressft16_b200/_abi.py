"""ctypes mirror of include/ddq.h (argument marshalling only).

Every computation runs inside libddq.so (hand-written sm_100a kernels + the C++
driver).  There is no Python or CPU fallback: if the library cannot be loaded, or
no CUDA device is present, the calls raise.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "libddq.so")

DDQ_OK = 0
STATUS = {0: "DDQ_OK", -1: "DDQ_EINVAL", -2: "DDQ_ENOTFOUND", -3: "DDQ_ENOMEM_HOST",
          -4: "DDQ_ENOMEM_DEVICE", -5: "DDQ_ECUDA", -6: "DDQ_ENCCL", -7: "DDQ_ESTATE",
          -8: "DDQ_ETIMEOUT", -9: "DDQ_EOVERFLOW"}

PRED_RANGE, PRED_IN, PRED_BITSET = 1, 2, 3
MAX_IN, MAX_PREDS, MAX_CARRY, MAX_AGGS, MAX_KEYS, MAX_OPS = 8, 4, 4, 8, 3, 32
CMP_EQ, CMP_LT, CMP_NE = 0, 1, 2  # FILTER_EQ comparison (ddq_op.eq_cmp)
OP_SELECT, OP_HASH_BUILD, OP_HASH_PROBE, OP_GATHER, OP_AGGREGATE, OP_FILTER_EQ, OP_STAR = 1, 2, 3, 4, 5, 6, 7
TERM_PRED, TERM_PROBE, TERM_FETCH = 1, 2, 3
AGG_COUNT, AGG_SUM, AGG_SUM_MUL, AGG_SUM_SUB, AGG_SUM_MUL_100M, AGG_SUM_MUL_100M_100P = 1, 2, 3, 4, 5, 6
AGG_MIN = 7  # min(a): S8(a6); generic global-table kernel
I32, I64 = 1, 2
PLACE_DATA_DRIVEN, PLACE_GPU_ONLY, PLACE_CPU_ONLY = 0, 1, 2
RAN_GPU, RAN_HOST, RAN_ABORTED = 1, 2, 3  # ddq_result.op_place


class DevPred(ctypes.Structure):
    _fields_ = [("col", ctypes.c_void_p), ("width", ctypes.c_int32), ("kind", ctypes.c_int32),
                ("lo", ctypes.c_int64), ("hi", ctypes.c_int64), ("n_in", ctypes.c_int32),
                ("_pad", ctypes.c_int32), ("in_vals", ctypes.c_int64 * MAX_IN)]


class DevAgg(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("width", ctypes.c_int32 * 3), ("arg", ctypes.c_void_p * 3)]


class Config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("cache_bytes", ctypes.c_uint64), ("heap_bytes", ctypes.c_uint64),
                ("gpu_workers", ctypes.c_int32), ("host_workers", ctypes.c_int32),
                ("placement", ctypes.c_int32), ("chopping", ctypes.c_int32),
                ("cache_policy", ctypes.c_int32), ("fault_alloc_every", ctypes.c_uint32),
                ("transfer_packing", ctypes.c_int32), ("prefetch", ctypes.c_int32),
                ("placement_period_ms", ctypes.c_int32), ("max_queries", ctypes.c_int32),
                ("fault_op_mask", ctypes.c_uint32)]


class Pred(ctypes.Structure):
    _fields_ = [("column", ctypes.c_int32), ("kind", ctypes.c_int32), ("lo", ctypes.c_int64),
                ("hi", ctypes.c_int64), ("n_in", ctypes.c_int32), ("_pad", ctypes.c_int32),
                ("in_vals", ctypes.c_int64 * MAX_IN)]


class Op(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("input", ctypes.c_int32), ("table", ctypes.c_int32),
                ("n_preds", ctypes.c_int32), ("preds", Pred * MAX_PREDS),
                ("key_col", ctypes.c_int32), ("payload_col", ctypes.c_int32),
                ("build", ctypes.c_int32), ("fk_col", ctypes.c_int32), ("emit_payload", ctypes.c_int32),
                ("gather_col", ctypes.c_int32),
                ("n_keys", ctypes.c_int32), ("key_src", ctypes.c_int32 * MAX_KEYS),
                ("n_aggs", ctypes.c_int32), ("agg_kind", ctypes.c_int32 * MAX_AGGS),
                ("agg_col", (ctypes.c_int32 * 3) * MAX_AGGS),
                ("max_groups", ctypes.c_int64), ("n_order", ctypes.c_int32),
                ("order_by", ctypes.c_int32 * 8), ("limit", ctypes.c_int64),
                ("key_bits", ctypes.c_int32 * MAX_KEYS), ("fk_vec", ctypes.c_int32),
                ("eq_vec", ctypes.c_int32 * 2), ("n_terms", ctypes.c_int32),
                ("term_kind", ctypes.c_int32 * 4), ("term_build", ctypes.c_int32 * 4),
                ("term_fk", ctypes.c_int32 * 4), ("term_emit", ctypes.c_int32 * 4),
                ("fetch_build", ctypes.c_int32), ("eq_cmp", ctypes.c_int32),
                ("build_key_set", ctypes.c_int32), ("n_avg", ctypes.c_int32),
                ("avg_sum", ctypes.c_int32 * 4), ("avg_count", ctypes.c_int32),
                ("avg_scale", ctypes.c_int32 * 4), ("gather_narrow", ctypes.c_int32)]


class DevTerm(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("width", ctypes.c_int32), ("col", ctypes.c_void_p),
                ("pred_kind", ctypes.c_int32), ("n_in", ctypes.c_int32), ("lo", ctypes.c_int64),
                ("hi", ctypes.c_int64), ("in_vals", ctypes.c_int64 * MAX_IN), ("index", ctypes.c_void_p),
                ("key_min", ctypes.c_int32), ("range", ctypes.c_uint32), ("table", ctypes.c_void_p),
                ("capacity", ctypes.c_uint32), ("_pad", ctypes.c_int32), ("out_payload", ctypes.c_void_p)]


class Plan(ctypes.Structure):
    _fields_ = [("n_ops", ctypes.c_int32), ("ops", Op * MAX_OPS)]


class Result(ctypes.Structure):
    _fields_ = [("n_rows", ctypes.c_int64), ("n_keys", ctypes.c_int32), ("n_aggs", ctypes.c_int32),
                ("keys", ctypes.POINTER(ctypes.c_int64)), ("aggs", ctypes.POINTER(ctypes.c_int64)),
                ("n_tids", ctypes.c_int64), ("tids", ctypes.POINTER(ctypes.c_int32)),
                ("gpu_ops", ctypes.c_int32), ("host_ops", ctypes.c_int32), ("aborts", ctypes.c_int32),
                ("exec_ms", ctypes.c_double), ("agg_null", ctypes.POINTER(ctypes.c_uint8)),
                ("n_avg", ctypes.c_int32), ("_pad", ctypes.c_int32), ("avgs", ctypes.POINTER(ctypes.c_double)),
                ("key_str", ctypes.POINTER(ctypes.c_char_p)), ("n_ops", ctypes.c_int32), ("_pad2", ctypes.c_int32),
                ("op_place", ctypes.POINTER(ctypes.c_uint8)), ("op_ms", ctypes.POINTER(ctypes.c_float))]


class Stats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in
                ("h2d_bytes", "d2h_bytes", "h2d_ns", "d2h_ns", "gpu_ops", "host_ops", "aborts",
                 "wasted_ns", "heap_peak_bytes", "heap_used_bytes", "cache_used_bytes", "cache_hits",
                 "cache_misses", "queries_done")]


# host all-gather callback of ddq_dist_init_host: (send, recv, bytes, user) -> 0 on success
ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)

# name -> (restype, argtypes)
_vp, _i32, _i64, _u32, _u64, _sz = (ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32,
                                    ctypes.c_uint64, ctypes.c_size_t)
_pp = ctypes.POINTER(ctypes.c_void_p)
SIGNATURES = {
    "ddq_last_error": (ctypes.c_char_p, []),
    "ddq_version": (ctypes.c_char_p, []),
    "ddq_op_scratch_bytes": (_sz, [_i64]),
    "ddq_op_select": (_i32, [ctypes.POINTER(DevPred), _i32, _vp, _vp, _i64, _pp, _pp, _i32, _vp, _vp, _vp, _sz, _vp]),
    "ddq_op_hash_init": (_i32, [_vp, _u32, _vp]),
    "ddq_op_hash_build": (_i32, [_vp, _vp, _vp, _vp, _i64, _vp, _u32, _vp, _vp]),
    "ddq_op_hash_probe": (_i32, [_vp, _u32, _vp, _vp, _vp, _i64, _pp, _pp, _i32, _vp, _vp, _vp, _vp, _sz, _vp]),
    "ddq_op_star": (_i32, [ctypes.POINTER(DevTerm), _i32, _i64, _vp, _vp, _i64, _vp, _vp]),
    "ddq_op_join_index_bytes": (_sz, [_u32]),
    "ddq_op_join_index_init": (_i32, [_vp, _u32, _vp]),
    "ddq_op_join_index_build": (_i32, [_vp, _vp, _vp, _vp, _i64, _i32, _u32, _vp, _vp, _vp]),
    "ddq_op_join_index_probe": (_i32, [_vp, _i32, _u32, _vp, _vp, _vp, _i64, _pp, _pp, _i32, _vp, _vp, _vp, _vp,
                                       _sz, _vp]),
    "ddq_op_gather": (_i32, [_vp, _i32, _vp, _vp, _i64, _vp, _vp]),
    "ddq_op_groupby_table_bytes": (_sz, [_u32, _i32]),
    "ddq_op_groupby_init": (_i32, [_vp, _u32, _i32, _vp]),
    "ddq_op_groupby": (_i32, [_vp, _vp, _i64, _pp, _pp, _i32, _vp, ctypes.POINTER(DevAgg), _i32, _vp, _u32, _vp,
                              _vp]),
    "ddq_op_groupby_compact": (_i32, [_vp, _u32, _i32, _vp, _vp, _vp, _vp]),
    "ddq_config_default": (None, [ctypes.POINTER(Config)]),
    "ddq_open": (_i32, [ctypes.POINTER(Config), ctypes.POINTER(_vp)]),
    "ddq_close": (None, [_vp]),
    "ddq_create_table": (_i32, [_vp, ctypes.c_char_p, _i64, _i64, ctypes.POINTER(_i32)]),
    "ddq_load_column": (_i32, [_vp, _i32, ctypes.c_char_p, _i32, _vp, _i64, ctypes.POINTER(_i32)]),
    "ddq_find_column": (_i32, [_vp, ctypes.c_char_p, ctypes.c_char_p, ctypes.POINTER(_i32)]),
    "ddq_column_stats": (_i32, [_vp, _i32, ctypes.POINTER(_i64), ctypes.POINTER(_i64), ctypes.POINTER(_i64)]),
    "ddq_set_dictionary": (_i32, [_vp, _i32, ctypes.POINTER(ctypes.c_char_p), _i32]),
    "ddq_dictionary_range": (_i32, [_vp, _i32, ctypes.c_char_p, ctypes.POINTER(_i32), ctypes.POINTER(_i32)]),
    "ddq_dictionary_like": (_i32, [_vp, _i32, ctypes.c_char_p, ctypes.POINTER(Pred)]),
    "ddq_cache_column": (_i32, [_vp, _i32]),
    "ddq_evict_column": (_i32, [_vp, _i32]),
    "ddq_column_is_cached": (_i32, [_vp, _i32]),
    "ddq_column_device_ptr": (_vp, [_vp, _i32]),
    "ddq_update_placement": (_i32, [_vp]),
    "ddq_column_access_count": (_u64, [_vp, _i32]),
    "ddq_reset_access_counts": (_i32, [_vp]),
    "ddq_submit": (_i32, [_vp, ctypes.POINTER(Plan), ctypes.POINTER(_i64)]),
    "ddq_wait": (_i32, [_vp, _i64, _i64]),
    "ddq_fetch": (_i32, [_vp, _i64, ctypes.POINTER(ctypes.POINTER(Result))]),
    "ddq_result_free": (None, [ctypes.POINTER(Result)]),
    "ddq_prepare": (_i32, [_vp, ctypes.POINTER(Plan), _i32, ctypes.POINTER(_vp)]),
    "ddq_prepared_launch": (_i32, [_vp, _vp]),
    "ddq_prepared_fetch": (_i32, [_vp, _vp, ctypes.POINTER(ctypes.POINTER(Result))]),
    "ddq_prepared_partials": (_i32, [_vp, _vp, ctypes.POINTER(_i64), _vp, _vp, _i64]),
    "ddq_prepared_group_capacity": (_i64, [_vp]),
    "ddq_prepared_kernel_count": (_i32, [_vp]),
    "ddq_prepared_profile": (_i32, [_vp, _vp, _i32, ctypes.POINTER(ctypes.c_float), ctypes.POINTER(ctypes.c_double),
                                    ctypes.POINTER(_i32)]),
    "ddq_prepared_partials_device": (_i32, [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_vp), ctypes.POINTER(_vp),
                                            ctypes.POINTER(_i64)]),
    "ddq_finalize_partials": (_i32, [ctypes.POINTER(Op), _i64, _vp, _vp, ctypes.POINTER(ctypes.POINTER(Result))]),
    "ddq_prepared_finalize": (_i32, [_vp, _i64, _vp, _vp, ctypes.POINTER(ctypes.POINTER(Result))]),
    "ddq_prepared_free": (None, [_vp]),
    "ddq_dist_nccl_unique_id": (_i32, [_vp]),
    "ddq_dist_init_nccl": (_i32, [_vp, _vp, _i32, _i32, _i32]),
    "ddq_dist_init_host": (_i32, [_vp, _i32, _i32, _vp, _vp]),
    "ddq_table_set_partitioned": (_i32, [_vp, _i32, _i32]),
    "ddq_dist_exchange": (_i32, [_vp, ctypes.POINTER(_vp), _i32, _vp]),
    "ddq_dist_result": (_i32, [_vp, _i32, ctypes.POINTER(ctypes.POINTER(Result))]),
    "ddq_cluster_open": (_i32, [ctypes.POINTER(Config), ctypes.POINTER(_i32), _i32, ctypes.POINTER(_vp)]),
    "ddq_cluster_close": (None, [_vp]),
    "ddq_cluster_size": (_i32, [_vp]),
    "ddq_cluster_db": (_vp, [_vp, _i32]),
    "ddq_cluster_submit": (_i32, [_vp, ctypes.POINTER(Plan), ctypes.POINTER(_i32), ctypes.POINTER(_i64)]),
    "ddq_cluster_fetch": (_i32, [_vp, _i32, _i64, ctypes.POINTER(ctypes.POINTER(Result))]),
    "ddq_cluster_update_placement": (_i32, [_vp]),
    "ddq_get_stats": (_i32, [_vp, ctypes.POINTER(Stats)]),
    "ddq_reset_stats": (_i32, [_vp]),
    "ddq_heap_try_alloc": (_vp, [_vp, _u64]),
    "ddq_heap_free": (None, [_vp, _vp]),
}

_lib = None


class DDQError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def lib():
    """Load libddq.so (building it in-tree if the sources are newer)."""
    global _lib
    if _lib is None:
        if not os.path.exists(SO) or os.environ.get("DDQ_REBUILD"):
            from . import build_native
            build_native.build()
        L = ctypes.CDLL(SO)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(status: int) -> None:
    if status != DDQ_OK:
        raise DDQError(status, lib().ddq_last_error().decode(errors="replace"))
