"""ctypes binding of libgcsm.so (include/gcsm.h). Argument marshalling only.

No fallback: if the CUDA library is missing this raises; nothing on the path
runs in Python.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
# GCSM_LIB selects a tuning variant built by build.build(out=..., defines=...) (development only)
LIB_PATH = os.environ.get("GCSM_LIB") or os.path.join(HERE, "libgcsm.so")

STATUS = {0: "GCSM_OK", 1: "GCSM_EINVAL", 2: "GCSM_ENOMEM", 3: "GCSM_EDEVICE", 4: "GCSM_ENCCL", 5: "GCSM_ESTATE",
          6: "GCSM_ETRUNC"}

# exported symbols of include/gcsm.h (checked by tests/test_abi.py)
SYMBOLS = ["gcsm_default_options", "gcsm_create", "gcsm_set_query", "gcsm_set_cache_budget", "gcsm_apply_batch",
           "gcsm_apply_batch_list", "gcsm_submit_batch", "gcsm_wait_batch", "gcsm_get_stats", "gcsm_add_query", "gcsm_num_queries",
           "gcsm_get_query_stats", "gcsm_query_automorphisms", "gcsm_last_error", "gcsm_destroy",
           "gcsm_nccl_unique_id", "gcsm_get_stream", "gcsm_export_csr", "gcsm_get_estimates", "gcsm_get_cached",
           "gcsm_plan_inspect", "gcsm_query_restrictions", "gcsm_shard",
           "gcsm_measure_host_link", "gcsm_binomial_samples", "gcsm_set_measure",
           "gcsm_num_vertices", "gcsm_add_vertices", "gcsm_link_peers", "gcsm_store_handle",
           "gcsm_link_store_peers"]


class Options(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("nccl_id", ctypes.c_void_p), ("seed", ctypes.c_uint64), ("host_threads", ctypes.c_int32),
                ("cache_policy", ctypes.c_int32), ("walks_override", ctypes.c_uint64), ("flags", ctypes.c_uint32),
                ("reserved", ctypes.c_uint32), ("vertex_capacity", ctypes.c_int64), ("staging_bytes", ctypes.c_uint64),
                ("store_rank", ctypes.c_int32), ("store_world", ctypes.c_int32), ("store_handle", ctypes.c_char_p)]


class Stats(ctypes.Structure):
    _fields_ = [(name, ctypes.c_uint64) for name in
                ["batches", "n_ins", "n_del", "dropped", "units", "n1", "walks", "max_degree", "cached_vertices",
                 "cache_bytes", "hit_bytes", "miss_bytes", "delta_bytes", "hit_bytes_ext", "miss_bytes_ext",
                 "delta_bytes_ext", "host_copied_bytes", "frontier", "kernel_launches", "h2d_bytes", "d2h_bytes", "added", "removed"]] + \
              [(name, ctypes.c_double) for name in
               ["ms_normalize", "ms_estimate", "ms_pack", "ms_copy", "ms_match", "ms_level2", "ms_extend",
                "ms_allreduce", "ms_merge", "ms_total"]] + \
              [(name, ctypes.c_uint64) for name in
               ["stage_fill_bytes", "stage_lists", "stage_hit_bytes", "bcomp_hit_bytes", "bcomp_miss_bytes",
                "bcomp_delta_bytes", "peer_bytes", "walk_fill_bytes", "walk_stage_lists", "walk_alg_bytes"]] + \
              [("ms_walks", ctypes.c_double)]


_lib = None


def load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is not built: run `python -c 'import __graft_entry__ as g; g.build()'` "
                           "(hand-written CUDA for sm_100a; there is no fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    P, I32, I64, U64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
    st = ctypes.c_int
    sig = {
        "gcsm_default_options": (None, [ctypes.POINTER(Options)]),
        "gcsm_create": (st, [I32, P, P, P, ctypes.POINTER(Options), ctypes.POINTER(P)]),
        "gcsm_set_query": (st, [P, I32, I32, P, P, P]),
        "gcsm_set_cache_budget": (st, [P, U64]),
        "gcsm_apply_batch": (st, [P, I64, P, I64, P, ctypes.POINTER(U64), ctypes.POINTER(U64)]),
        "gcsm_apply_batch_list": (st, [P, I64, P, I64, P, P, U64, P, U64, ctypes.POINTER(U64), ctypes.POINTER(U64)]),
        "gcsm_submit_batch": (st, [P, I64, P, I64, P]),
        "gcsm_wait_batch": (st, [P, ctypes.POINTER(U64), ctypes.POINTER(U64)]),
        "gcsm_get_stats": (st, [P, ctypes.POINTER(Stats)]),
        "gcsm_add_query": (st, [P, I32, I32, P, P, P, ctypes.POINTER(I32)]),
        "gcsm_num_queries": (I32, [P]),
        "gcsm_get_query_stats": (st, [P, I32, ctypes.POINTER(Stats)]),
        "gcsm_query_automorphisms": (U64, [P]),
        "gcsm_last_error": (ctypes.c_char_p, [P]),
        "gcsm_destroy": (None, [P]),
        "gcsm_nccl_unique_id": (st, [P]),
        "gcsm_get_stream": (st, [P, ctypes.POINTER(P)]),
        "gcsm_export_csr": (st, [P, P, P, U64]),
        "gcsm_get_estimates": (st, [P, P, P, U64, ctypes.POINTER(U64)]),
        "gcsm_get_cached": (st, [P, P, U64, ctypes.POINTER(U64)]),
        "gcsm_plan_inspect": (st, [I32, I32, P, P, P, P, P, P, P]),
        "gcsm_shard": (st, [I64, P, I32, P]),
        "gcsm_binomial_samples": (st, [U64, I64, ctypes.c_double, I64, P]),
        "gcsm_set_measure": (st, [P, ctypes.c_uint32]),
        "gcsm_num_vertices": (I32, [P]),
        "gcsm_store_handle": (st, [P, P, U64]),
        "gcsm_link_store_peers": (st, [P]),
        "gcsm_link_peers": (st, [P, I32]),
        "gcsm_add_vertices": (st, [P, I32, P, ctypes.POINTER(I32)]),
        "gcsm_query_restrictions": (st, [I32, I32, P, P, P, P, I32, P, ctypes.POINTER(U64)]),
        "gcsm_measure_host_link": (st, [I32, U64, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double),
                                        ctypes.POINTER(ctypes.c_double)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib
