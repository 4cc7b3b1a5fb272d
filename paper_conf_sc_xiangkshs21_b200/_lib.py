"""ctypes binding of libcuts.so (include/cuts.h) — argument marshalling only.

Every step of the hot path runs in the CUDA kernels of libcuts.so; this module
only declares the C signatures.  There is no fallback: if the shared library is
missing or fails to load, importing the package raises.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("CUTS_LIB") or os.path.join(_HERE, "libcuts.so")   # CUTS_LIB: A/B builds

CUTS_OK, CUTS_EINVAL, CUTS_ENOMEM, CUTS_ECUDA = 0, -1, -2, -3
CUTS_EOVERFLOW, CUTS_ETRUNC, CUTS_ESTATE, CUTS_EUNSUPPORTED, CUTS_ECOMM = -4, -5, -6, -7, -8
STATUS_NAMES = {0: "CUTS_OK", -1: "CUTS_EINVAL", -2: "CUTS_ENOMEM", -3: "CUTS_ECUDA", -4: "CUTS_EOVERFLOW",
                -5: "CUTS_ETRUNC", -6: "CUTS_ESTATE", -7: "CUTS_EUNSUPPORTED", -8: "CUTS_ECOMM"}
CUTS_BFS, CUTS_HYBRID = 0, 1
CUTS_DEBUG_TIMING, CUTS_DEBUG_BYTES = 1, 2
MAX_K = 8
GROUP_HIST_WORDS = 432
DIST_UID_BYTES = 128

# the symbols include/cuts.h declares (tests check the library exports all of them)
EXPORTED = ["cuts_version", "cuts_create", "cuts_destroy", "cuts_last_error", "cuts_load_graph",
            "cuts_load_digraph", "cuts_set_query_directed",
            "cuts_set_query", "cuts_set_root_range", "cuts_set_root_slice", "cuts_level1_size", "cuts_count",
            "cuts_enumerate", "cuts_get_stats", "cuts_set_debug", "cuts_trie_decode", "cuts_set_hub_threshold",
            "cuts_set_prefixes", "cuts_set_donation", "cuts_dist_unique_id", "cuts_set_dist",
            "cuts_allreduce_count", "cuts_debug_group_hist", "cuts_set_partition_depth", "cuts_partition_size"]

# callback types of cuts_set_donation
POLL_FN = ctypes.CFUNCTYPE(ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64)
SHIP_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint64)


class cuts_opts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("stream", ctypes.c_size_t), ("arena", ctypes.c_void_p),
                ("arena_bytes", ctypes.c_uint64), ("seed", ctypes.c_uint64)]


class cuts_stats(ctypes.Structure):
    _fields_ = [("k", ctypes.c_uint32), ("order", ctypes.c_uint32 * MAX_K),
                ("level_size", ctypes.c_uint64 * (MAX_K + 1)),
                ("count_lo", ctypes.c_uint64), ("count_hi", ctypes.c_uint64),
                ("level1_canonical", ctypes.c_uint64), ("chunks", ctypes.c_uint64),
                ("windows", ctypes.c_uint64), ("launches", ctypes.c_uint64),
                ("peak_arena_bytes", ctypes.c_uint64), ("items", ctypes.c_uint64),
                ("ms_total", ctypes.c_double), ("ms_extend", ctypes.c_double), ("ms_plan", ctypes.c_double),
                ("extend_launches", ctypes.c_uint64), ("alg_bytes_extend", ctypes.c_uint64),
                ("alg_bytes_plan", ctypes.c_uint64), ("hubs", ctypes.c_uint64),
                ("hub_threshold", ctypes.c_uint64), ("donations", ctypes.c_uint64),
                ("donated_entries", ctypes.c_uint64), ("alg_bytes_extend_needed", ctypes.c_uint64),
                ("free_identity", ctypes.c_uint64), ("fused_levels", ctypes.c_uint64),
                ("ms_tail", ctypes.c_double), ("tail_launches", ctypes.c_uint64),
                ("tail_word_ops", ctypes.c_uint64)]


_lib = None


def load() -> ctypes.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'`"
                          " (there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    P, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    u32p, u64p = ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint64)
    sig = {
        "cuts_version": ([], i32),
        "cuts_create": ([ctypes.POINTER(P), ctypes.POINTER(cuts_opts)], i32),
        "cuts_destroy": ([P], None),
        "cuts_last_error": ([P], ctypes.c_char_p),
        "cuts_load_graph": ([P, u32, u64, P, P, i32], i32),
        "cuts_set_query": ([P, u32, u32p, u32p, u32p], i32),
        "cuts_load_digraph": ([P, u32, u64, P, P, i32], i32),
        "cuts_set_query_directed": ([P, u32, u32p, u32p, u32p], i32),
        "cuts_set_root_range": ([P, u64, u64], i32),
        "cuts_set_root_slice": ([P, u64, u64, u32, u32], i32),
        "cuts_level1_size": ([P, u64p, u64p], i32),
        "cuts_count": ([P, i32, u64p], i32),
        "cuts_enumerate": ([P, i32, P, u64, u64p], i32),
        "cuts_get_stats": ([P, ctypes.POINTER(cuts_stats)], i32),
        "cuts_set_debug": ([P, u32], i32),
        "cuts_set_hub_threshold": ([P, u32], i32),
        "cuts_trie_decode": ([P, u32, u64p, ctypes.POINTER(P), ctypes.POINTER(P), P], i32),
        "cuts_set_prefixes": ([P, u32, u64, P], i32),
        "cuts_set_donation": ([P, POLL_FN, SHIP_FN, P], i32),
        "cuts_dist_unique_id": ([P], i32),
        "cuts_set_dist": ([P, i32, i32, P, P], i32),
        "cuts_allreduce_count": ([P, u64, u64, u64p, u64p], i32),
        "cuts_debug_group_hist": ([P, u64p], i32),
        "cuts_set_partition_depth": ([P, u32], i32),
        "cuts_partition_size": ([P, u64p], i32),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    _lib = lib
    return lib
