"""ctypes declarations of libsigmo.so (include/sigmo.h) -- argument
marshalling only.  Every function of the C ABI is exposed under its own name.
Loading fails loudly when the library is missing: there is no CPU fallback."""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libsigmo.so")

SIGMO_OK = 0
STATUS_NAMES = {0: "SIGMO_OK", -1: "SIGMO_ERR_INVALID_ARG", -2: "SIGMO_ERR_INVALID_GRAPH", -3: "SIGMO_ERR_LIMIT",
                -4: "SIGMO_ERR_STATE", -5: "SIGMO_ERR_OOM", -6: "SIGMO_ERR_CUDA"}
SIGMO_FIND_ALL = 0
SIGMO_FIND_FIRST = 1
SIGMO_ENUM_NODE_SETS = 1
SIGMO_FILTER_NEIGHBOR_SUPPORT = 1

# every symbol declared in include/sigmo.h
EXPORTS = ["sigmo_create", "sigmo_load_batch", "sigmo_filter", "sigmo_join", "sigmo_num_pairs",
           "sigmo_get_pair_results", "sigmo_get_dense_results", "sigmo_get_query_totals", "sigmo_get_candidates",
           "sigmo_get_signatures", "sigmo_get_packed_batch", "sigmo_check_join", "sigmo_enumerate",
           "sigmo_get_embeddings", "sigmo_get_node_sets", "sigmo_set_wildcards", "sigmo_set_induced", "sigmo_set_timing",
           "sigmo_get_timings", "sigmo_validate_batch",
           "sigmo_last_error", "sigmo_version", "sigmo_destroy"]


class sigmo_graph_batch(ctypes.Structure):
    _fields_ = [("num_graphs", ctypes.c_int64), ("num_nodes", ctypes.c_int64),
                ("graph_offsets", ctypes.POINTER(ctypes.c_int64)),
                ("row_offsets", ctypes.POINTER(ctypes.c_int64)),
                ("col_indices", ctypes.POINTER(ctypes.c_int32)),
                ("node_labels", ctypes.POINTER(ctypes.c_uint8)),
                ("edge_labels", ctypes.POINTER(ctypes.c_uint8))]


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)


class sigmo_allocator(ctypes.Structure):
    _fields_ = [("alloc", ALLOC_FN), ("free", FREE_FN), ("user", ctypes.c_void_p)]


class sigmo_timings(ctypes.Structure):
    _fields_ = [("query_prep_ms", ctypes.c_float), ("filter_ms", ctypes.c_float), ("support_ms", ctypes.c_float),
                ("mapping_ms", ctypes.c_float), ("join_ms", ctypes.c_float),
                ("filter_launches", ctypes.c_int64), ("join_launches", ctypes.c_int64),
                ("h2d_bytes", ctypes.c_int64), ("filter_calls", ctypes.c_int64),
                ("join_calls", ctypes.c_int64), ("dfs_steps", ctypes.c_int64),
                ("dfs_iters", ctypes.c_int64), ("dfs_tail_iters", ctypes.c_int64), ("dfs_max_stack", ctypes.c_int64),
                ("filter_jit", ctypes.c_int64), ("jit_compile_ms", ctypes.c_double)]


_lib = None


def load_library(path: str | None = None) -> ctypes.CDLL:
    """Load libsigmo.so.  Raises if it has not been built (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    path = path or os.environ.get("SIGMO_LIB") or LIB_PATH  # SIGMO_LIB: alternative in-tree build (experiments)
    if not os.path.exists(path):
        raise RuntimeError(f"libsigmo.so not found at {path}: build it with "
                           f"`python -c 'import __graft_entry__ as g; g.build()'` (there is no CPU fallback)")
    lib = ctypes.CDLL(path)
    P = ctypes.POINTER
    vp = ctypes.c_void_p
    st = ctypes.c_int
    lib.sigmo_create.argtypes = [ctypes.c_int, vp, P(sigmo_allocator), P(vp)]
    lib.sigmo_load_batch.argtypes = [vp, P(sigmo_graph_batch), P(sigmo_graph_batch)]
    lib.sigmo_filter.argtypes = [vp, ctypes.c_int, ctypes.c_uint32]
    lib.sigmo_join.argtypes = [vp, ctypes.c_int, P(ctypes.c_uint64)]
    lib.sigmo_num_pairs.argtypes = [vp, P(ctypes.c_int64)]
    lib.sigmo_get_pair_results.argtypes = [vp, ctypes.c_int64, P(ctypes.c_int64), P(ctypes.c_int64),
                                           P(ctypes.c_int32), P(ctypes.c_uint64)]
    lib.sigmo_get_dense_results.argtypes = [vp, P(ctypes.c_uint64)]
    lib.sigmo_get_query_totals.argtypes = [vp, vp, ctypes.c_int]
    lib.sigmo_get_candidates.argtypes = [vp, P(ctypes.c_uint32)]
    lib.sigmo_get_signatures.argtypes = [vp, ctypes.c_int, ctypes.c_int, P(ctypes.c_uint64)]
    lib.sigmo_get_packed_batch.argtypes = [vp, ctypes.c_int, P(ctypes.c_int64), P(ctypes.c_int64), P(ctypes.c_int64),
                                           P(ctypes.c_int64), P(ctypes.c_int64), P(ctypes.c_int32),
                                           P(ctypes.c_uint8), P(ctypes.c_uint8)]
    lib.sigmo_check_join.argtypes = [vp]
    i64p, i32p = P(ctypes.c_int64), P(ctypes.c_int32)
    lib.sigmo_enumerate.argtypes = [vp, ctypes.c_uint32, i64p]
    lib.sigmo_get_embeddings.argtypes = [vp, ctypes.c_int64, i64p, i64p, i32p, i64p, ctypes.c_int64,
                                         P(ctypes.c_uint8), i64p, i32p]
    lib.sigmo_get_node_sets.argtypes = [vp, ctypes.c_int64, i64p, i64p, ctypes.c_int64, P(ctypes.c_uint64), i64p]
    lib.sigmo_set_timing.argtypes = [vp, ctypes.c_int]
    lib.sigmo_set_induced.argtypes = [vp, ctypes.c_int]
    lib.sigmo_set_wildcards.argtypes = [vp, ctypes.c_int]
    lib.sigmo_get_timings.argtypes = [vp, P(sigmo_timings)]
    lib.sigmo_validate_batch.argtypes = [P(sigmo_graph_batch), ctypes.c_int, ctypes.c_char_p, ctypes.c_size_t]
    lib.sigmo_last_error.argtypes = [vp]
    lib.sigmo_last_error.restype = ctypes.c_char_p
    lib.sigmo_version.argtypes = []
    lib.sigmo_version.restype = ctypes.c_char_p
    lib.sigmo_destroy.argtypes = [vp]
    for name in EXPORTS:
        f = getattr(lib, name)
        if name not in ("sigmo_last_error", "sigmo_version"):
            f.restype = st
    _lib = lib
    return lib
