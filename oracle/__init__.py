"""SIGMo CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  It
shares no code with the CUDA path (``paper_conf_sc_carocfc25_b200``) and the
CUDA path never imports it.  Inputs come from the shared seeded generator
module ``synth`` (inputs only, no method arithmetic).

Contents (each function cites the passage it follows):
  * ``count_dense`` / ``count_pairs``  -- the join result by plain
    backtracking, in C (``sigmo_oracle.c``), no signature filter
    (Def. 2.1, NLSM P:446-453; Find All / Find First
    P:193-196).
  * ``brute``     -- brute-force enumeration of injective maps (pin P4).
  * ``filter_ref`` -- signatures, candidate bitmap, GMCR and the optional
    neighbour-support fixed point (Alg. 1, section 4.2 P:846-885,
    section 4.5), readings R4-R11 of DESIGN.md.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

FIND_ALL = 0
FIND_FIRST = 1
INDUCED = 2  # mode bit: induced-subgraph embeddings (R21)
WILDCARD = 4  # mode bit: query atom label 0 = any atom, bond label 0 = any bond (R22)


class _Batch(ctypes.Structure):
    _fields_ = [("num_graphs", ctypes.c_int64),
                ("graph_offsets", ctypes.POINTER(ctypes.c_int64)),
                ("row_offsets", ctypes.POINTER(ctypes.c_int64)),
                ("col_indices", ctypes.POINTER(ctypes.c_int32)),
                ("node_labels", ctypes.POINTER(ctypes.c_uint8)),
                ("edge_labels", ctypes.POINTER(ctypes.c_uint8))]


def build_lib(force: bool = False) -> str:
    src = os.path.join(_HERE, "sigmo_oracle.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-pthread", src, "-o", _LIB_PATH])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build_lib()
        lib = ctypes.CDLL(_LIB_PATH)
        bp = ctypes.POINTER(_Batch)
        u64p = ctypes.POINTER(ctypes.c_uint64)
        i64p = ctypes.POINTER(ctypes.c_int64)
        ip = ctypes.POINTER(ctypes.c_int)
        lib.oracle_count_dense.argtypes = [bp, bp, ctypes.c_int, ctypes.c_int, u64p, u64p, ip]
        lib.oracle_count_pairs.argtypes = [bp, bp, ctypes.c_int, ctypes.c_int, ctypes.c_int64, i64p, i64p, u64p,
                                           u64p, ip]
        lib.oracle_enumerate_pair.argtypes = [bp, bp, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
                                              ctypes.POINTER(ctypes.c_int32), ctypes.c_int64, i64p]
        _lib = lib
    return _lib


def _as_struct(B):
    s = _Batch()
    s.num_graphs = B.num_graphs
    s.graph_offsets = B.graph_offsets.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
    s.row_offsets = B.row_offsets.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
    s.col_indices = B.col_indices.ctypes.data_as(ctypes.POINTER(ctypes.c_int32))
    s.node_labels = B.node_labels.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))
    s.edge_labels = B.edge_labels.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))
    return s


def default_threads() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


class OracleResult:
    def __init__(self, values, work, overflow):
        self.values = values
        self.work = work
        self.overflow = overflow


def count_dense(Q, D, mode: int = FIND_ALL, nthreads: int | None = None, with_work: bool = False):
    """Dense [NQ, ND] uint64 results: Find All counts or Find First 0/1 flags."""
    lib = _load()
    nthreads = nthreads or default_threads()
    out = np.zeros((Q.num_graphs, D.num_graphs), np.uint64)
    work = ctypes.c_uint64(0)
    ovf = ctypes.c_int(0)
    qs, ds = _as_struct(Q), _as_struct(D)
    rc = lib.oracle_count_dense(ctypes.byref(qs), ctypes.byref(ds), mode, nthreads,
                                out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), ctypes.byref(work),
                                ctypes.byref(ovf))
    if rc != 0:
        raise RuntimeError(f"oracle_count_dense failed rc={rc}")
    if ovf.value:
        raise OverflowError("oracle count exceeded 2^64-1")
    return OracleResult(out, work.value, ovf.value) if with_work else out


def count_pairs(Q, D, pq, pg, mode: int = FIND_ALL, nthreads: int | None = None, with_work: bool = False):
    """Results for an explicit pair list (query pq[i], data graph pg[i])."""
    lib = _load()
    nthreads = nthreads or default_threads()
    pq = np.ascontiguousarray(pq, dtype=np.int64)
    pg = np.ascontiguousarray(pg, dtype=np.int64)
    out = np.zeros(pq.shape[0], np.uint64)
    work = ctypes.c_uint64(0)
    ovf = ctypes.c_int(0)
    qs, ds = _as_struct(Q), _as_struct(D)
    rc = lib.oracle_count_pairs(ctypes.byref(qs), ctypes.byref(ds), mode, nthreads, pq.shape[0],
                                pq.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                pg.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), ctypes.byref(work),
                                ctypes.byref(ovf))
    if rc != 0:
        raise RuntimeError(f"oracle_count_pairs failed rc={rc}")
    if ovf.value:
        raise OverflowError("oracle count exceeded 2^64-1")
    return OracleResult(out, work.value, ovf.value) if with_work else out


def enumerate_pair(Q, D, q: int, g: int, mode: int = FIND_ALL) -> np.ndarray:
    """Every embedding of query q in data graph g (enumerate mode, SURVEY
    8(f) N1): int32 [n, n_q], row k = the molecule-local data node of each
    query node (query node order) in the k-th embedding.  mode: FIND_ALL or
    INDUCED and/or WILDCARD (Find First is meaningless here)."""
    lib = _load()
    qs, ds = _as_struct(Q), _as_struct(D)
    nq = int(Q.graph_offsets[q + 1] - Q.graph_offsets[q])
    cap = 64
    while True:
        out = np.zeros((cap, max(nq, 1)), np.int32)
        n = ctypes.c_int64(0)
        rc = lib.oracle_enumerate_pair(ctypes.byref(qs), ctypes.byref(ds), int(q), int(g), int(mode) & ~FIND_FIRST,
                                       out.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), cap, ctypes.byref(n))
        if rc != 0:
            raise RuntimeError(f"oracle_enumerate_pair failed rc={rc}")
        if n.value <= cap:
            return out[:n.value, :nq]
        cap = int(n.value)


def node_sets(emb: np.ndarray) -> list:
    """NLSM's output: the distinct node SETS X = f(V_q) of a
    pair's embeddings, as sorted tuples, in sorted order."""
    return sorted({tuple(sorted(int(x) for x in row)) for row in emb})


def count_totals(Q, D, mode: int = FIND_ALL, nthreads: int | None = None, chunk: int = 100_000):
    """Per-query sums over all data graphs of count_dense (uint64 [NQ]), in
    chunks of data graphs so that large batches need no [NQ, ND] array."""
    tot = np.zeros(Q.num_graphs, np.uint64)
    for g0 in range(0, D.num_graphs, chunk):
        tot += count_dense(Q, D.slice(g0, min(g0 + chunk, D.num_graphs)), mode, nthreads).sum(axis=1, dtype=np.uint64)
    return tot
