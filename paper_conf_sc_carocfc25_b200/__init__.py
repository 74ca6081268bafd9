"""B200-native SIGMo hot path: thin Python binding over libsigmo.so.

The binding only marshals arguments; every step of the path (signatures,
filter, GMCR, join, reductions) runs in the CUDA kernels of ``csrc/``.
PyTorch is used for streams and the process group only.  See
``include/sigmo.h`` for the contract of each call and DESIGN.md for the
design.
"""
from __future__ import annotations

import ctypes
from typing import Optional

import numpy as np

from . import _native
from ._native import (SIGMO_FILTER_NEIGHBOR_SUPPORT, SIGMO_FIND_ALL, SIGMO_FIND_FIRST, STATUS_NAMES,
                      load_library)

__all__ = ["Context", "SigmoError", "validate_batch", "load_library", "SIGMO_FIND_ALL", "SIGMO_FIND_FIRST",
           "SIGMO_FILTER_NEIGHBOR_SUPPORT", "as_c_batch"]


class SigmoError(RuntimeError):
    def __init__(self, status: int, message: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {message}")
        self.status = status
        self.message = message


def _arr(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def _pinned(a, dt):
    """A copy of `a` in page-locked host memory (torch's pinned allocator), so
    that sigmo_load_batch's copies of it are plain DMA."""
    import torch
    t = torch.from_numpy(np.ascontiguousarray(a, dtype=dt)).pin_memory()
    return t.numpy(), t


class _CBatch:
    """Keeps the numpy arrays alive while the C struct points at them.
    pinned=True: the arrays are copied once into page-locked memory (what a
    data loader feeding the GPU holds)."""

    def __init__(self, b, pinned: bool = False):
        self._keep = []
        conv = _arr
        if pinned:
            def conv(a, dt):
                x, t = _pinned(a, dt)
                self._keep.append(t)
                return x
        self.goff = conv(b.graph_offsets, np.int64)
        self.roff = conv(b.row_offsets, np.int64)
        self.col = conv(b.col_indices, np.int32)
        self.nlab = conv(b.node_labels, np.uint8)
        self.elab = conv(b.edge_labels, np.uint8)
        s = _native.sigmo_graph_batch()
        s.num_graphs = int(self.goff.shape[0] - 1)
        s.num_nodes = int(self.nlab.shape[0])
        s.graph_offsets = self.goff.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
        s.row_offsets = self.roff.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
        s.col_indices = self.col.ctypes.data_as(ctypes.POINTER(ctypes.c_int32))
        s.node_labels = self.nlab.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))
        s.edge_labels = self.elab.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))
        self.struct = s
        self.num_graphs = s.num_graphs
        self.num_nodes = s.num_nodes


def as_c_batch(b, pinned: bool = False) -> _CBatch:
    return b if isinstance(b, _CBatch) else _CBatch(b, pinned)


def validate_batch(batch, is_query: bool):
    """sigmo_validate_batch: host-only structural validation -> (status, message)."""
    lib = load_library()
    cb = as_c_batch(batch)
    buf = ctypes.create_string_buffer(512)
    st = lib.sigmo_validate_batch(ctypes.byref(cb.struct), 1 if is_query else 0, buf, 512)
    return st, buf.value.decode()


def _stream_handle(stream) -> int:
    if stream is None:
        import torch
        return int(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return stream
    return int(stream.cuda_stream)


def _torch_allocator(device: int):
    """sigmo_allocator backed by PyTorch's caching allocator (include/sigmo.h
    sigmo_create; SURVEY 8(b) ownership): the library's device buffers come
    from, and return to, torch's pool on the ctx stream."""
    import torch

    def alloc(nbytes, stream, user):
        try:
            return int(torch.cuda.caching_allocator_alloc(int(nbytes), device, int(stream or 0)))
        except Exception:  # out of memory: the library reports SIGMO_ERR_OOM
            return None

    def free(ptr, stream, user):
        try:
            torch.cuda.caching_allocator_delete(int(ptr))
        except Exception:  # interpreter teardown: the process is exiting anyway
            pass

    a = _native.sigmo_allocator()
    a.alloc = _native.ALLOC_FN(alloc)
    a.free = _native.FREE_FN(free)
    a.user = None
    return a


class Context:
    """One sigmo_ctx: a device, a stream and the device state of one batch.

    ``allocator="torch"`` (default) routes the library's device buffers through
    PyTorch's caching allocator; ``"cuda"`` uses the library's own
    cudaMallocAsync pool."""

    def __init__(self, device: int = 0, stream=None, allocator: str = "torch"):
        self._lib = load_library()
        self.device = device
        self._handle = ctypes.c_void_p()
        self._stream = _stream_handle(stream)
        self._alloc = _torch_allocator(device) if allocator == "torch" else None
        st = self._lib.sigmo_create(device, ctypes.c_void_p(self._stream),
                                    ctypes.byref(self._alloc) if self._alloc is not None else None,
                                    ctypes.byref(self._handle))
        if st != 0:
            raise SigmoError(st, f"sigmo_create(device={device}) failed")
        self.nq = self.nd = self.vq = self.vd = 0

    # -- helpers --
    def _check(self, st: int, what: str):
        if st != 0:
            msg = self._lib.sigmo_last_error(self._handle)
            raise SigmoError(st, f"{what}: {msg.decode() if msg else ''}")

    def close(self):
        if self._handle:
            self._lib.sigmo_destroy(self._handle)
            self._handle = ctypes.c_void_p()

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- ABI calls --
    def load_batch(self, queries, data):
        cq, cd = as_c_batch(queries), as_c_batch(data)
        self._check(self._lib.sigmo_load_batch(self._handle, ctypes.byref(cq.struct), ctypes.byref(cd.struct)),
                    "sigmo_load_batch")
        self.nq, self.nd, self.vq, self.vd = cq.num_graphs, cd.num_graphs, cq.num_nodes, cd.num_nodes
        return self

    def filter(self, levels: int = 4, neighbor_support: bool = False, flags: Optional[int] = None):
        f = flags if flags is not None else (SIGMO_FILTER_NEIGHBOR_SUPPORT if neighbor_support else 0)
        self._check(self._lib.sigmo_filter(self._handle, int(levels), int(f)), "sigmo_filter")
        return self

    def join(self, mode=SIGMO_FIND_ALL, total: bool = True):
        if isinstance(mode, str):
            mode = {"all": SIGMO_FIND_ALL, "first": SIGMO_FIND_FIRST}[mode]
        if total:
            t = ctypes.c_uint64(0)
            self._check(self._lib.sigmo_join(self._handle, int(mode), ctypes.byref(t)), "sigmo_join")
            return int(t.value)
        self._check(self._lib.sigmo_join(self._handle, int(mode), None), "sigmo_join")
        return None

    def num_pairs(self) -> int:
        n = ctypes.c_int64(0)
        self._check(self._lib.sigmo_num_pairs(self._handle, ctypes.byref(n)), "sigmo_num_pairs")
        return int(n.value)

    def pair_results(self):
        P = self.num_pairs()
        di = np.zeros(P, np.int64)
        qi = np.zeros(P, np.int32)
        r = np.zeros(P, np.uint64)
        n = ctypes.c_int64(0)
        self._check(self._lib.sigmo_get_pair_results(self._handle, P, ctypes.byref(n),
                                                     di.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                                     qi.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)),
                                                     r.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))),
                    "sigmo_get_pair_results")
        return di, qi, r

    def dense_results(self) -> np.ndarray:
        out = np.zeros((self.nq, self.nd), np.uint64)
        self._check(self._lib.sigmo_get_dense_results(self._handle,
                                                      out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))),
                    "sigmo_get_dense_results")
        return out

    def query_totals(self, device_tensor=None):
        """Host numpy uint64 [NQ], or copy into a device tensor (torch int64/uint64, NQ)."""
        if device_tensor is not None:
            self._check(self._lib.sigmo_get_query_totals(self._handle, ctypes.c_void_p(device_tensor.data_ptr()), 1),
                        "sigmo_get_query_totals")
            return device_tensor
        out = np.zeros(self.nq, np.uint64)
        self._check(self._lib.sigmo_get_query_totals(self._handle, ctypes.c_void_p(out.ctypes.data), 0),
                    "sigmo_get_query_totals")
        return out

    def candidates(self) -> np.ndarray:
        W = (self.vd + 31) // 32
        out = np.zeros((self.vq, W), np.uint32)
        self._check(self._lib.sigmo_get_candidates(self._handle, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))),
                    "sigmo_get_candidates")
        return out

    def signatures(self, which: int, radius: int) -> np.ndarray:
        n = self.vq if which == 0 else self.vd
        out = np.zeros(n, np.uint64)
        self._check(self._lib.sigmo_get_signatures(self._handle, int(which), int(radius),
                                                   out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))),
                    "sigmo_get_signatures")
        return out

    def packed_batch(self, which: int):
        """sigmo_get_packed_batch: the CSR-GO arrays as packed on the device
        (graph_offsets, row_offsets, col_indices, node_labels, edge_labels)."""
        G, V, E = ctypes.c_int64(0), ctypes.c_int64(0), ctypes.c_int64(0)
        self._check(self._lib.sigmo_get_packed_batch(self._handle, int(which), ctypes.byref(G), ctypes.byref(V),
                                                     ctypes.byref(E), None, None, None, None, None),
                    "sigmo_get_packed_batch")
        go, ro = np.zeros(G.value + 1, np.int64), np.zeros(V.value + 1, np.int64)
        co, nl, el = np.zeros(E.value, np.int32), np.zeros(V.value, np.uint8), np.zeros(E.value, np.uint8)
        P = ctypes.POINTER
        self._check(self._lib.sigmo_get_packed_batch(
            self._handle, int(which), None, None, None, go.ctypes.data_as(P(ctypes.c_int64)),
            ro.ctypes.data_as(P(ctypes.c_int64)), co.ctypes.data_as(P(ctypes.c_int32)),
            nl.ctypes.data_as(P(ctypes.c_uint8)), el.ctypes.data_as(P(ctypes.c_uint8))), "sigmo_get_packed_batch")
        return go, ro, co, nl, el

    def enumerate(self, node_sets: bool = False) -> int:
        """sigmo_enumerate: every embedding of every GMCR
        pair, written on the device; returns the total."""
        n = ctypes.c_int64(0)
        self._check(self._lib.sigmo_enumerate(self._handle, _native.SIGMO_ENUM_NODE_SETS if node_sets else 0,
                                              ctypes.byref(n)), "sigmo_enumerate")
        return int(n.value)

    def embeddings(self):
        """(data_idx [P], query_idx [P], offsets [P+1], maps uint8 [n, stride]): pair k's
        embeddings are maps[offsets[k]:offsets[k+1]], column i = data node of query node i."""
        P, n, st = ctypes.c_int64(0), ctypes.c_int64(0), ctypes.c_int32(0)
        null = None
        self._check(self._lib.sigmo_get_embeddings(self._handle, 0, ctypes.byref(P), null, null, null, 0, null,
                                                   ctypes.byref(n), ctypes.byref(st)), "sigmo_get_embeddings")
        di, qi = np.zeros(P.value, np.int64), np.zeros(P.value, np.int32)
        off, maps = np.zeros(P.value + 1, np.int64), np.zeros((n.value, st.value), np.uint8)
        Pt = ctypes.POINTER
        self._check(self._lib.sigmo_get_embeddings(
            self._handle, P.value, ctypes.byref(P), di.ctypes.data_as(Pt(ctypes.c_int64)),
            qi.ctypes.data_as(Pt(ctypes.c_int32)), off.ctypes.data_as(Pt(ctypes.c_int64)), n.value,
            maps.ctypes.data_as(Pt(ctypes.c_uint8)), ctypes.byref(n), ctypes.byref(st)), "sigmo_get_embeddings")
        return di, qi, off, maps

    def node_sets(self):
        """(offsets [P+1], sets uint64 [n]) of the distinct node sets per pair
        (bit j = molecule-local data node j), pairs in embeddings() order."""
        P, n = ctypes.c_int64(0), ctypes.c_int64(0)
        self._check(self._lib.sigmo_get_node_sets(self._handle, 0, ctypes.byref(P), None, 0, None, ctypes.byref(n)),
                    "sigmo_get_node_sets")
        off, sets = np.zeros(P.value + 1, np.int64), np.zeros(n.value, np.uint64)
        Pt = ctypes.POINTER
        self._check(self._lib.sigmo_get_node_sets(self._handle, P.value, ctypes.byref(P),
                                                  off.ctypes.data_as(Pt(ctypes.c_int64)), n.value,
                                                  sets.ctypes.data_as(Pt(ctypes.c_uint64)), ctypes.byref(n)),
                    "sigmo_get_node_sets")
        return off, sets

    def check(self):
        """sigmo_check_join: raise if the last join exceeded an internal capacity."""
        self._check(self._lib.sigmo_check_join(self._handle), "sigmo_check_join")

    def set_induced(self, enable: bool = True):
        """Induced-subgraph mode for the next load_batch (include/sigmo.h sigmo_set_induced)."""
        self._check(self._lib.sigmo_set_induced(self._handle, 1 if enable else 0), "sigmo_set_induced")

    def set_wildcards(self, enable: bool = True):
        """Wildcard atoms / bonds for the next load_batch: query label 0 = '*', bond 0 = '~'
        (include/sigmo.h sigmo_set_wildcards)."""
        self._check(self._lib.sigmo_set_wildcards(self._handle, 1 if enable else 0), "sigmo_set_wildcards")

    def set_timing(self, enable=True, count_steps: bool = False):
        """bit 0: per-stage CUDA-event timing; count_steps (bit 1): the join counts its DFS steps."""
        flags = (1 if enable else 0) | (2 if count_steps else 0)
        self._check(self._lib.sigmo_set_timing(self._handle, flags), "sigmo_set_timing")

    def timings(self) -> dict:
        t = _native.sigmo_timings()
        self._check(self._lib.sigmo_get_timings(self._handle, ctypes.byref(t)), "sigmo_get_timings")
        return {k: getattr(t, k) for k, _ in t._fields_}

    @property
    def stream(self) -> int:
        return self._stream


def version() -> str:
    return load_library().sigmo_version().decode()
