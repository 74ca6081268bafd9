"""Streamed batches (10M molecules in batches of 250k per
GPU) and query-size routing, above the C ABI.

Data batches go through three contexts used in turn, each on its own CUDA
stream and driven from its own host thread: while the GPU runs filter + join
of batch i in one context, batch i+1 is loaded (``sigmo_load_batch``: H2D
copy, device validation and packing) into the next one, so the copies
overlap the kernels of batch i.  Per-query totals are accumulated on the
device (int64 adds on the context's stream) and read back once.

Query routing: the per-lane join (``k_join_lane``) handles queries of at most
``LANE_MAX_QUERY_NODES`` nodes; a query set with larger ones (the 20-30-atom
ring systems of configs[3]/[4]) is split into two groups, each with its own
contexts, so that the small queries keep the fast path and only the large
ones take the dense-bitmap path.  Counts are exact integers, so the split
and the batching leave every per-query total unchanged (P6 additivity).
"""
from __future__ import annotations

from typing import Iterable, List, Optional

import numpy as np

from . import Context, SIGMO_FIND_ALL

LANE_MAX_QUERY_NODES = 11  # csrc/sigmo_internal.h kJoinLaneMaxQ


class HostBatch:
    """Plain CSR-GO arrays (the fields ``as_c_batch`` reads)."""

    def __init__(self, graph_offsets, row_offsets, col_indices, node_labels, edge_labels):
        self.graph_offsets = graph_offsets
        self.row_offsets = row_offsets
        self.col_indices = col_indices
        self.node_labels = node_labels
        self.edge_labels = edge_labels

    @property
    def num_graphs(self) -> int:
        return int(self.graph_offsets.shape[0] - 1)


def _subset(batch, idx):
    """Sub-batch of the graphs `idx` (in that order), node ids renumbered."""
    goff = np.asarray(batch.graph_offsets, dtype=np.int64)
    roff = np.asarray(batch.row_offsets, dtype=np.int64)
    col = np.asarray(batch.col_indices, dtype=np.int64)
    nlab = np.asarray(batch.node_labels, dtype=np.uint8)
    elab = np.asarray(batch.edge_labels, dtype=np.uint8)
    g_off, r_off, cols, nls, els = [0], [0], [], [], []
    for g in idx:
        a, b = int(goff[g]), int(goff[g + 1])
        e0, e1 = int(roff[a]), int(roff[b])
        base = g_off[-1]
        g_off.append(base + (b - a))
        r_off.extend((roff[a + 1:b + 1] - e0 + r_off[-1]).tolist())
        cols.append(col[e0:e1] - a + base)
        nls.append(nlab[a:b])
        els.append(elab[e0:e1])
    cat = lambda xs, dt: np.concatenate(xs).astype(dt) if xs else np.zeros(0, dt)
    return HostBatch(np.asarray(g_off, np.int64), np.asarray(r_off, np.int64), cat(cols, np.int32),
                     cat(nls, np.uint8), cat(els, np.uint8))


def split_queries(Q, max_nodes: int = LANE_MAX_QUERY_NODES) -> List[np.ndarray]:
    """Query indices grouped by join path: [small] or [small, large]."""
    sizes = np.diff(np.asarray(Q.graph_offsets, dtype=np.int64))
    small = np.nonzero(sizes <= max_nodes)[0]
    large = np.nonzero(sizes > max_nodes)[0]
    return [g for g in (small, large) if g.size > 0]


class StreamRunner:
    """Run the hot path over a sequence of data batches with ``buffers``
    rotating contexts (each on its own stream; 3 by default, so a batch's copy
    never waits for the join of the batch two earlier, which still owns the
    previous buffer); ``run`` returns the per-query totals (uint64 [NQ],
    original query order) summed over all batches."""

    def __init__(self, queries, device: int = 0, levels: int = 4, mode: int = SIGMO_FIND_ALL,
                 split: bool = True, levels_large: Optional[int] = None, induced: bool = False,
                 neighbor_support: bool = False, buffers: int = 3):
        import torch
        self.torch = torch
        self.device = device
        self.levels = levels
        # the group of large queries (general join) may filter deeper: its DFS is
        # expensive and pruning pays more (levels sweep)
        self.levels_large = levels if levels_large is None else levels_large
        self.mode = mode
        self.nq = queries.num_graphs
        groups = split_queries(queries) if split else [np.arange(self.nq)]
        if len(groups) == 1:
            self.groups = [(groups[0], queries)]
        else:
            self.groups = [(g, _subset(queries, g)) for g in groups]
        dev = torch.device("cuda", device)
        self.dev = dev
        self.nbuf = max(2, int(buffers))
        self.streams = [torch.cuda.Stream(dev) for _ in range(self.nbuf)]
        # contexts[buffer][group]
        self.ctx = [[Context(device, self.streams[b]) for _ in self.groups] for b in range(self.nbuf)]
        self.neighbor_support = neighbor_support
        from concurrent.futures import ThreadPoolExecutor
        self.pool = ThreadPoolExecutor(self.nbuf)
        import threading
        # load + filter of one batch at a time (measured: without this lock the
        # e2e step of configs[2] takes 16.0 instead of 14.6 ms)
        self.copy_lock = threading.Lock()
        if induced:  # DESIGN.md R21 (set before the first load_batch)
            for row in self.ctx:
                for c in row:
                    c.set_induced(True)
        # accumulators per buffer (each only touched on its own stream)
        self.acc = [[torch.zeros(len(g), dtype=torch.int64, device=dev) for g, _ in self.groups]
                    for _ in range(self.nbuf)]
        self.tmp = [[torch.zeros(len(g), dtype=torch.int64, device=dev) for g, _ in self.groups]
                    for _ in range(self.nbuf)]
        self.batches_done = 0
        cur = torch.cuda.current_stream(dev)
        for st in self.streams:  # the buffers above were zeroed on the current stream
            st.wait_stream(cur)

    def group_levels(self, gi: int) -> int:
        """Filter levels of query group gi (the large-query group is the second)."""
        return self.levels_large if (len(self.groups) > 1 and gi == 1) else self.levels

    def reset(self):
        for s, row in zip(self.streams, self.acc):
            with self.torch.cuda.stream(s):
                for a in row:
                    a.zero_()
        self.batches_done = 0

    def submit(self, data):
        """Enqueue one data batch (host GraphBatch or as_c_batch) on the next buffer."""
        b = self.batches_done % self.nbuf
        self._submit_on(b, data)
        self.batches_done += 1

    def _submit_on(self, b: int, data):
        torch = self.torch
        torch.cuda.set_device(self.dev)  # worker threads start on the default device
        s = self.streams[b]
        for gi, (_, qb) in enumerate(self.groups):
            c = self.ctx[b][gi]
            # load + filter of one batch at a time: their host-to-device copies go
            # through one copy engine in submission order, so the next batch's
            # large copies must not be queued ahead of this batch's small ones
            with self.copy_lock:
                c.load_batch(qb, data)  # waits only for this buffer's previous H2D
                c.filter(self.group_levels(gi), neighbor_support=self.neighbor_support)
            c.join(self.mode, total=False)
            c.query_totals(device_tensor=self.tmp[b][gi])
            with torch.cuda.stream(s):
                self.acc[b][gi].add_(self.tmp[b][gi])

    def totals(self) -> np.ndarray:
        """Synchronise all buffers and gather the totals in query order."""
        torch = self.torch
        for s in self.streams:
            s.synchronize()
        for row in self.ctx:  # the device-pointer totals path never synchronized: check capacities once
            for c in row:
                if c.nq and self.batches_done:
                    try:
                        c.check()
                    except Exception as e:
                        if "before sigmo_join" not in str(e):
                            raise
        out = np.zeros(self.nq, np.uint64)
        for gi, (idx, _) in enumerate(self.groups):
            out[idx] = sum(self.acc[b][gi] for b in range(self.nbuf)).cpu().numpy().astype(np.uint64)
        return out

    def run(self, batches: Iterable) -> np.ndarray:
        """All batches, the two buffers driven from two host threads: a buffer's
        sigmo_load_batch (copy, device validation, layout read-back) and filter
        proceed while the other buffer's join runs, so the copies overlap the
        kernels (the library releases the GIL in every call; the two contexts
        share nothing)."""
        self.reset()
        futs = [None] * self.nbuf
        for d in batches:
            b = self.batches_done % self.nbuf
            if futs[b] is not None:
                futs[b].result()  # this buffer's previous batch is enqueued
            futs[b] = self.pool.submit(self._submit_on, b, d)
            self.batches_done += 1
        for f in futs:
            if f is not None:
                f.result()
        return self.totals()

    def close(self):
        self.pool.shutdown()
        for row in self.ctx:
            for c in row:
                c.close()

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()
