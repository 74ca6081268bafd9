"""Data-parallel sharding of the molecule batch (paper
section 5.4.2: static partition of molecules over ranks, queries
replicated).

One process per GPU.  Rank r owns a contiguous range of molecules chosen so
that the ranks hold (nearly) equal atom counts -- filter bytes and join work
scale with atoms -- and runs the whole hot path on it.  The only exchange step
is an all-reduce (sum) of the per-query totals, which are order-free integers,
so the sharded result equals the single-GPU result exactly.
"""
from __future__ import annotations

from typing import Optional, Sequence, Tuple

import numpy as np


def shard_bounds(graph_offsets: np.ndarray, world: int) -> np.ndarray:
    """Molecule boundaries b[0..world] (b[0]=0, b[world]=G) splitting the batch
    into `world` contiguous shards of nearly equal atom count."""
    goff = np.asarray(graph_offsets, dtype=np.int64)
    G = goff.shape[0] - 1
    V = int(goff[-1])
    if world <= 0:
        raise ValueError("world must be >= 1")
    targets = (np.arange(world + 1, dtype=np.float64) * V / world)
    # first molecule whose start reaches the atom target
    b = np.searchsorted(goff[:-1], targets, side="left").astype(np.int64) if G > 0 else np.zeros(world + 1, np.int64)
    b[0], b[-1] = 0, G
    return np.maximum.accumulate(np.minimum(b, G))


def shard_range(graph_offsets: np.ndarray, rank: int, world: int) -> Tuple[int, int]:
    b = shard_bounds(graph_offsets, world)
    return int(b[rank]), int(b[rank + 1])


def equal_count_range(n_total: int, rank: int, world: int) -> Tuple[int, int]:
    """Equal-molecule-count shard (used when molecules are generated per rank)."""
    return n_total * rank // world, n_total * (rank + 1) // world


def allreduce_totals(totals, group=None):
    """Sum per-query totals over ranks (torch int64 tensor, in place).  On the
    NCCL backend the tensor is on the rank's GPU (NVLink); on gloo it is CPU."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(totals, op=dist.ReduceOp.SUM, group=group)
    return totals


def run_shard(ctx, queries, data, levels: int, mode: int, totals_out=None, group=None):
    """Run filter + join of one rank's shard on its context and all-reduce the
    per-query totals (device int64 tensor [NQ]); returns that tensor."""
    import torch
    ctx.load_batch(queries, data)
    ctx.filter(levels)
    ctx.join(mode, total=False)
    if totals_out is None:
        totals_out = torch.zeros(ctx.nq, dtype=torch.int64, device=torch.device("cuda", ctx.device))
    ctx.query_totals(device_tensor=totals_out)
    return allreduce_totals(totals_out, group)
