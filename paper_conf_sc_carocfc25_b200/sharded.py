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
    """Equal-molecule-count shard (the paper's static split)."""
    return n_total * rank // world, n_total * (rank + 1) // world


def stream_shard_bounds(natoms, world: int, balance: str = "atoms", costs=None) -> np.ndarray:
    """Shard boundaries over a molecule stream of known atom counts:
    balance = "count" (equal molecules, the paper's static split), "atoms"
    (equal atoms: filter bytes scale with atoms; the default) or "cost"
    (equal modelled cost, N2: `costs` per molecule, see molecule_costs)."""
    natoms = np.asarray(natoms, dtype=np.int64)
    G = natoms.shape[0]
    if balance == "count":
        return np.array([G * r // world for r in range(world + 1)], np.int64)
    if balance == "atoms":
        goff = np.concatenate([[0], np.cumsum(natoms)])
        return shard_bounds(goff, world)
    if balance == "cost":
        if costs is None:
            raise ValueError("balance='cost' needs the per-molecule costs")
        return cost_bounds(costs, world)
    raise ValueError(f"unknown balance {balance!r}")


# ---------------------------------------------------------------------------
# Rank bookkeeping of a timed multi-GPU run (bench.py): per-rank device
# times reduce with MAX (the job ends when the slowest rank ends), counts
# with SUM (whole-job throughput = all ranks' units / max time).
# ---------------------------------------------------------------------------
def rank_reduce(max_vals, sum_vals, device=None):
    """All-reduce a list of float64 per-rank times with MAX and a list of
    int64 per-rank counts with SUM (one collective each; NCCL on the rank's
    GPU, gloo on the CPU); identity without a process group."""
    import torch
    import torch.distributed as dist
    dev = device if device is not None else torch.device("cpu")
    mx = torch.tensor(list(max_vals), dtype=torch.float64, device=dev)
    sm = torch.tensor([int(x) for x in sum_vals], dtype=torch.int64, device=dev)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        dist.all_reduce(sm, op=dist.ReduceOp.SUM)
    return [float(x) for x in mx.tolist()], [int(x) for x in sm.tolist()]


def barrier():
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.barrier()


def throughput(units_total: int, steps: int, max_ms: float) -> float:
    """Whole-job rate: units of all ranks over the slowest rank's time."""
    return units_total * steps / (max_ms / 1000.0) if max_ms > 0 else 0.0


# ---------------------------------------------------------------------------
# Cost-model partitioning.  The paper's static
# equal-molecule split leaves a 4-8 % runtime CV across GPUs and names
# adaptive load balancing as the remedy.  Here the per-molecule
# cost of a batch is modelled from what the filter already produced -- its
# atom count (filter bytes) plus its GMCR pairs (join work, section 4.5
# P:1240-1282) -- gathered over ranks once, and the next batch of the same
# molecules (streaming, repeated queries) is split at equal modelled cost.
# ---------------------------------------------------------------------------
def cost_bounds(costs, world: int) -> np.ndarray:
    """Molecule boundaries b[0..world] splitting a per-molecule cost vector into
    `world` contiguous shards of nearly equal summed cost (each shard's excess
    over the ideal share is below the largest single-molecule cost)."""
    c = np.asarray(costs, dtype=np.float64)
    if world <= 0:
        raise ValueError("world must be >= 1")
    if c.ndim != 1 or (c.size and c.min() < 0):
        raise ValueError("costs must be a 1-D non-negative vector")
    G = c.shape[0]
    pref = np.concatenate([[0.0], np.cumsum(c)])
    targets = np.arange(world + 1, dtype=np.float64) * pref[-1] / world
    b = np.searchsorted(pref[:-1], targets, side="left").astype(np.int64) if G > 0 else np.zeros(world + 1, np.int64)
    b[0], b[-1] = 0, G
    return np.maximum.accumulate(np.minimum(b, G))


def molecule_costs(graph_offsets, pair_data_idx, w_atom: float = 1.0, w_pair: float = 4.0) -> np.ndarray:
    """Per-molecule cost model: w_atom * atoms + w_pair * GMCR pairs of the
    molecule.  pair_data_idx: data-graph index of every surviving pair
    (Context.pair_results()[0], local indices)."""
    goff = np.asarray(graph_offsets, dtype=np.int64)
    G = goff.shape[0] - 1
    pairs = np.bincount(np.asarray(pair_data_idx, dtype=np.int64), minlength=G)[:G] if G > 0 else np.zeros(0)
    return w_atom * np.diff(goff).astype(np.float64) + w_pair * pairs.astype(np.float64)


def measured_costs(graph_offsets, ms: float) -> np.ndarray:
    """Feedback cost model (adaptive balancing, N2): the rank's measured device
    time of its previous batch spread over its molecules by atoms -- every
    molecule of a shard costs atoms x (ms / atoms of the shard).  Gathered over
    ranks and split with cost_bounds, shards that ran slow per atom (e.g.
    ring-rich regions of a library) shrink for the next batch."""
    natoms = np.diff(np.asarray(graph_offsets, dtype=np.int64)).astype(np.float64)
    tot = natoms.sum()
    return natoms * (float(ms) / tot) if tot > 0 else natoms


def gather_costs(local_costs, group=None) -> np.ndarray:
    """Concatenate every rank's per-molecule costs in rank order (the ranks'
    shards are contiguous and ordered).  All-gathers the lengths, then the
    zero-padded vectors (float64; CPU tensors on gloo, device tensors on NCCL)."""
    import torch
    import torch.distributed as dist
    loc = np.asarray(local_costs, dtype=np.float64)
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return loc.copy()
    world = dist.get_world_size(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl" else torch.device("cpu")
    n = torch.tensor([loc.shape[0]], dtype=torch.int64, device=dev)
    ns = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(ns, n, group=group)
    ns = [int(x.item()) for x in ns]
    m = max(max(ns), 1)
    buf = torch.zeros(m, dtype=torch.float64, device=dev)
    buf[:loc.shape[0]] = torch.from_numpy(loc).to(dev)
    outs = [torch.zeros_like(buf) for _ in range(world)]
    dist.all_gather(outs, buf, group=group)
    return np.concatenate([o[:k].cpu().numpy() for o, k in zip(outs, ns)])


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
