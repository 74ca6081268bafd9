"""Multi-process (N>1) host logic on CPU: shard bounds and the all-reduce of
per-query totals over a world_size-2 gloo group.  The per
shard totals come from the oracle here (no GPU); on the B200 the same
reduction runs on the NCCL group with the library's device totals."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_sc_carocfc25_b200 import sharded


def test_shard_bounds_cover_and_balance():
    D = synth.molecules(123, 0, 1000)
    for world in (1, 2, 3, 4, 8):
        b = sharded.shard_bounds(D.graph_offsets, world)
        assert b[0] == 0 and b[-1] == D.num_graphs and np.all(np.diff(b) >= 0)
        atoms = [int(D.graph_offsets[b[r + 1]] - D.graph_offsets[b[r]]) for r in range(world)]
        assert sum(atoms) == D.num_nodes
        assert max(atoms) - min(atoms) <= 2 * int(D.sizes().max())
    # degenerate: more ranks than molecules, empty batch
    small = synth.molecules(1, 0, 3)
    b = sharded.shard_bounds(small.graph_offsets, 8)
    assert b[0] == 0 and b[-1] == 3 and np.all(np.diff(b) >= 0)
    e = sharded.shard_bounds(np.zeros(1, np.int64), 4)
    assert np.all(e == 0)
    assert sharded.equal_count_range(10, 1, 3) == (3, 6)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    Q = synth.config_queries(1)
    D = synth.config_data(1, count=120)
    g0, g1 = sharded.shard_range(D.graph_offsets, rank, world)
    part = D.slice(g0, g1)
    for mode in (oracle.FIND_ALL, oracle.FIND_FIRST):
        local = oracle.count_dense(Q, part, mode, nthreads=2).sum(axis=1).astype(np.int64)
        t = torch.from_numpy(local.copy())
        sharded.allreduce_totals(t)
        np.save(os.path.join(out_dir, f"r{rank}_m{mode}.npy"), t.numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_allreduce_equals_unsharded(tmp_path):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    Q = synth.config_queries(1)
    D = synth.config_data(1, count=120)
    for mode in (oracle.FIND_ALL, oracle.FIND_FIRST):
        ref = oracle.count_dense(Q, D, mode).sum(axis=1).astype(np.int64)
        for r in range(world):
            got = np.load(os.path.join(tmp_path, f"r{r}_m{mode}.npy"))
            assert np.array_equal(got, ref), (r, mode)


# ---------------------------------------------------------------- N2 cost-model partitioning
def test_cost_bounds_balance():
    rng = np.random.default_rng(3)
    for G in (0, 1, 5, 1000):
        c = rng.pareto(1.5, G) + 0.1  # heavy-tailed per-molecule cost
        for world in (1, 2, 3, 8):
            b = sharded.cost_bounds(c, world)
            assert b[0] == 0 and b[-1] == G and np.all(np.diff(b) >= 0)
            if G:
                shard = [c[b[r]:b[r + 1]].sum() for r in range(world)]
                assert abs(sum(shard) - c.sum()) < 1e-9 * c.sum()
                assert max(shard) <= c.sum() / world + c.max() + 1e-9
    # unit costs reduce to the equal-count split; atom costs to shard_bounds
    assert np.array_equal(sharded.cost_bounds(np.ones(10), 2), [0, 5, 10])
    D = synth.molecules(123, 0, 500)
    for world in (2, 4):
        assert np.array_equal(sharded.cost_bounds(D.sizes(), world), sharded.shard_bounds(D.graph_offsets, world))
    with pytest.raises(ValueError):
        sharded.cost_bounds([1.0, -1.0], 2)


def test_molecule_costs_model():
    goff = np.array([0, 3, 3, 10], np.int64)
    c = sharded.molecule_costs(goff, [0, 2, 2, 2], w_atom=1.0, w_pair=4.0)
    assert np.array_equal(c, [3 + 4, 0, 7 + 12])


def _cost_worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    Q = synth.config_queries(1)
    D = synth.config_data(1, count=150)
    g0, g1 = sharded.shard_range(D.graph_offsets, rank, world)
    part = D.slice(g0, g1)
    # GMCR-pair proxy on CPU: the oracle's positive pairs of the shard (local indices)
    dense = oracle.count_dense(Q, part, oracle.FIND_FIRST, nthreads=2)
    local = sharded.molecule_costs(part.graph_offsets, np.nonzero(dense)[1])
    glob = sharded.gather_costs(local)
    np.save(os.path.join(out_dir, f"c{rank}.npy"), glob)
    np.save(os.path.join(out_dir, f"b{rank}.npy"), sharded.cost_bounds(glob, world))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_gathered_costs_equal_unsharded(tmp_path):
    world = 2
    mp.spawn(_cost_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    Q = synth.config_queries(1)
    D = synth.config_data(1, count=150)
    dense = oracle.count_dense(Q, D, oracle.FIND_FIRST)
    ref = sharded.molecule_costs(D.graph_offsets, np.nonzero(dense)[1])
    for r in range(world):
        assert np.array_equal(np.load(os.path.join(tmp_path, f"c{r}.npy")), ref)
        assert np.array_equal(np.load(os.path.join(tmp_path, f"b{r}.npy")), sharded.cost_bounds(ref, world))


# ---------------------------------------------------------------- bench rank logic (gloo world 2)
def _rank_worker(rank, world, port, out_dir):
    """What bench.py does at N>1 minus the GPU: each rank takes its shard of the
    world x M molecule stream (atom-balanced bounds computed from the stream's
    atom counts, identically on every rank), times its 'steps', and the ranks
    reduce times with MAX and counts with SUM (sharded.rank_reduce)."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    M = 150
    sizes = synth.molecule_sizes(synth.DATA_SEED_BASE + 1, 0, M * world)
    out = {}
    for bal in ("count", "atoms"):
        b = sharded.stream_shard_bounds(sizes, world, bal)
        Q = synth.config_queries(1)
        D = synth.config_data(1, first=int(b[rank]), count=int(b[rank + 1] - b[rank]))
        sharded.barrier()
        counts = oracle.count_dense(Q, D, nthreads=2)
        fake_ms = 10.0 + rank  # a per-rank device time
        (mx,), (matches, pairs) = sharded.rank_reduce([fake_ms], [int(counts.sum()), Q.num_graphs * D.num_graphs])
        out[bal] = (b.tolist(), mx, matches, pairs, sharded.throughput(matches, 1, mx))
    # the cost split (N2): gathered per-molecule costs, identical bounds on all ranks
    b = sharded.stream_shard_bounds(sizes, world, "atoms")
    D = synth.config_data(1, first=int(b[rank]), count=int(b[rank + 1] - b[rank]))
    local = sharded.molecule_costs(D.graph_offsets, np.repeat(np.arange(D.num_graphs), 2))
    costs = sharded.gather_costs(local)
    out["cost"] = sharded.stream_shard_bounds(sizes, world, "cost", costs=costs).tolist()
    np.save(os.path.join(out_dir, f"rank{rank}.npy"), np.array([out], dtype=object), allow_pickle=True)
    dist.destroy_process_group()


def test_gloo_world2_bench_rank_logic(tmp_path):
    world = 2
    mp.spawn(_rank_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    outs = [np.load(os.path.join(tmp_path, f"rank{r}.npy"), allow_pickle=True)[0] for r in range(world)]
    M = 150
    Q = synth.config_queries(1)
    D = synth.config_data(1, count=M * world)
    total = int(oracle.count_dense(Q, D).sum())
    sizes = synth.molecule_sizes(synth.DATA_SEED_BASE + 1, 0, M * world)
    for bal in ("count", "atoms"):
        b0, mx0, m0, p0, v0 = outs[0][bal]
        b1, mx1, m1, p1, v1 = outs[1][bal]
        assert b0 == b1 and b0[0] == 0 and b0[-1] == M * world   # identical, covering bounds
        assert mx0 == mx1 == 11.0                                # MAX of the per-rank times
        assert m0 == m1 == total                                  # SUM of the per-rank matches
        assert p0 == Q.num_graphs * M * world
        assert v0 == total / 0.011
    atoms = [int(sizes[outs[0]["atoms"][0][r]:outs[0]["atoms"][0][r + 1]].sum()) for r in range(world)]
    assert abs(atoms[0] - atoms[1]) <= int(sizes.max())            # atom-balanced within one molecule
    assert outs[0]["cost"] == outs[1]["cost"]
