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
