"""GPU parity of the induced-subgraph mode (R21)
through the C ABI (sigmo_set_induced) vs the oracle's induced mode (mode
bit 2), bit-exact on every pair: tiny random graphs, edge cases (empty,
single-atom, > 64-atom graphs, disconnected and single-node queries), the
configs[0] library, a configs[1] slice and the 20-30-atom ring-system queries."""
import numpy as np
import pytest

import oracle
import synth
from synth import GraphBatch

pytestmark = pytest.mark.gpu
IND = oracle.INDUCED


@pytest.fixture(scope="module")
def sigmo():
    import torch
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_sc_carocfc25_b200 as s
    torch.cuda.set_device(0)
    return s


@pytest.fixture()
def ctx(sigmo):
    c = sigmo.Context(0)
    c.set_induced(True)
    yield c
    c.close()


def check(ctx, sigmo, Q, D, levels=4):
    ctx.load_batch(Q, D)
    ctx.filter(levels)
    tot = ctx.join(sigmo.SIGMO_FIND_ALL)
    ref = oracle.count_dense(Q, D, IND)
    got = ctx.dense_results()
    assert np.array_equal(got, ref)
    assert tot == int(ref.sum())
    ctx.join(sigmo.SIGMO_FIND_FIRST)
    assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D, IND | oracle.FIND_FIRST))
    return ref


def test_induced_random_tiny(ctx, sigmo):
    rng = np.random.default_rng(4242)
    ds = [synth.random_labelled_graph(rng, int(rng.integers(0, 12)), float(rng.uniform(0.1, 0.8)),
                                      labels=(6, 7), bonds=(1, 2)) for _ in range(400)]
    qs = [synth.random_labelled_graph(rng, int(rng.integers(1, 7)), float(rng.uniform(0.3, 1.0)),
                                      labels=(6, 7), bonds=(1, 2)) for _ in range(40)]
    Q, D = GraphBatch.from_graphs(qs), GraphBatch.from_graphs(ds)
    for L in (1, 3):
        ref = check(ctx, sigmo, Q, D, L)
    assert (ref < oracle.count_dense(Q, D)).sum() > 100  # induced pruning is exercised


def test_induced_edge_cases(ctx, sigmo):
    graphs = synth.molecules(synth.DATA_SEED_BASE + 77, 0, 120, mode=2).graphs()
    graphs.insert(0, ([], []))
    graphs.insert(5, ([6], []))
    graphs.append(([6, 6, 8, 6], [(0, 1, 1), (2, 3, 1)]))
    graphs.insert(50, ([6] * 100, [(i, i + 1, 1) for i in range(99)] + [(0, 99, 1)]))
    graphs.append(([6] * 4, [(i, j, 1) for i in range(4) for j in range(i + 1, 4)]))  # K4
    D = GraphBatch.from_graphs(graphs)
    qs = synth.library(synth.C1_NAMES) + [([6], []), ([6, 8], []), ([6, 6], []), ([6, 6, 6], [(0, 1, 1)]),
                                          ([6] * 3, [(0, 1, 1), (1, 2, 1)]),
                                          ([6] * 4, [(0, 1, 1), (1, 2, 1), (2, 3, 1), (3, 0, 1)])]
    check(ctx, sigmo, GraphBatch.from_graphs(qs), D)


def test_induced_c1_and_c2_slice(ctx, sigmo):
    check(ctx, sigmo, synth.config_queries(1), synth.config_data(1))
    D = synth.config_data(2, count=20000)
    check(ctx, sigmo, synth.config_queries(2), D)


def test_induced_ring_systems(ctx, sigmo):
    check(ctx, sigmo, synth.config_queries(4), synth.config_data(4, count=300))


def test_induced_toggle_restores_monomorphism(ctx, sigmo):
    Q, D = synth.config_queries(1), synth.config_data(1)
    ctx.set_induced(False)
    ctx.load_batch(Q, D)
    ctx.filter(4)
    ctx.join(sigmo.SIGMO_FIND_ALL)
    assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D))


def test_induced_general_path_forced(sigmo, monkeypatch):
    """the same batches through the general k_join (SIGMO_JOIN_LEGACY routes
    the load away from the lane join) -- both induced implementations agree
    with the oracle."""
    monkeypatch.setenv("SIGMO_JOIN_LEGACY", "1")
    c = sigmo.Context(0)
    c.set_induced(True)
    try:
        check(c, sigmo, synth.config_queries(1), synth.config_data(1))
        check(c, sigmo, synth.config_queries(2), synth.config_data(2, count=5000))
    finally:
        c.close()
