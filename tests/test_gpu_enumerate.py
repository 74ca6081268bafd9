"""GPU parity of embedding enumeration (NLSM's output X,
PAPER.md P:446-453; atom typing needs every isomorphism): for every
GMCR pair the device's list of mappings f equals the oracle's enumerate mode
as a set, and the distinct node sets equal NLSM's X."""
import numpy as np
import pytest

import oracle
import synth
from synth import GraphBatch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sigmo():
    import torch
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_sc_carocfc25_b200 as s
    torch.cuda.set_device(0)
    return s


def decode(maps, nq):
    return sorted(tuple(int(x) for x in row[:nq]) for row in maps)


def check_enumeration(sigmo, Q, D, levels=4, induced=False, pairs=None):
    mode = oracle.INDUCED if induced else oracle.FIND_ALL
    with sigmo.Context(0) as ctx:
        ctx.set_induced(induced)
        ctx.load_batch(Q, D)
        ctx.filter(levels)
        total = ctx.enumerate(node_sets=True)
        di, qi, off, maps = ctx.embeddings()
        soff, sets = ctx.node_sets()
        counts = ctx.pair_results()[2]
    ref = oracle.count_dense(Q, D, mode)
    assert total == int(ref.sum()) == int(off[-1])
    assert np.array_equal(np.diff(off), counts)
    qsz = np.diff(Q.graph_offsets)
    ks = range(len(di)) if pairs is None else pairs
    n_checked = 0
    for k in ks:
        q, g = int(qi[k]), int(di[k])
        emb = oracle.enumerate_pair(Q, D, q, g, mode)
        got = decode(maps[off[k]:off[k + 1]], int(qsz[q]))
        assert got == sorted(map(tuple, emb.tolist())), (q, g)
        ns = [tuple(j for j in range(64) if (int(s) >> j) & 1) for s in sets[soff[k]:soff[k + 1]]]
        assert sorted(ns) == oracle.node_sets(emb), (q, g)  # device order: ascending masks
        n_checked += 1
    return n_checked


def test_enumerate_c1_every_pair(sigmo):
    """configs[0] (10 functional groups x 200 molecules, incl. > 32-atom
    molecules on the wide join launch): every pair's mappings and node sets."""
    assert check_enumeration(sigmo, synth.config_queries(1), synth.config_data(1)) > 200


def test_enumerate_c2_slice(sigmo):
    """A 5,000-molecule configs[1] slice: totals and per-pair counts of all
    pairs, full mapping / node-set comparison on a sample of 1,500 pairs."""
    Q, D = synth.config_queries(2), synth.config_data(2, first=7_000, count=5_000)
    rng = np.random.default_rng(3)
    with sigmo.Context(0) as ctx:
        ctx.load_batch(Q, D)
        ctx.filter(4)
        P = ctx.num_pairs()
    sample = sorted(int(x) for x in rng.choice(P, min(P, 1500), replace=False))
    assert check_enumeration(sigmo, Q, D, pairs=sample) == len(sample)


def test_enumerate_induced_and_edge_cases(sigmo):
    """Induced mode; single-atom queries (embeddings = label-equal atoms);
    9-11-node queries (16-byte records); benzene / naphthalene closed forms."""
    C = 6
    benzene = ([C] * 6, [(i, (i + 1) % 6, 4) for i in range(6)])
    naph = ([C] * 10, [(i, (i + 1) % 6, 4) for i in range(6)] + [(5, 6, 4), (6, 7, 4), (7, 8, 4), (8, 9, 4), (9, 0, 4)])
    Q = GraphBatch.from_graphs([benzene, ([C], []), ([7], [])])
    D = GraphBatch.from_graphs([benzene, naph, ([C, 7, C], [(0, 1, 1), (1, 2, 1)])])
    check_enumeration(sigmo, Q, D)
    with sigmo.Context(0) as ctx:
        ctx.load_batch(Q, D)
        ctx.filter(3)
        assert ctx.enumerate(node_sets=True) == 12 + 24 + 6 + 10 + 2 + 1
        di, qi, off, maps = ctx.embeddings()
        soff, sets = ctx.node_sets()
        k = [i for i in range(len(di)) if qi[i] == 0 and di[i] == 1][0]  # benzene in naphthalene
        assert off[k + 1] - off[k] == 24 and soff[k + 1] - soff[k] == 2
    check_enumeration(sigmo, synth.config_queries(1), synth.config_data(1, count=60), induced=True)
    big = GraphBatch.from_graphs(synth.random_subgraph_queries(synth.QUERY_SEED_BASE + 91, 12, kmin=9, kmax=11))
    check_enumeration(sigmo, big, synth.config_data(2, count=400))
