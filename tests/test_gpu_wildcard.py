"""GPU parity of wildcard atoms and bonds (PAPER.md
P:2639-2645; R22): query label 0 = '*' (any atom), query bond 0 =
'~' (any bond), bit-exact vs the oracle's wildcard mode on every pair; the
filter bitmap equals the wildcard filter reference."""
import numpy as np
import pytest

import oracle
import synth
from oracle import filter_ref as fr
from synth import GraphBatch

pytestmark = pytest.mark.gpu
WC = oracle.WILDCARD


@pytest.fixture(scope="module")
def sigmo():
    import torch
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_sc_carocfc25_b200 as s
    torch.cuda.set_device(0)
    return s


def wildcarded(graphs, seed, p_atom=0.3, p_bond=0.3):
    rng = np.random.default_rng(seed)
    out = []
    for lab, edges in graphs:
        lab = [0 if rng.random() < p_atom else x for x in lab]
        edges = [(u, v, 0 if rng.random() < p_bond else b) for (u, v, b) in edges]
        out.append((lab, edges))
    return GraphBatch.from_graphs(out)


def run(sigmo, Q, D, levels=4, induced=False, ns=False, env=None):
    with sigmo.Context(0) as c:
        c.set_wildcards(True)
        c.set_induced(induced)
        c.load_batch(Q, D)
        c.filter(levels, neighbor_support=ns)
        c.join(sigmo.SIGMO_FIND_ALL)
        fa = c.dense_results()
        c.join(sigmo.SIGMO_FIND_FIRST)
        ff = c.dense_results()
        bm = c.candidates()
        npairs = c.num_pairs()
    return fa, ff, bm, npairs


@pytest.mark.parametrize("induced", [False, True], ids=["mono", "induced"])
def test_wildcard_random_tiny(sigmo, induced):
    rng = np.random.default_rng(17)
    ds = [synth.random_labelled_graph(rng, int(rng.integers(1, 9)), float(rng.uniform(0.2, 0.8)),
                                      labels=(6, 7, 8), bonds=(1, 2)) for _ in range(60)]
    qs = [synth.random_labelled_graph(rng, int(rng.integers(1, 6)), float(rng.uniform(0.3, 1.0)),
                                      labels=(6, 7), bonds=(1, 2)) for _ in range(50)]
    Q, D = wildcarded(qs, 5), GraphBatch.from_graphs(ds)
    im = oracle.INDUCED if induced else 0
    ref = oracle.count_dense(Q, D, WC | im)
    assert ref.sum() > 100
    fa, ff, _, _ = run(sigmo, Q, D, levels=3, induced=induced)
    assert np.array_equal(fa, ref)
    assert np.array_equal(ff, (ref > 0).astype(np.uint64))


@pytest.mark.parametrize("levels", [1, 2, 4])
def test_wildcard_c1_bitmap_and_counts(sigmo, levels):
    """configs[0] queries with '*' atoms and '~' bonds (lane path, incl. the
    wide > 32-atom launch): bitmap = the wildcard filter reference, every pair
    = the oracle; with the neighbour-support flag too."""
    Q0, D = synth.config_queries(1), synth.config_data(1)
    Q = wildcarded(Q0.graphs(), 100 + levels)
    ref = oracle.count_dense(Q, D, WC)
    fa, ff, bm, npairs = run(sigmo, Q, D, levels=levels)
    assert np.array_equal(fa, ref) and np.array_equal(ff, (ref > 0).astype(np.uint64))
    Cb = fr.candidates_bool(Q, D, levels, wildcard=True)
    assert np.array_equal(bm, fr.to_bitmap(Cb))
    assert npairs == int(fr.gmcr(Q, D, Cb).sum())
    fa, _, bm, npairs = run(sigmo, Q, D, levels=levels, ns=True)
    assert np.array_equal(fa, ref)
    F = fr.neighbour_support(Q, D, Cb, wildcard=True)
    assert np.array_equal(bm, fr.to_bitmap(F))
    assert npairs == int(fr.gmcr(Q, D, F).sum())


def test_wildcard_c2_slice_and_general_path(sigmo, monkeypatch):
    """A 5,000-molecule configs[1] slice with wildcarded queries on the lane
    path, and the general join (forced) on ring-system queries with
    wildcards: every pair = the oracle."""
    Q = wildcarded(synth.config_queries(2).graphs(), 7, 0.2, 0.2)
    D = synth.config_data(2, first=3_000, count=5_000)
    fa, ff, _, _ = run(sigmo, Q, D, levels=2)
    ref = oracle.count_dense(Q, D, WC)
    assert np.array_equal(fa, ref) and np.array_equal(ff, (ref > 0).astype(np.uint64))
    Qr = wildcarded(synth.config_queries(4).graphs()[-6:] + synth.config_queries(1).graphs()[:4], 9, 0.15, 0.15)
    Dr = synth.config_data(4, count=300)
    fa, ff, _, _ = run(sigmo, Qr, Dr, levels=3)
    ref = oracle.count_dense(Qr, Dr, WC)
    assert np.array_equal(fa, ref) and np.array_equal(ff, (ref > 0).astype(np.uint64))
    monkeypatch.setenv("SIGMO_JOIN_LEGACY", "1")
    fa, ff, _, _ = run(sigmo, Q, synth.config_data(2, count=500), levels=3)
    ref = oracle.count_dense(Q, synth.config_data(2, count=500), WC)
    assert np.array_equal(fa, ref) and np.array_equal(ff, (ref > 0).astype(np.uint64))
