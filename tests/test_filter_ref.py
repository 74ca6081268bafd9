"""Pins for the CPU filter reference (oracle/filter_ref.py): signature closed
forms, an all-pairs-distance restatement, saturation,
soundness against brute-force embeddings, monotonicity, GMCR soundness and
the neighbour-support fixed point (P8)."""
import numpy as np
import pytest

import oracle
import synth
from oracle import filter_ref as fr
from oracle.brute import brute_embeddings
from synth import GraphBatch

C, N, O = 6, 7, 8


def ring(n, lab=C, bond=1):
    return [lab] * n, [(i, (i + 1) % n, bond) for i in range(n)]


def path(n, lab=C, bond=1):
    return [lab] * n, [(i, i + 1, bond) for i in range(n - 1)]


def star(d, lab=C, bond=1):
    return [lab] * (d + 1), [(0, i, bond) for i in range(1, d + 1)]


def carbon_count(B, r):
    return fr.raw_signatures(B, r)[r][:, fr.field_of(C)]


def test_field_table_is_64_bits_and_lsb_first():
    assert sum(w for _, w in fr.FIELDS) == 64
    assert fr.OFFSETS[0] == 0 and fr.field_of(C) == 0 and fr.field_of(200) == fr.NF - 1


def test_signature_closed_forms_cycles():
    for n in range(3, 12):
        B = GraphBatch.from_graphs([ring(n)])
        for r in range(1, 8):
            assert np.all(carbon_count(B, r) == min(2 * r, n - 1)), (n, r)


def test_signature_closed_forms_benzene_and_star():
    B = GraphBatch.from_graphs([ring(6, C, 4)])
    assert [int(carbon_count(B, r)[0]) for r in (1, 2, 3, 4)] == [2, 4, 5, 5]
    S = GraphBatch.from_graphs([star(3)])
    for r in (1, 2, 3):
        c = carbon_count(S, r)
        assert c[0] == 3
        assert np.all(c[1:] == (1 if r == 1 else 3))


def test_signature_pack_and_saturation():
    # chain of 100 N atoms: N field is 6 bits, saturates at 63 (R8)
    B = GraphBatch.from_graphs([path(100, N)])
    r = 60
    sig = fr.signatures(B, r)
    nf = fr.field_of(N)
    vals = (sig >> np.uint64(fr.OFFSETS[nf])) & np.uint64(63)
    raw = fr.raw_signatures(B, r)[r][:, nf]
    assert raw.max() > 63
    assert np.array_equal(vals.astype(np.int64), np.minimum(raw, 63))
    # other fields are zero
    mask = np.uint64(((1 << 6) - 1) << int(fr.OFFSETS[nf]))
    assert np.all(sig & ~mask == 0)


def test_incremental_ring_update_equals_cumulative_distance_count():
    """Alg. 1's ring update (R_k = N^k \\ N^(k-1)) accumulated over k equals the
    direct count of nodes within distance k (R4), via Floyd-Warshall."""
    rng = np.random.default_rng(5)
    gs = [synth.random_labelled_graph(rng, int(rng.integers(1, 12)), 0.25, labels=(C, N, O, 16, 9))
          for _ in range(30)]
    B = GraphBatch.from_graphs(gs)
    S = fr.raw_signatures(B, 5)
    base = 0
    for lab, edges in gs:
        n = len(lab)
        d = np.full((n, n), 10 ** 6)
        np.fill_diagonal(d, 0)
        for (u, v, _) in edges:
            d[u, v] = d[v, u] = 1
        for k in range(n):
            d = np.minimum(d, d[:, k:k + 1] + d[k:k + 1, :])
        for r in range(1, 6):
            for v in range(n):
                for f in range(fr.NF):
                    want = sum(1 for u in range(n) if u != v and d[v, u] <= r and fr.field_of(lab[u]) == f)
                    assert S[r][base + v, f] == want
        base += n


def test_candidates_level1_is_label_equality_and_monotone():
    D = synth.molecules(synth.DATA_SEED_BASE + 1, 0, 40)
    Q = synth.config_queries(1)
    C1 = fr.candidates_bool(Q, D, 1)
    assert np.array_equal(C1, Q.node_labels[:, None] == D.node_labels[None, :])
    prev = C1
    for L in range(2, 6):
        CL = fr.candidates_bool(Q, D, L)
        assert not np.any(CL & ~prev)  # C_{L} subset of C_{L-1}
        prev = CL
    assert prev.sum() < C1.sum()


def _embedding_images(qs, ds):
    """set of (global query node, global data node) used by some embedding."""
    used = set()
    qb = 0
    for q in qs:
        db = 0
        for d in ds:
            for f in brute_embeddings(q, d):
                for i, v in enumerate(f):
                    used.add((qb + i, db + v))
            db += len(d[0])
        qb += len(q[0])
    return used


def test_filter_soundness_vs_brute_embeddings():
    rng = np.random.default_rng(77)
    ds = [synth.random_labelled_graph(rng, int(rng.integers(2, 8)), 0.45, labels=(C, N), bonds=(1, 2))
          for _ in range(25)]
    qs = [synth.random_labelled_graph(rng, int(rng.integers(1, 5)), 0.6, labels=(C, N), bonds=(1, 2))
          for _ in range(25)]
    Q, D = GraphBatch.from_graphs(qs), GraphBatch.from_graphs(ds)
    used = _embedding_images(qs, ds)
    assert len(used) > 50
    counts = oracle.count_dense(Q, D)
    for L in (1, 2, 3, 4, 6):
        for ns in (False, True):
            Cb = fr.candidates_bool(Q, D, L)
            if ns:
                Cb = fr.neighbour_support(Q, D, Cb)
            for (vq, vd) in used:
                assert Cb[vq, vd], (L, ns, vq, vd)
            G = fr.gmcr(Q, D, Cb)
            assert np.all(counts[~G] == 0)  # GMCR-pruned pairs have no embedding


def test_exact_distance_signatures_would_be_unsound():
    """R4 counterexample: P4 (path of 4 C) embeds into C5, but an exact-distance
    (ring-only) signature would prune it; the cumulative reading keeps it."""
    q, d = path(4), ring(5)
    Q, D = GraphBatch.from_graphs([q]), GraphBatch.from_graphs([d])
    assert oracle.count_dense(Q, D)[0, 0] == 10
    SQ, SD = fr.raw_signatures(Q, 3), fr.raw_signatures(D, 3)
    exact_q = SQ[3] - SQ[2]   # nodes at distance exactly 3
    exact_d = SD[3] - SD[2]
    assert np.any(exact_q[0] > exact_d[0])  # the exact-distance rule would prune the end node
    Cb = fr.candidates_bool(Q, D, 4)
    assert Cb.all(axis=1).all()


def test_neighbour_support_fixed_point_properties():
    D = synth.molecules(synth.DATA_SEED_BASE + 3, 0, 30)
    Q = synth.config_queries(1)
    C2 = fr.candidates_bool(Q, D, 2)
    F = fr.neighbour_support(Q, D, C2)
    assert not np.any(F & ~C2)
    assert np.array_equal(fr.neighbour_support(Q, D, F), F)  # fixed point
    # greatest: any arc-consistent subset of C2 is contained in F -- the image
    # set of all embeddings is arc-consistent
    counts = oracle.count_dense(Q, D)
    G = fr.gmcr(Q, D, F)
    assert np.all(counts[~G] == 0)
    assert F.sum() <= C2.sum()


def test_bitmap_view_bit_order():
    Cb = np.zeros((2, 70), bool)
    Cb[0, 0] = Cb[0, 33] = Cb[1, 69] = True
    bm = fr.to_bitmap(Cb)
    assert bm.shape == (2, 3)
    assert bm[0, 0] == 1 and bm[0, 1] == 2 and bm[1, 2] == 1 << 5


def test_gmcr_rule_hand_computed():
    """GMCR: a pair survives iff EVERY query node has a
    candidate in the data graph.  Hand-built candidate matrix where the
    'any node' and 'every node' readings differ."""
    from synth import GraphBatch
    Q = GraphBatch.from_graphs([([C, O], [(0, 1, 1)]),       # q0: C-O
                                ([C, C], [(0, 1, 1)])])      # q1: C-C
    D = GraphBatch.from_graphs([([C, C, C], [(0, 1, 1), (1, 2, 1)]),  # g0: propane (no O)
                                ([C, O], [(0, 1, 1)])])               # g1: methanol-like
    Cb = np.zeros((4, 5), bool)
    Cb[0, [0, 1, 2, 3]] = True   # q0 node C: candidates in g0 and g1
    Cb[1, 4] = True              # q0 node O: only g1's O
    Cb[2, [0, 1, 2, 3]] = True   # q1 nodes: every C
    Cb[3, [0, 1, 2, 3]] = True
    expect = np.array([[False, True],    # q0 survives only where its O has a candidate
                       [True, True]])    # q1: both nodes have candidates in g0 and g1
    assert np.array_equal(fr.gmcr(Q, D, Cb), expect)
    Cb[3, 3] = False                      # q1's second node loses its only candidate in g1
    expect[1, 1] = False
    assert np.array_equal(fr.gmcr(Q, D, Cb), expect)


def test_neighbour_support_bond_labels_hand_computed():
    """Neighbour support (R9) with bond labels: a query C=C (double bond) on
    all-single-bond data has no support at all, so the fixed point is empty,
    although every data C has a C neighbour (a rule ignoring the bond label
    would keep them); on C=C-C only the double-bonded pair survives."""
    from synth import GraphBatch
    Q = GraphBatch.from_graphs([([C, C], [(0, 1, 2)])])
    D = GraphBatch.from_graphs([([C, C, C], [(0, 1, 1), (1, 2, 1)])])
    C0 = fr.candidates_bool(Q, D, 1)
    assert C0.all()
    assert not fr.neighbour_support(Q, D, C0).any()
    D2 = GraphBatch.from_graphs([([C, C, C], [(0, 1, 2), (1, 2, 1)])])
    F = fr.neighbour_support(Q, D2, fr.candidates_bool(Q, D2, 1))
    assert np.array_equal(F, np.array([[True, True, False], [True, True, False]]))
    # the support must come from a CANDIDATE neighbour: drop node 1 from C(q1)
    Cb = fr.candidates_bool(Q, D2, 1)
    Cb[1, 1] = False
    F = fr.neighbour_support(Q, D2, Cb)
    # q0 needs a double-bond neighbour in C(q1) = {0, 2}: only node 1 has one (node 0);
    # q1 then needs a double-bond neighbour in C(q0) = {1}: only node 0 has one
    assert np.array_equal(F, np.array([[False, True, False], [True, False, False]]))


def test_wildcard_filter_soundness():
    """Wildcard mode (R22): a '*' query atom's candidates start from every
    atom and it adds to no signature field; the filter (with and without the
    neighbour-support fixed point, '~' bonds matching any label) keeps every
    embedding image of the oracle's wildcard mode at every level."""
    from synth import GraphBatch
    rng = np.random.default_rng(91)
    D = synth.molecules(synth.DATA_SEED_BASE + 5, 0, 25)
    qs = []
    for lab, edges in synth.library(synth.C1_NAMES) + synth.random_subgraph_queries(synth.QUERY_SEED_BASE + 5, 8):
        lab = [0 if rng.random() < 0.35 else x for x in lab]
        edges = [(u, v, 0 if rng.random() < 0.35 else b) for (u, v, b) in edges]
        qs.append((lab, edges))
    Q = GraphBatch.from_graphs(qs)
    imgs = set()
    for q in range(Q.num_graphs):
        for g in range(D.num_graphs):
            for f in oracle.enumerate_pair(Q, D, q, g, oracle.WILDCARD).tolist():
                imgs.update((int(Q.graph_offsets[q]) + i, int(D.graph_offsets[g]) + v) for i, v in enumerate(f))
    assert len(imgs) > 50
    for L in (1, 2, 4):
        Cb = fr.candidates_bool(Q, D, L, wildcard=True)
        F = fr.neighbour_support(Q, D, Cb, wildcard=True)
        for (vq, vd) in imgs:
            assert Cb[vq, vd] and F[vq, vd], (L, vq, vd)
