"""Pins for the CPU oracle (oracle/) against things other than itself:
the paper's worked example, closed forms, brute force, networkx (an
independent VF2) and invariants.  SURVEY.md 8(c) pins P1-P6."""
import itertools
import math
import os

import numpy as np
import pytest

import oracle
import synth
from oracle.brute import brute_count
from synth import GraphBatch

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")

C, N, O = 6, 7, 8


def read_golden_arrays(name):
    out = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, *vals = line.split()
            out[k] = [int(v) for v in vals]
    return out


def count(qgraphs, dgraphs, mode=oracle.FIND_ALL):
    return oracle.count_dense(GraphBatch.from_graphs(qgraphs), GraphBatch.from_graphs(dgraphs), mode)


def ring(n, lab=C, bond=1):
    return [lab] * n, [(i, (i + 1) % n, bond) for i in range(n)]


def path(n, lab=C, bond=1):
    return [lab] * n, [(i, i + 1, bond) for i in range(n - 1)]


def star(d, lab=C, bond=1):
    return [lab] * (d + 1), [(0, i, bond) for i in range(1, d + 1)]


def complete(n, lab=C, bond=1):
    return [lab] * n, [(i, j, bond) for i in range(n) for j in range(i + 1, n)]


# ---------------------------------------------------------------- P1 / P2
def test_fig3_csrgo_exact():
    g = read_golden_arrays("fig3_csrgo.txt")
    B = synth.fig3_batch()
    assert B.graph_offsets.tolist() == g["graph_offsets"]
    assert B.row_offsets.tolist() == g["row_offsets"]
    assert B.col_indices.tolist() == g["col_indices"]


def test_fig3_closed_form_counts():
    gold = read_golden_arrays("fig3_counts.txt")
    queries = {"edge": path(2), "path3": path(3), "cycle5": ring(5), "claw": star(3)}
    D = synth.fig3_batch()
    Q = GraphBatch.from_graphs([queries[k] for k in gold])
    res = oracle.count_dense(Q, D)
    for i, k in enumerate(gold):
        assert res[i].tolist() == gold[k], k
    ff = oracle.count_dense(Q, D, oracle.FIND_FIRST)
    assert ff.tolist() == (res > 0).astype(np.uint64).tolist()


# ---------------------------------------------------------------- P3
def naphthalene():
    labels = [C] * 10
    edges = [(i, (i + 1) % 6, 4) for i in range(6)]  # ring A: 0..5
    edges += [(5, 6, 4), (6, 7, 4), (7, 8, 4), (8, 9, 4), (9, 0, 4)]  # ring B shares bond 0-5
    return labels, edges


def test_closed_forms_rings():
    benzene = ring(6, C, 4)
    assert count([benzene], [benzene])[0, 0] == 12            # north_star: 12 = |Aut(C6)|
    assert count([benzene], [naphthalene()])[0, 0] == 24      # two rings x 12
    assert count([ring(6, C, 1)], [benzene])[0, 0] == 0        # bond label mismatch
    assert count([path(3, C, 4)], [benzene])[0, 0] == 12       # P3 in C6: 6 centres x 2
    assert count([path(3)], [ring(3)])[0, 0] == 6              # mono, not induced (R1)
    for n in range(3, 10):
        assert count([ring(n)], [ring(n)])[0, 0] == 2 * n      # C_n in C_n


def test_closed_forms_single_bond_and_stars():
    rng = np.random.default_rng(1)
    for _ in range(20):
        n = int(rng.integers(2, 12))
        lab, edges = synth.random_labelled_graph(rng, n, 0.4, labels=(C,), bonds=(1,))
        assert count([path(2)], [(lab, edges)])[0, 0] == 2 * len(edges)  # X-X in G = 2|E|
    for d in range(0, 7):
        expect = d * (d - 1) * (d - 2) if d >= 3 else 0
        assert count([star(3)], [star(d)])[0, 0] == expect     # K1,3 at degree-d centre
    for n in range(1, 7):
        assert count([complete(n)], [complete(n)])[0, 0] == math.factorial(n)  # K_n in K_n


def test_degenerate_cases():
    assert count([path(5)], [path(4)])[0, 0] == 0              # query larger than data
    lab = [C, N, C, O, C]
    g = (lab, [(0, 1, 1), (1, 2, 1), (2, 3, 2), (3, 4, 1)])
    assert count([([C], [])], [g])[0, 0] == 3                  # single node = #label matches
    assert count([([N], [])], [g])[0, 0] == 1
    assert count([([7], [])], [([], [])])[0, 0] == 0           # empty data graph
    # disconnected query: two isolated C = ordered pairs of distinct C atoms
    assert count([([C, C], [])], [g])[0, 0] == 6


# ---------------------------------------------------------------- P4 brute force
def test_oracle_vs_brute_force_random_tiny():
    rng = np.random.default_rng(12345)
    qs, ds = [], []
    for _ in range(120):
        ds.append(synth.random_labelled_graph(rng, int(rng.integers(1, 9)), float(rng.uniform(0.2, 0.8)),
                                              labels=(C, N), bonds=(1, 2)))
    for _ in range(100):
        qs.append(synth.random_labelled_graph(rng, int(rng.integers(1, 6)), float(rng.uniform(0.3, 1.0)),
                                              labels=(C, N), bonds=(1, 2)))
    res = count(qs, ds)
    ff = count(qs, ds, oracle.FIND_FIRST)
    n_pos = 0
    for i, q in enumerate(qs):
        for j, d in enumerate(ds):
            b = brute_count(q, d)
            assert res[i, j] == b, (i, j)
            assert ff[i, j] == (1 if b else 0)
            n_pos += b > 0
    assert n_pos > 100  # the sample exercises matching pairs


# ---------------------------------------------------------------- P5 networkx
def _nx(g):
    import networkx as nx
    lab, edges = g
    G = nx.Graph()
    for i, l in enumerate(lab):
        G.add_node(i, l=l)
    for (u, v, b) in edges:
        G.add_edge(u, v, b=b)
    return G


def test_oracle_vs_networkx_molecules():
    from networkx.algorithms import isomorphism as iso
    D = synth.molecules(synth.DATA_SEED_BASE + 99, 0, 40)
    qs = synth.library() + synth.random_subgraph_queries(7, 10)
    Q = GraphBatch.from_graphs(qs)
    res = oracle.count_dense(Q, D)
    nm = iso.categorical_node_match("l", None)
    em = iso.categorical_edge_match("b", None)
    total = 0
    for g in range(D.num_graphs):
        G = _nx(D.graph(g))
        for qi, q in enumerate(qs):
            GM = iso.GraphMatcher(G, _nx(q), node_match=nm, edge_match=em)
            c = sum(1 for _ in GM.subgraph_monomorphisms_iter())
            assert res[qi, g] == c, (qi, g)
            total += c
    assert total > 0


# ---------------------------------------------------------------- P6 invariants
def test_invariants_automorphism_divisibility_and_first():
    D = synth.molecules(synth.DATA_SEED_BASE + 98, 0, 60)
    qs = synth.library()
    Q = GraphBatch.from_graphs(qs)
    res = oracle.count_dense(Q, D)
    ff = oracle.count_dense(Q, D, oracle.FIND_FIRST)
    assert np.array_equal(ff, (res > 0).astype(np.uint64))
    aut = oracle.count_dense(Q, Q).diagonal()
    assert np.all(aut >= 1)
    assert np.all(res % aut[:, None] == 0)


def test_invariants_additivity_and_relabel():
    D = synth.molecules(synth.DATA_SEED_BASE + 97, 0, 50)
    Q = synth.config_queries(1)
    full = oracle.count_dense(Q, D)
    parts = [oracle.count_dense(Q, D.slice(a, b)) for a, b in [(0, 17), (17, 30), (30, 50)]]
    assert np.array_equal(np.concatenate(parts, axis=1), full)
    # disjoint union of two molecules counts = sum only for connected queries
    rng = np.random.default_rng(3)
    for g in range(10):
        lab, edges = D.graph(g)
        perm = rng.permutation(len(lab))
        inv = np.argsort(perm)
        lab2 = [lab[int(inv[i])] for i in range(len(lab))]
        edges2 = [(int(perm[u]), int(perm[v]), b) for (u, v, b) in edges]
        r2 = oracle.count_dense(Q, GraphBatch.from_graphs([(lab2, edges2)]))
        assert np.array_equal(r2[:, 0], full[:, g])


def test_pair_list_matches_dense():
    D = synth.molecules(synth.DATA_SEED_BASE + 96, 0, 30)
    Q = synth.config_queries(1)
    full = oracle.count_dense(Q, D)
    pq, pg = np.meshgrid(np.arange(Q.num_graphs), np.arange(D.num_graphs), indexing="ij")
    out = oracle.count_pairs(Q, D, pq.ravel(), pg.ravel())
    assert np.array_equal(out.reshape(full.shape), full)
    out1 = oracle.count_pairs(Q, D, pq.ravel(), pg.ravel(), nthreads=1)
    assert np.array_equal(out1, out)


# ---------------------------------------------------------------- N4 induced mode (R21)
IND = oracle.INDUCED


def test_induced_closed_forms():
    assert count([path(3)], [ring(3)], IND)[0, 0] == 0         # P3 needs a non-edge; K3 has none
    assert count([path(3)], [ring(3)])[0, 0] == 6              # vs monomorphism (R1)
    assert count([path(3, C, 4)], [ring(6, C, 4)], IND)[0, 0] == 12   # C6 has no chords
    assert count([ring(4)], [complete(4)], IND)[0, 0] == 0     # K4 has both diagonals
    assert count([ring(4)], [complete(4)])[0, 0] == 24
    for n in range(1, 6):
        assert count([complete(n)], [complete(n + 1)], IND)[0, 0] == math.factorial(n + 1)  # cliques induce
    # two isolated C in P4 (C-C-C-C): ordered non-adjacent pairs = 2 * (C(4,2) - 3)
    assert count([([C, C], [])], [path(4)], IND)[0, 0] == 6
    assert count([([C, C], [])], [path(4)], IND | oracle.FIND_FIRST)[0, 0] == 1
    # a non-edge with a bond of another label still counts as an edge (any bond)
    q = ([C, C, C], [(0, 1, 1), (1, 2, 1)])
    d = ([C, C, C], [(0, 1, 1), (1, 2, 1), (0, 2, 2)])
    assert count([q], [d])[0, 0] == 2 and count([q], [d], IND)[0, 0] == 0


def test_induced_vs_brute_force_and_subset():
    rng = np.random.default_rng(777)
    qs = [synth.random_labelled_graph(rng, int(rng.integers(1, 6)), float(rng.uniform(0.3, 1.0)),
                                      labels=(C, N), bonds=(1, 2)) for _ in range(60)]
    ds = [synth.random_labelled_graph(rng, int(rng.integers(1, 9)), float(rng.uniform(0.2, 0.8)),
                                      labels=(C, N), bonds=(1, 2)) for _ in range(80)]
    ind = count(qs, ds, IND)
    ff = count(qs, ds, IND | oracle.FIND_FIRST)
    mono = count(qs, ds)
    n_pos = n_strict = 0
    for i, q in enumerate(qs):
        for j, d in enumerate(ds):
            b = brute_count(q, d, induced=True)
            assert ind[i, j] == b, (i, j)
            assert ff[i, j] == (1 if b else 0)
            assert ind[i, j] <= mono[i, j]
            n_pos += b > 0
            n_strict += ind[i, j] < mono[i, j]
    assert n_pos > 40 and n_strict > 40  # both matching and induced-pruned pairs are exercised


def test_induced_vs_networkx_molecules():
    pytest.importorskip("networkx")
    from networkx.algorithms import isomorphism as iso
    D = synth.molecules(synth.DATA_SEED_BASE + 98, 0, 30)
    qs = synth.library() + synth.random_subgraph_queries(8, 10)
    res = oracle.count_dense(GraphBatch.from_graphs(qs), D, IND)
    nm = iso.categorical_node_match("l", None)
    em = iso.categorical_edge_match("b", None)
    total = 0
    for g in range(D.num_graphs):
        G = _nx(D.graph(g))
        for qi, q in enumerate(qs):
            GM = iso.GraphMatcher(G, _nx(q), node_match=nm, edge_match=em)
            c = sum(1 for _ in GM.subgraph_isomorphisms_iter())  # induced (node-induced subgraph isomorphism)
            assert res[qi, g] == c, (qi, g)
            total += c
    assert total > 0


# ---------------------------------------------------------------- N1 enumerate mode
def test_enumerate_vs_brute_force_random_tiny():
    """Enumerate mode (NLSM P:446-453): the set of mappings
    equals brute-force enumeration of injective tuples (Def. 2.1 conditions
    (1)-(2), bond labels), monomorphic and induced, on random tiny graphs."""
    from oracle.brute import brute_embeddings
    rng = np.random.default_rng(777)
    n_emb = 0
    for it in range(400):
        d = synth.random_labelled_graph(rng, int(rng.integers(1, 8)), float(rng.uniform(0.2, 0.8)),
                                        labels=(C, N), bonds=(1, 2))
        q = synth.random_labelled_graph(rng, int(rng.integers(1, 5)), float(rng.uniform(0.3, 1.0)),
                                        labels=(C, N), bonds=(1, 2))
        Q, D = GraphBatch.from_graphs([q]), GraphBatch.from_graphs([d])
        for induced in (False, True):
            got = oracle.enumerate_pair(Q, D, 0, 0, oracle.INDUCED if induced else oracle.FIND_ALL)
            ref = sorted(brute_embeddings(q, d, induced))
            assert sorted(map(tuple, got.tolist())) == ref, (it, induced)
            assert len(got) == len(set(map(tuple, got.tolist())))  # no mapping twice
            n_emb += len(ref)
    assert n_emb > 300


def test_enumerate_closed_forms():
    """Benzene: the 12 embeddings of the aromatic 6-ring are the 12
    automorphisms of C6 and form ONE node set (NLSM's X); naphthalene: 24
    embeddings, 2 node sets (the two rings); a single bond C-C in propane:
    2|E| = 4 mappings, 2 node sets."""
    benzene = ring(6, C, 4)
    got = oracle.enumerate_pair(GraphBatch.from_graphs([benzene]), GraphBatch.from_graphs([benzene]), 0, 0)
    assert len(got) == 12 and oracle.node_sets(got) == [(0, 1, 2, 3, 4, 5)]
    # every embedding is a rotation or reflection of the ring
    for f in got.tolist():
        step = (f[1] - f[0]) % 6
        assert step in (1, 5) and all((f[i + 1] - f[i]) % 6 == step for i in range(5))
    naph = naphthalene()
    got = oracle.enumerate_pair(GraphBatch.from_graphs([benzene]), GraphBatch.from_graphs([naph]), 0, 0)
    assert len(got) == 24 and len(oracle.node_sets(got)) == 2
    got = oracle.enumerate_pair(GraphBatch.from_graphs([path(2)]), GraphBatch.from_graphs([path(3)]), 0, 0)
    assert sorted(map(tuple, got.tolist())) == [(0, 1), (1, 0), (1, 2), (2, 1)]
    assert oracle.node_sets(got) == [(0, 1), (1, 2)]
    # consistent with the counting mode on a molecule sample
    Q, D = synth.config_queries(1), synth.config_data(1, count=20)
    dense = oracle.count_dense(Q, D)
    for q in range(Q.num_graphs):
        for g in range(D.num_graphs):
            assert len(oracle.enumerate_pair(Q, D, q, g)) == dense[q, g]


# ---------------------------------------------------------------- N3 wildcard mode
WC = oracle.WILDCARD
ANY = 0  # query atom label 0 = SMARTS '*', query bond label 0 = SMARTS '~' (R22)


def test_wildcard_closed_forms():
    """'*' matches every atom; '*~*' every bond twice (2|E|); 'C~C' any C-C
    bond, 'C-C' only single ones; a 6-ring of '*' atoms and '~' bonds has the
    12 automorphic embeddings in benzene AND in cyclohexane, while the
    aromatic-bond ring has none in cyclohexane (R22)."""
    benzene, cyclohexane = ring(6, C, 4), ring(6, C, 1)
    mol = ([C, C, C, O], [(0, 1, 2), (1, 2, 1), (2, 3, 1)])  # C=C-C-O
    assert count([([ANY], [])], [benzene, mol], WC).tolist() == [[6, 4]]
    assert count([([ANY, ANY], [(0, 1, ANY)])], [benzene, mol], WC).tolist() == [[12, 6]]
    assert count([([C, C], [(0, 1, ANY)])], [mol], WC).tolist() == [[4]]
    assert count([([C, C], [(0, 1, 1)])], [mol], WC).tolist() == [[2]]
    assert count([([C, ANY], [(0, 1, 1)])], [mol], WC).tolist() == [[3]]  # C1-C2 both ways, C2-O3
    wring = ([ANY] * 6, [(i, (i + 1) % 6, ANY) for i in range(6)])
    assert count([wring, benzene], [benzene, cyclohexane], WC).tolist() == [[12, 12], [12, 0]]
    # without the wildcard bit, label 0 / bond 0 are literal values (nothing in these molecules)
    assert count([([ANY], [])], [benzene], oracle.FIND_ALL).tolist() == [[0]]


def test_wildcard_vs_brute_force_random_tiny():
    """Wildcard mode vs brute force (conditions (1') and (2')), monomorphic and
    induced, Find All and Find First, on random tiny graphs whose queries have
    wildcard atoms and bonds; with no label-0 atom or bond the mode equals the
    exact one."""
    from oracle.brute import brute_count
    rng = np.random.default_rng(4242)
    qs, ds = [], []
    for _ in range(80):
        ds.append(synth.random_labelled_graph(rng, int(rng.integers(1, 8)), float(rng.uniform(0.2, 0.8)),
                                              labels=(C, N, O), bonds=(1, 2)))
    for _ in range(60):
        lab, edges = synth.random_labelled_graph(rng, int(rng.integers(1, 5)), float(rng.uniform(0.3, 1.0)),
                                                 labels=(C, N), bonds=(1, 2))
        lab = [ANY if rng.random() < 0.3 else x for x in lab]
        edges = [(u, v, ANY if rng.random() < 0.3 else b) for (u, v, b) in edges]
        qs.append((lab, edges))
    n_pos = 0
    for induced in (False, True):
        im = oracle.INDUCED if induced else 0
        res = count(qs, ds, WC | im)
        ff = count(qs, ds, WC | im | oracle.FIND_FIRST)
        for i, q in enumerate(qs):
            for j, d in enumerate(ds):
                b = brute_count(q, d, induced=induced, wildcard=True)
                assert res[i, j] == b, (i, j, induced)
                assert ff[i, j] == (1 if b else 0)
                n_pos += b > 0
    assert n_pos > 200
    exact = [q for q in qs if ANY not in q[0] and all(b != ANY for (_, _, b) in q[1])]
    assert np.array_equal(count(exact, ds, WC), count(exact, ds))
