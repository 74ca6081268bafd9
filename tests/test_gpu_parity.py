"""GPU parity: the CUDA path through the C ABI vs the CPU oracle (bit-exact).

Every count and flag is an exact integer: bitmaps,
signatures, GMCR pairs, Find All counts and Find First flags must be equal
element by element.  Sizes span many filter tiles (1024 data nodes each),
many join chunks and ragged tails."""
import os

import numpy as np
import pytest

import oracle
import synth
from oracle import filter_ref as fr
from synth import GraphBatch

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


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
    yield c
    c.close()


def run(ctx, Q, D, levels, mode):
    ctx.load_batch(Q, D)
    ctx.filter(levels)
    total = ctx.join(mode)
    return total, ctx.dense_results()


def ring(n, lab=6, bond=1):
    return [lab] * n, [(i, (i + 1) % n, bond) for i in range(n)]


def path(n, lab=6, bond=1):
    return [lab] * n, [(i, i + 1, bond) for i in range(n - 1)]


def star(d, lab=6, bond=1):
    return [lab] * (d + 1), [(0, i, bond) for i in range(1, d + 1)]


def test_fig3_closed_forms(ctx, sigmo):
    D = synth.fig3_batch()
    Q = GraphBatch.from_graphs([path(2), path(3), ring(5), star(3)])
    expect = np.array([[10, 6], [10, 6], [10, 0], [0, 6]], np.uint64)
    for L in (1, 2, 3, 4, 7):
        tot, dense = run(ctx, Q, D, L, sigmo.SIGMO_FIND_ALL)
        assert np.array_equal(dense, expect), L
        assert tot == int(expect.sum())
        ctx.join(sigmo.SIGMO_FIND_FIRST)
        assert np.array_equal(ctx.dense_results(), (expect > 0).astype(np.uint64))


def test_fig3_packed_readback(ctx):
    """P1: the library's own CSR-GO packing of the Fig. 3 worked example
    (P:763-790), read back from the device, equals the arrays printed in the
    paper (tests/golden/fig3_csrgo.txt)."""
    from test_oracle import read_golden_arrays
    g = read_golden_arrays("fig3_csrgo.txt")
    D = synth.fig3_batch()
    ctx.load_batch(GraphBatch.from_graphs([path(2)]), D)
    go, ro, co, nl, el = ctx.packed_batch(1)
    assert go.tolist() == g["graph_offsets"]
    assert ro.tolist() == g["row_offsets"]
    assert co.tolist() == g["col_indices"]
    assert nl.tolist() == [6] * 9 and el.tolist() == [1] * 16
    go, ro, co, nl, el = ctx.packed_batch(0)
    assert go.tolist() == [0, 2] and ro.tolist() == [0, 1, 2] and co.tolist() == [1, 0]


def test_signatures_match_reference(ctx):
    Q = synth.config_queries(4)  # includes 20-30-atom ring systems
    D = synth.config_data(1)
    ctx.load_batch(Q, D)
    for r in (1, 2, 3, 5):
        assert np.array_equal(ctx.signatures(0, r), fr.signatures(Q, r)), ("query", r)
        assert np.array_equal(ctx.signatures(1, r), fr.signatures(D, r)), ("data", r)


def test_signature_saturation(ctx):
    # a 100-atom N chain: the 6-bit N field saturates at 63 (R8)
    D = GraphBatch.from_graphs([path(100, 7), ring(6, 6, 4)])
    Q = GraphBatch.from_graphs([path(3, 7)])
    ctx.load_batch(Q, D)
    for r in (1, 10, 40, 70):
        assert np.array_equal(ctx.signatures(1, r), fr.signatures(D, r)), r


@pytest.mark.parametrize("levels", [1, 2, 3, 4, 5])
def test_c1_bitmap_and_counts(ctx, sigmo, levels):
    Q, D = synth.config_queries(1), synth.config_data(1)
    ctx.load_batch(Q, D)
    ctx.filter(levels)
    assert np.array_equal(ctx.candidates(), fr.candidates(Q, D, levels))
    Cb = fr.candidates_bool(Q, D, levels)
    G = fr.gmcr(Q, D, Cb)
    assert ctx.num_pairs() == int(G.sum())
    tot = ctx.join(sigmo.SIGMO_FIND_ALL)
    ref = oracle.count_dense(Q, D)
    assert np.array_equal(ctx.dense_results(), ref)
    assert tot == int(ref.sum())
    di, qi, r = ctx.pair_results()
    assert np.array_equal(G[qi, di], np.ones(len(di), bool))  # exactly the GMCR pairs
    assert np.all(np.diff(di) >= 0)
    assert np.array_equal(ctx.query_totals(), ref.sum(axis=1).astype(np.uint64))
    ctx.join(sigmo.SIGMO_FIND_FIRST)
    assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D, oracle.FIND_FIRST))


def test_levels_monotone_and_sound(ctx):
    Q, D = synth.config_queries(2), synth.config_data(2, count=300)
    ctx.load_batch(Q, D)
    prev = None
    for L in range(1, 8):
        ctx.filter(L)
        bm = ctx.candidates()
        if prev is not None:
            assert not np.any(bm & ~prev)
        prev = bm
    ctx.filter(6)
    assert np.array_equal(ctx.candidates(), fr.candidates(Q, D, 6))


def test_edge_cases_batch(ctx, sigmo):
    """empty data graphs, single-atom graphs, disconnected graphs, single-node
    and disconnected queries, graphs > 64 atoms (multi-word masks)."""
    rng = np.random.default_rng(11)
    mols = synth.molecules(synth.DATA_SEED_BASE + 77, 0, 120, mode=2)
    graphs = mols.graphs()
    graphs.insert(0, ([], []))
    graphs.insert(5, ([6], []))
    graphs.insert(9, ([], []))
    graphs.append(([6, 6, 8, 6], [(0, 1, 1), (2, 3, 1)]))
    graphs.append(([], []))
    big = ([6] * 100, [(i, i + 1, 1) for i in range(99)] + [(0, 99, 1)])
    graphs.insert(50, big)
    D = GraphBatch.from_graphs(graphs)
    assert D.sizes().max() > 64
    qs = synth.library(synth.C1_NAMES) + [([6], []), ([8], []), ([6, 8], []), ([6, 6, 6], [(0, 1, 1)]),
                                          path(7), ring(6, 6, 4)]
    Q = GraphBatch.from_graphs(qs)
    for L in (1, 3, 5):
        tot, dense = run(ctx, Q, D, L, sigmo.SIGMO_FIND_ALL)
        ref = oracle.count_dense(Q, D)
        assert np.array_equal(dense, ref), L
        assert np.array_equal(ctx.candidates(), fr.candidates(Q, D, L))
        ctx.join(sigmo.SIGMO_FIND_FIRST)
        assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D, oracle.FIND_FIRST))


def test_large_ring_system_queries(ctx, sigmo):
    Q = synth.config_queries(4)
    D = synth.config_data(4, count=400)
    ctx.load_batch(Q, D)
    ctx.filter(4)
    ctx.join(sigmo.SIGMO_FIND_ALL)
    assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D))
    ctx.join(sigmo.SIGMO_FIND_FIRST)
    assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D, oracle.FIND_FIRST))


def test_random_tiny_graphs_vs_oracle(ctx, sigmo):
    rng = np.random.default_rng(2024)
    ds = [synth.random_labelled_graph(rng, int(rng.integers(0, 12)), float(rng.uniform(0.1, 0.7)),
                                      labels=(6, 7), bonds=(1, 2)) for _ in range(400)]
    qs = [synth.random_labelled_graph(rng, int(rng.integers(1, 6)), float(rng.uniform(0.3, 1.0)),
                                      labels=(6, 7), bonds=(1, 2)) for _ in range(40)]
    Q, D = GraphBatch.from_graphs(qs), GraphBatch.from_graphs(ds)
    for L in (1, 2, 4):
        _, dense = run(ctx, Q, D, L, sigmo.SIGMO_FIND_ALL)
        assert np.array_equal(dense, oracle.count_dense(Q, D)), L


def test_empty_data_batch_and_state_errors(ctx, sigmo):
    Q = synth.config_queries(1)
    with pytest.raises(sigmo.SigmoError) as e:
        ctx.filter(2)
    assert e.value.status == -4
    ctx.load_batch(Q, GraphBatch.empty())
    with pytest.raises(sigmo.SigmoError) as e:
        ctx.join(sigmo.SIGMO_FIND_ALL)
    assert e.value.status == -4
    ctx.filter(3)
    assert ctx.num_pairs() == 0
    assert ctx.join(sigmo.SIGMO_FIND_ALL) == 0
    assert ctx.query_totals().sum() == 0
    with pytest.raises(sigmo.SigmoError) as e:
        ctx.filter(17)
    assert e.value.status == -1


def test_c2_full_size_parity(ctx, sigmo):
    """configs[1] at full size in the bench's launch configuration: every one
    of the 5M pairs bit-exact against the oracle (Find All and Find First)."""
    Q, D = synth.config_queries(2), synth.config_data(2)
    ctx.load_batch(Q, D)
    ctx.filter(4)
    tot = ctx.join(sigmo.SIGMO_FIND_ALL)
    got = ctx.dense_results()
    ref = oracle.count_dense(Q, D)
    assert tot == int(ref.sum())
    assert np.array_equal(got, ref)
    ctx.join(sigmo.SIGMO_FIND_FIRST)
    assert np.array_equal(ctx.dense_results(), (ref > 0).astype(np.uint64))
    # bitmap on sampled molecules vs the filter reference
    rng = np.random.default_rng(5)
    gs = sorted(int(g) for g in rng.choice(D.num_graphs, 60, replace=False))
    bm = ctx.candidates()
    Cb = fr.candidates_bool(Q, D, 4, data_graphs=gs)
    ref_bits = fr.to_bitmap(Cb)
    for g in gs:
        lo, hi = int(D.graph_offsets[g]), int(D.graph_offsets[g + 1])
        for v in range(lo, hi):
            w, b = v >> 5, v & 31
            assert np.array_equal((bm[:, w] >> b) & 1, (ref_bits[:, w] >> b) & 1), (g, v)


@pytest.mark.parametrize("env", [{"SIGMO_FILTER_JIT": "0"}, {"SIGMO_FILTER_JIT": "0", "SIGMO_FILTER_TABLES_GLOBAL": "1"},
                                 {"SIGMO_FILTER_TABLES_GLOBAL": "1"}, {}],
                         ids=["generic", "generic-global", "jit-global", "jit"])
def test_lane_filter_variants(sigmo, monkeypatch, env):
    """Every build of the lane-path filter (the table-driven generic kernel and
    the NVRTC-specialised one; query tables in shared or global memory) gives
    the same bitmap, GMCR pairs and counts as the references."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    Q, D = synth.config_queries(2), synth.config_data(2, count=3000)
    ref = oracle.count_dense(Q, D)
    with sigmo.Context(0) as c:
        c.load_batch(Q, D)
        for L in (1, 3, 4):
            c.filter(L)
            c.set_timing(True)
            c.join(sigmo.SIGMO_FIND_ALL)
            assert np.array_equal(c.dense_results(), ref), L
            assert c.timings()["filter_jit"] == (0 if env.get("SIGMO_FILTER_JIT") == "0" else 1), L
        Cb = fr.candidates_bool(Q, D, 4, data_graphs=list(range(0, 3000, 97)))
        G = fr.gmcr(Q, D, fr.candidates_bool(Q, D, 4))
        assert c.num_pairs() == int(G.sum())
        ref_bits = fr.to_bitmap(Cb)
        bm = c.candidates()
        for g in range(0, 3000, 97):
            lo, hi = int(D.graph_offsets[g]), int(D.graph_offsets[g + 1])
            for v in range(lo, hi):
                w, b = v >> 5, v & 31
                assert np.array_equal((bm[:, w] >> b) & 1, (ref_bits[:, w] >> b) & 1), (g, v)


def test_join_stack_spill_path(sigmo, monkeypatch):
    """Force the smallest shared-memory DFS stack so that the global spill /
    restore path runs (deep 20-30-atom ring-system queries), results unchanged."""
    monkeypatch.setenv("SIGMO_JOIN_SCS", "128")
    Q = synth.config_queries(4)
    D = synth.config_data(4, count=150)
    with sigmo.Context(0) as c:
        c.load_batch(Q, D)
        c.filter(2)
        c.set_timing(True)
        c.join(sigmo.SIGMO_FIND_ALL)
        assert np.array_equal(c.dense_results(), oracle.count_dense(Q, D))
        c.join(sigmo.SIGMO_FIND_FIRST)
        assert np.array_equal(c.dense_results(), oracle.count_dense(Q, D, oracle.FIND_FIRST))


def test_shard_additivity_gpu(sigmo):
    """Molecule shards (balanced by atoms) run one after another on the GPU:
    per-query totals add up to the unsharded run and to the oracle (P6)."""
    from paper_conf_sc_carocfc25_b200 import sharded
    Q, D = synth.config_queries(2), synth.config_data(2, count=3000)
    ref = oracle.count_dense(Q, D).sum(axis=1).astype(np.uint64)
    with sigmo.Context(0) as c:
        c.load_batch(Q, D)
        c.filter(3)
        c.join(sigmo.SIGMO_FIND_ALL)
        assert np.array_equal(c.query_totals(), ref)
        acc = np.zeros(Q.num_graphs, np.uint64)
        for r in range(3):
            g0, g1 = sharded.shard_range(D.graph_offsets, r, 3)
            c.load_batch(Q, D.slice(g0, g1))
            c.filter(3)
            c.join(sigmo.SIGMO_FIND_ALL)
            acc += c.query_totals()
        assert np.array_equal(acc, ref)


@pytest.mark.parametrize("levels", [1, 2, 4])
def test_neighbour_support_bitmap_and_counts(ctx, sigmo, levels):
    """SIGMO_FILTER_NEIGHBOR_SUPPORT: bitmap = the greatest fixed point of the
    CPU reference, GMCR pairs = reference GMCR of that bitmap, counts unchanged."""
    Q, D = synth.config_queries(1), synth.config_data(1)
    ctx.load_batch(Q, D)
    ctx.filter(levels, neighbor_support=True)
    Cb = fr.neighbour_support(Q, D, fr.candidates_bool(Q, D, levels))
    assert np.array_equal(ctx.candidates(), fr.to_bitmap(Cb))
    assert ctx.num_pairs() == int(fr.gmcr(Q, D, Cb).sum())
    ctx.join(sigmo.SIGMO_FIND_ALL)
    assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D))
    ctx.join(sigmo.SIGMO_FIND_FIRST)
    assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D, oracle.FIND_FIRST))


def test_neighbour_support_edge_cases(ctx, sigmo):
    mols = synth.molecules(synth.DATA_SEED_BASE + 78, 0, 60, mode=2)
    graphs = mols.graphs()
    graphs.insert(3, ([], []))
    graphs.insert(7, ([6], []))
    graphs.append(([6] * 80, [(i, i + 1, 1) for i in range(79)]))
    D = GraphBatch.from_graphs(graphs)
    qs = synth.library(synth.C1_NAMES) + [([6], []), ([6, 8], []), path(5), ring(6, 6, 4)]
    Q = GraphBatch.from_graphs(qs)
    ctx.load_batch(Q, D)
    ctx.filter(3, neighbor_support=True)
    Cb = fr.neighbour_support(Q, D, fr.candidates_bool(Q, D, 3))
    assert np.array_equal(ctx.candidates(), fr.to_bitmap(Cb))
    ctx.join(sigmo.SIGMO_FIND_ALL)
    assert np.array_equal(ctx.dense_results(), oracle.count_dense(Q, D))


def test_cost_model_from_device_gmcr(ctx, sigmo):
    """N2 cost model (sharded.molecule_costs) fed by the device GMCR pair list
    equals the model fed by the reference GMCR; the rebalanced split covers
    the batch and is at least as balanced in modelled cost as the atom split."""
    from paper_conf_sc_carocfc25_b200 import sharded
    Q, D = synth.config_queries(1), synth.config_data(1)
    ctx.load_batch(Q, D)
    ctx.filter(4)
    ctx.join(sigmo.SIGMO_FIND_ALL)
    di, _, _ = ctx.pair_results()
    c = sharded.molecule_costs(D.graph_offsets, di)
    G = fr.gmcr(Q, D, fr.candidates_bool(Q, D, 4))
    assert np.array_equal(c, sharded.molecule_costs(D.graph_offsets, np.nonzero(G)[1]))
    for world in (2, 4, 8):
        b = sharded.cost_bounds(c, world)
        a = sharded.shard_bounds(D.graph_offsets, world)
        cb = max(c[b[r]:b[r + 1]].sum() for r in range(world))
        ca = max(c[a[r]:a[r + 1]].sum() for r in range(world))
        assert b[-1] == D.num_graphs and cb <= ca + c.max()


def test_neighbour_support_lane_path_c2(sigmo):
    """Neighbour support on the lane path (k_support_lane: per-pair refined
    windows, GMCR rebuilt) on a 20k-molecule configs[1] slice incl. > 32-atom
    molecules: GMCR pairs = the reference GMCR of the fixed point on sampled
    molecules, every pair's Find All / Find First result = the oracle's."""
    Q, D = synth.config_queries(2), synth.config_data(2, first=60_000, count=20_000)
    ref = oracle.count_dense(Q, D)
    with sigmo.Context(0) as c:
        c.load_batch(Q, D)
        c.filter(4)
        n_plain = c.num_pairs()
        c.filter(4, neighbor_support=True)
        n_ns = c.num_pairs()
        assert n_ns < n_plain
        c.join(sigmo.SIGMO_FIND_ALL)
        assert np.array_equal(c.dense_results(), ref)
        c.join(sigmo.SIGMO_FIND_FIRST)
        assert np.array_equal(c.dense_results(), (ref > 0).astype(np.uint64))
        di, qi, _ = c.pair_results()
    gs = list(range(0, 20_000, 97))
    for g in gs[:40]:
        Dg = D.slice(g, g + 1)
        F = fr.neighbour_support(Q, Dg, fr.candidates_bool(Q, Dg, 4))
        want = set(np.nonzero(fr.gmcr(Q, Dg, F)[:, 0])[0].tolist())
        assert set(qi[di == g].tolist()) == want, g


def test_lane_join_extra_back_edges(ctx, sigmo):
    """Queries with a plan depth of > 2 back-edges (K4, K5, a fused bicycle)
    run the lane join's instantiation with the extra back-edge loop; the same
    data with queries of <= 2 back-edges per depth runs the lean one
    (JoinParams::extras).  Both against the oracle, Find All and Find First."""
    rng = np.random.default_rng(5)
    ds = [synth.random_labelled_graph(rng, int(rng.integers(4, 30)), float(rng.uniform(0.15, 0.6)),
                                      labels=(6, 6, 7)) for _ in range(300)]
    D = GraphBatch.from_graphs(ds)
    k4 = ([6] * 4, [(i, j, 1) for i in range(4) for j in range(i + 1, 4)])
    k5 = ([6] * 5, [(i, j, 1) for i in range(5) for j in range(i + 1, 5)])
    bicycle = ([6] * 6, [(0, 1, 1), (1, 2, 1), (2, 3, 1), (3, 0, 1), (1, 4, 1), (4, 5, 1), (5, 3, 1), (0, 2, 1)])
    for qs in ([k4, k5, bicycle, path(4)], [path(4), ring(5), ring(4), ([6, 7], [(0, 1, 1)])]):
        Q = GraphBatch.from_graphs(qs)
        for mode, om in ((sigmo.SIGMO_FIND_ALL, oracle.FIND_ALL), (sigmo.SIGMO_FIND_FIRST, oracle.FIND_FIRST)):
            _, dense = run(ctx, Q, D, 2, mode)
            assert np.array_equal(dense, oracle.count_dense(Q, D, om)), (len(qs), mode)


def test_lane_join_step_counting(ctx, sigmo):
    """sigmo_set_timing bit 1: the join counts its DFS steps (the counting
    instantiation); without it the lean one runs and reports 0; both give the
    oracle's counts."""
    Q, D = synth.config_queries(2), synth.config_data(2, count=2000)
    ref = oracle.count_dense(Q, D)
    ctx.load_batch(Q, D)
    ctx.filter(2)
    ctx.set_timing(False, count_steps=True)
    ctx.join(sigmo.SIGMO_FIND_ALL)
    steps = ctx.timings()["dfs_steps"]
    assert np.array_equal(ctx.dense_results(), ref)
    ctx.set_timing(False)
    ctx.join(sigmo.SIGMO_FIND_ALL)
    assert ctx.timings()["dfs_steps"] == 0
    assert np.array_equal(ctx.dense_results(), ref)
    # every step pops one candidate: at least one step per surviving pair with a non-empty root window
    assert steps >= int((ref > 0).sum())


def test_query_program_reuse_across_loads(ctx, sigmo):
    """A load with the same query batch as the previous one reuses the query
    programs and (when the matching order is unchanged) the join's plan
    entries; data batches with other label frequencies (another order), another
    query batch and the way back all match the oracle."""
    Q1 = synth.config_queries(2)
    Q2 = GraphBatch.from_graphs(synth.library(["benzene", "pyridine", "ester", "nitrile"]))
    rng = np.random.default_rng(9)
    D1 = synth.config_data(2, count=800)
    D2 = synth.config_data(2, first=5000, count=800)
    # label-skewed batch: many nitrogens (the planner's rarest-label root changes)
    ds = [synth.random_labelled_graph(rng, int(rng.integers(3, 20)), 0.3, labels=(7, 7, 7, 6, 8)) for _ in range(300)]
    D3 = GraphBatch.from_graphs(ds)
    for Q, D in ((Q1, D1), (Q1, D2), (Q1, D3), (Q1, D1), (Q2, D1), (Q1, D2)):
        for L in (2, 4):
            for mode, om in ((sigmo.SIGMO_FIND_ALL, oracle.FIND_ALL), (sigmo.SIGMO_FIND_FIRST, oracle.FIND_FIRST)):
                _, dense = run(ctx, Q, D, L, mode)
                assert np.array_equal(dense, oracle.count_dense(Q, D, om)), (Q.num_graphs, L, mode)
