"""Element-wise GPU parity at the BASELINE.json sizes, in the launch
configurations bench.py times (bit-exact vs the oracle on
every pair of every config; Def. 2.1, NLSM P:446-453).

Every (query, molecule) pair is compared: the oracle (plain backtracking, no
filter) computes dense chunks of 100k molecules and the device's sparse GMCR
pair list is scattered into the same dense chunk -- so pairs pruned by the
filter are checked to be 0 as well.  Also: the join is independent of its
work schedule (refill batch, CTAs per SM)."""
import numpy as np
import pytest

import oracle
import synth
from paper_conf_sc_carocfc25_b200 import stream

pytestmark = pytest.mark.gpu

CHUNK = 100_000
IND = oracle.INDUCED  # induced-subgraph embeddings (R21)


@pytest.fixture(scope="module")
def sigmo():
    import torch
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_sc_carocfc25_b200 as s
    torch.cuda.set_device(0)
    return s


def check_every_pair(Q, D, di, qi, r, mode, qidx=None):
    """Scatter the device pair list (data graph di, query qi -> result r,
    sorted by di) into dense chunks and compare each with the oracle.  qidx:
    the queries of a routed group (pair query ids index into it)."""
    nq = Q.num_graphs
    rows = np.arange(nq) if qidx is None else np.asarray(qidx)
    QQ = Q if qidx is None else synth.GraphBatch.from_graphs([Q.graphs()[int(i)] for i in rows])
    for g0 in range(0, D.num_graphs, CHUNK):
        g1 = min(g0 + CHUNK, D.num_graphs)
        lo, hi = np.searchsorted(di, g0), np.searchsorted(di, g1)
        dense = np.zeros((len(rows), g1 - g0), np.uint64)
        dense[qi[lo:hi], di[lo:hi] - g0] = r[lo:hi]
        ref = oracle.count_dense(QQ, D.slice(g0, g1), mode)
        bad = np.argwhere(dense != ref)
        assert bad.size == 0, (g0, bad[:5].tolist(), dense[tuple(bad[0])], ref[tuple(bad[0])])


@pytest.mark.parametrize("induced", [False, True], ids=["mono", "induced"])
def test_c3_every_pair(sigmo, induced):
    """configs[2] (100 queries x 1M molecules, L=4, the default bench
    workload; with --induced the induced one): every one of the 1e8 pairs,
    Find All counts and Find First flags."""
    Q, D = synth.config_queries(3), synth.config_data(3)
    im = IND if induced else 0
    with sigmo.Context(0) as ctx:
        ctx.set_induced(induced)
        ctx.load_batch(Q, D)
        ctx.filter(4)
        tot = ctx.join(sigmo.SIGMO_FIND_ALL)
        di, qi, r = ctx.pair_results()
        assert tot == int(r.sum())
        check_every_pair(Q, D, di, qi, r, oracle.FIND_ALL | im)
        ctx.join(sigmo.SIGMO_FIND_FIRST)
        di, qi, r = ctx.pair_results()
        check_every_pair(Q, D, di, qi, r, oracle.FIND_FIRST | im)


def routed_pairs(sigmo, Q, D, mode, levels=4):
    """Run Q x D as StreamRunner does (queries <= 11 nodes on the lane path,
    larger ones on the general path, one context each); yield (group query
    indices, pair list)."""
    for idx in stream.split_queries(Q):
        sub = synth.GraphBatch.from_graphs([Q.graphs()[int(i)] for i in idx])
        with sigmo.Context(0) as ctx:
            ctx.load_batch(sub, D)
            ctx.filter(levels)
            ctx.join(mode)
            yield idx, ctx.pair_results()


def test_c4_every_pair_all_shares(sigmo):
    """configs[3] (500 queries incl. 30 ring systems of 20-30 atoms x 1M
    molecules, Find First) as the bench runs it at 8 GPUs: 8 shares of 125k
    molecules, queries routed by size; every pair of every share."""
    Q = synth.config_queries(4)
    for s in range(8):
        D = synth.config_data(4, first=125_000 * s, count=125_000)
        for idx, (di, qi, r) in routed_pairs(sigmo, Q, D, sigmo.SIGMO_FIND_FIRST):
            check_every_pair(Q, D, di, qi, r, oracle.FIND_FIRST, qidx=idx)


def test_c5_every_pair_one_batch(sigmo):
    """configs[4] (1,000 queries incl. 30 ring systems, Find All) streamed in
    batches of 250k molecules: every pair of one full batch (the 5th batch of
    rank 0), queries routed by size as StreamRunner does."""
    Q = synth.config_queries(5)
    D = synth.config_data(5, first=4 * 250_000, count=250_000)
    for idx, (di, qi, r) in routed_pairs(sigmo, Q, D, sigmo.SIGMO_FIND_ALL):
        check_every_pair(Q, D, di, qi, r, oracle.FIND_ALL, qidx=idx)


@pytest.mark.parametrize("env", [{"SIGMO_JOIN_BATCH": "1"}, {"SIGMO_JOIN_BATCH": "4"}, {"SIGMO_JOIN_BATCH": "32"},
                                 {"SIGMO_JOIN_BPS": "1"}, {"SIGMO_JOIN_BPS": "1", "SIGMO_JOIN_BATCH": "32"}],
                         ids=["batch1", "batch4", "batch32", "bps1", "bps1-batch32"])
def test_join_schedule_independence(sigmo, monkeypatch, env):
    """The lane join's result does not depend on its schedule: refill batch
    (lanes that must be free before a warp refills) and CTAs per SM (which
    changes the pair-chunk interleaving and the work donation of the drained
    phase); Find All and Find First, every pair of a 20k-molecule configs[1]
    slice including > 32-atom molecules (both join launches)."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    Q, D = synth.config_queries(2), synth.config_data(2, first=40_000, count=20_000)
    ref = oracle.count_dense(Q, D)
    with sigmo.Context(0) as ctx:
        ctx.load_batch(Q, D)
        ctx.filter(4)
        ctx.join(sigmo.SIGMO_FIND_ALL)
        assert np.array_equal(ctx.dense_results(), ref)
        ctx.join(sigmo.SIGMO_FIND_FIRST)
        assert np.array_equal(ctx.dense_results(), (ref > 0).astype(np.uint64))
