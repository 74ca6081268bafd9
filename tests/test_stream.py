"""Streamed batches and query-size routing (paper_conf_sc_carocfc25_b200.stream,
SURVEY.md 8(d) C5 and configs[3]/[4] with 20-30-atom ring-system queries).
CPU: the query split and the CSR-GO sub-batch are structurally exact.  GPU:
streamed, split totals equal the oracle's totals over the concatenated data."""
import numpy as np
import pytest

import oracle
import synth
from paper_conf_sc_carocfc25_b200 import stream


def test_split_and_subset_cpu():
    Q = synth.config_queries(4)
    groups = stream.split_queries(Q)
    sizes = np.diff(Q.graph_offsets)
    assert len(groups) == 2
    assert np.all(sizes[groups[0]] <= stream.LANE_MAX_QUERY_NODES)
    assert np.all(sizes[groups[1]] > stream.LANE_MAX_QUERY_NODES)
    assert sorted(np.concatenate(groups).tolist()) == list(range(Q.num_graphs))
    for g in groups:
        sub = stream._subset(Q, g)
        assert sub.num_graphs == len(g)
        for k, q in enumerate(g):
            labs, edges = Q.graph(int(q))
            a, b = int(sub.graph_offsets[k]), int(sub.graph_offsets[k + 1])
            assert sub.node_labels[a:b].tolist() == list(labs)
            got = set()
            for v in range(a, b):
                for e in range(int(sub.row_offsets[v]), int(sub.row_offsets[v + 1])):
                    got.add((v - a, int(sub.col_indices[e]) - a, int(sub.edge_labels[e])))
            want = set()
            for u, v, bd in edges:
                want.add((u, v, bd))
                want.add((v, u, bd))
            assert got == want
    # a small sub-batch through the oracle equals the same rows of the full batch
    D = synth.config_data(1, count=40)
    h = stream._subset(Q, groups[0][:25])
    sub = synth.GraphBatch(h.graph_offsets, h.row_offsets, h.col_indices, h.node_labels, h.edge_labels)
    assert np.array_equal(oracle.count_dense(sub, D), oracle.count_dense(Q, D)[groups[0][:25]])


@pytest.mark.gpu
def test_stream_runner_matches_oracle():
    import torch
    import __graft_entry__
    __graft_entry__.build()
    torch.cuda.set_device(0)
    Q = synth.config_queries(4)  # 470 small + 30 ring-system queries -> two routed groups
    batches = [synth.config_data(4, first=300 * i, count=300) for i in range(4)]
    D = synth.GraphBatch.concat(batches)
    with stream.StreamRunner(Q, 0, levels=4) as sr:
        assert len(sr.groups) == 2
        got = sr.run(batches)
        assert np.array_equal(got, oracle.count_totals(Q, D))
        got2 = sr.run(batches[::-1])  # order-free integer sums
        assert np.array_equal(got2, got)
    with stream.StreamRunner(Q, 0, levels=2, mode=oracle.FIND_FIRST) as sr:
        assert np.array_equal(sr.run(batches), oracle.count_totals(Q, D, oracle.FIND_FIRST))
