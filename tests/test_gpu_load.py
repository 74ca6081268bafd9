"""Device-side load of large data batches (k_load_data: per-entry validation
and CSR-GO packing on the GPU, sigmo_load_batch contract in include/sigmo.h):
same packed arrays and results as the host path, every invalid-input class
reported with the offending graph."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sigmo():
    import torch
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_sc_carocfc25_b200 as s
    torch.cuda.set_device(0)
    return s


def test_device_load_equals_host_load(sigmo, monkeypatch):
    Q, D = synth.config_queries(2), synth.config_data(2, count=5_000)  # ~125k nodes: device path
    assert D.num_nodes >= 65536
    out = {}
    for host in ("0", "1"):
        monkeypatch.setenv("SIGMO_HOST_LOAD", host)
        with sigmo.Context(0) as c:
            c.load_batch(Q, sigmo.as_c_batch(D, pinned=host == "0"))
            go, ro, co, nl, el = c.packed_batch(1)
            assert np.array_equal(go, D.graph_offsets) and np.array_equal(ro, D.row_offsets)
            assert np.array_equal(co, D.col_indices) and np.array_equal(nl, D.node_labels)
            assert np.array_equal(el, D.edge_labels)
            c.filter(2)
            c.join(sigmo.SIGMO_FIND_ALL)
            out[host] = c.dense_results()
    assert np.array_equal(out["0"], out["1"])
    assert np.array_equal(out["0"], oracle.count_dense(Q, D))


def _corrupt(D, kind, g):
    col = D.col_indices.copy()
    el = D.edge_labels.copy()
    ro = D.row_offsets.copy()
    a = int(D.graph_offsets[g])
    e = int(ro[a])  # first adjacency entry of the graph's first node
    if kind == "outside":
        col[e] = int(D.graph_offsets[g + 1]) + 1
    elif kind == "self":
        col[e] = a
    elif kind == "duplicate":
        col[e + 1] = col[e]
    elif kind == "asymmetric":
        el[e] = 3 if el[e] != 3 else 2
    elif kind == "row_offsets":
        ro[a + 1] = ro[a] - 1 if ro[a] > 0 else ro[a]
        ro[a + 1], ro[a] = ro[a], ro[a + 1] if ro[a] > 0 else ro[a]
    return synth.GraphBatch(D.graph_offsets, ro, col, D.node_labels, el)


@pytest.mark.parametrize("kind,msg", [("outside", "outside its graph"), ("self", "self-loop"),
                                      ("duplicate", "duplicate edge"), ("asymmetric", "asymmetric")])
def test_device_load_rejects_invalid_graphs(sigmo, kind, msg):
    Q, D = synth.config_queries(1), synth.config_data(2, count=3_000)
    assert D.num_nodes >= 65536
    g = 1234
    while int(D.row_offsets[int(D.graph_offsets[g]) + 1] - D.row_offsets[int(D.graph_offsets[g])]) < 2:
        g += 1  # a first node with >= 2 neighbours (the duplicate case needs two entries)
    bad = _corrupt(D, kind, g)
    with sigmo.Context(0) as c:
        with pytest.raises(sigmo.SigmoError) as e:
            c.load_batch(Q, bad)
        assert e.value.status == -2, e.value
        assert msg in str(e.value) and f"data graph {g}" in str(e.value), str(e.value)
        c.load_batch(Q, D)  # the context stays usable
        c.filter(2)
        assert c.join(sigmo.SIGMO_FIND_ALL) == int(oracle.count_dense(Q, D).sum())
