"""CPU-side checks of the boundary: libsigmo.so loads without a GPU, exports
every symbol include/sigmo.h declares, and sigmo_validate_batch returns the
documented error class for every invalid-input class (no compute calls)."""
import ctypes
import os
import re

import numpy as np
import pytest

import synth
from synth import GraphBatch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_sc_carocfc25_b200 as sigmo
    return sigmo


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "sigmo.h")).read()
    return sorted(set(re.findall(r"\b(sigmo_[a-z_]+)\s*\(", txt)))


def test_library_exports_every_header_symbol(lib):
    syms = header_symbols()
    assert len(syms) >= 16
    L = ctypes.CDLL(os.path.join(ROOT, "paper_conf_sc_carocfc25_b200", "libsigmo.so"))
    for s in syms:
        assert hasattr(L, s), s
    from paper_conf_sc_carocfc25_b200 import _native
    assert sorted(_native.EXPORTS) == syms
    assert lib.version().startswith("sigmo-b200")


def test_no_cpu_fallback_without_library(monkeypatch, tmp_path):
    from paper_conf_sc_carocfc25_b200 import _native
    monkeypatch.setattr(_native, "_lib", None)
    with pytest.raises(RuntimeError, match="no CPU fallback"):
        _native.load_library(str(tmp_path / "missing.so"))


def _ok(lib, b, q=False):
    st, msg = lib.validate_batch(b, q)
    return st, msg


def test_validate_accepts_valid_batches(lib):
    assert _ok(lib, synth.fig3_batch())[0] == 0
    assert _ok(lib, synth.config_queries(2), True)[0] == 0
    assert _ok(lib, synth.molecules(5, 0, 500))[0] == 0
    assert _ok(lib, GraphBatch.empty())[0] == 0
    # single-node query, disconnected graphs
    assert _ok(lib, GraphBatch.from_graphs([([6], [])]), True)[0] == 0
    assert _ok(lib, GraphBatch.from_graphs([([6, 6, 7], [(0, 1, 1)])]))[0] == 0
    # empty data graph inside a batch
    assert _ok(lib, GraphBatch.from_graphs([([6], []), ([], []), ([6, 6], [(0, 1, 1)])]))[0] == 0


def _mutate(b, **kw):
    d = dict(graph_offsets=b.graph_offsets.copy(), row_offsets=b.row_offsets.copy(),
             col_indices=b.col_indices.copy(), node_labels=b.node_labels.copy(), edge_labels=b.edge_labels.copy())
    d.update(kw)
    return GraphBatch(**d)


INVALID_GRAPH, LIMIT = -2, -3


def test_validate_rejects_invalid_graphs(lib):
    B = synth.fig3_batch()
    # non-monotone graph offsets
    assert _ok(lib, _mutate(B, graph_offsets=np.array([0, 7, 5])))[0] == INVALID_GRAPH
    # graph_offsets[0] != 0
    assert _ok(lib, _mutate(B, graph_offsets=np.array([1, 5, 9])))[0] == INVALID_GRAPH
    # row offsets decreasing
    ro = B.row_offsets.copy()
    ro[3], ro[4] = ro[4], ro[3]
    assert _ok(lib, _mutate(B, row_offsets=ro))[0] == INVALID_GRAPH
    # column outside the owning graph (node 0 -> node 6 of G1)
    col = B.col_indices.copy()
    col[0] = 6
    assert _ok(lib, _mutate(B, col_indices=col))[0] == INVALID_GRAPH
    # self loop
    col = B.col_indices.copy()
    col[0] = 0
    assert _ok(lib, _mutate(B, col_indices=col))[0] == INVALID_GRAPH
    # asymmetric edge label
    el = B.edge_labels.copy()
    el[0] = 2
    st, msg = _ok(lib, _mutate(B, edge_labels=el))
    assert st == INVALID_GRAPH and "asymmetric" in msg
    # duplicate edge: node 0 lists 1 twice (and 1 lists 0 twice to stay symmetric)
    g = GraphBatch(np.array([0, 2]), np.array([0, 2, 4]), np.array([1, 1, 0, 0]), np.array([6, 6]),
                   np.array([1, 1, 1, 1]))
    st, msg = _ok(lib, g)
    assert st == INVALID_GRAPH and "duplicate" in msg
    # empty query graph
    assert _ok(lib, GraphBatch.from_graphs([([], [])]), True)[0] == INVALID_GRAPH
    # num_nodes inconsistent with graph offsets
    assert _ok(lib, _mutate(B, graph_offsets=np.array([0, 5, 8])))[0] != 0


def test_validate_limits(lib):
    big_q = GraphBatch.from_graphs([([6] * 33, [(i, i + 1, 1) for i in range(32)])])
    assert _ok(lib, big_q, True)[0] == LIMIT
    ok_q = GraphBatch.from_graphs([([6] * 32, [(i, i + 1, 1) for i in range(31)])])
    assert _ok(lib, ok_q, True)[0] == 0
    big_d = GraphBatch.from_graphs([([6] * 257, [(i, i + 1, 1) for i in range(256)])])
    assert _ok(lib, big_d)[0] == LIMIT
    ok_d = GraphBatch.from_graphs([([6] * 256, [(i, i + 1, 1) for i in range(255)])])
    assert _ok(lib, ok_d)[0] == 0


def test_library_has_no_unresolved_internal_symbols():
    """Every internal (namespace sigmo) function the library calls is defined
    in it: a missing launcher would only surface at dlopen on the GPU box."""
    import subprocess
    from paper_conf_sc_carocfc25_b200 import build as B
    out = subprocess.run(["nm", "-D", "--undefined-only", B.LIB], capture_output=True, text=True).stdout
    missing = [l.split()[-1] for l in out.splitlines() if "_ZN5sigmo" in l]
    assert missing == [], missing
