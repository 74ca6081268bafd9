"""Brute-force enumeration of embeddings -- TEST INFRASTRUCTURE ONLY (pin P4).

Enumerates every injective tuple (f(0), ..., f(n_q-1)) of data nodes and keeps
those satisfying Def. 2.1 conditions (1) and (2) with bond labels
compared on every query edge (R1-R3).  Exponential; use
only for n_g <= 8, n_q <= 5.
"""
from __future__ import annotations

import itertools


def _induced_ok(f, qedges, bond, nq):
    """Condition (3) of the induced reading (G_D[X]; R21):
    non-adjacent query nodes map to non-adjacent data nodes."""
    qadj = {(u, v) for (u, v, _) in qedges} | {(v, u) for (u, v, _) in qedges}
    return all((f[u], f[v]) not in bond for u in range(nq) for v in range(nq) if u != v and (u, v) not in qadj)


def _label_ok(ql, dl, wildcard):
    return ql == dl or (wildcard and ql == 0)          # (1); wildcard '*' = label 0 (R22)


def _bond_ok(db, qb, wildcard):
    return db is not None and (db == qb or (wildcard and qb == 0))  # (2); wildcard '~' = bond 0


def brute_embeddings(qgraph, dgraph, induced: bool = False, wildcard: bool = False):
    """Yield every embedding f (tuple, f[i] = data node of query node i)."""
    qlab, qedges = qgraph
    dlab, dedges = dgraph
    nq, nd = len(qlab), len(dlab)
    bond = {}
    for (u, v, b) in dedges:
        bond[(u, v)] = b
        bond[(v, u)] = b
    for f in itertools.permutations(range(nd), nq):
        if any(not _label_ok(qlab[i], dlab[f[i]], wildcard) for i in range(nq)):           # condition (1)
            continue
        if any(not _bond_ok(bond.get((f[u], f[v])), b, wildcard) for (u, v, b) in qedges):  # condition (2)
            continue
        if induced and not _induced_ok(f, qedges, bond, nq):
            continue
        yield f


def brute_count(qgraph, dgraph, induced: bool = False, wildcard: bool = False) -> int:
    """qgraph/dgraph: (labels, [(u, v, bond), ...]) with local ids."""
    return sum(1 for _ in brute_embeddings(qgraph, dgraph, induced, wildcard))


def brute_dense(qgraphs, dgraphs, find_first: bool = False, induced: bool = False, wildcard: bool = False):
    out = [[brute_count(q, d, induced, wildcard) for d in dgraphs] for q in qgraphs]
    if find_first:
        out = [[1 if c else 0 for c in row] for row in out]
    return out
