"""CPU filter reference -- TEST INFRASTRUCTURE ONLY.

Plain numpy/Python restatement of SIGMo's filter (Alg. 1, PAPER.md
P:549-605), the masked-bitset signature (section 4.2), the GMCR
mapping rule (section 4.5) and the optional neighbour-support
fixed point (BASELINE.json north_star; R9).  Shares nothing with the
CUDA path; the field table below is this module's own copy of reading R7.

Readings:
  R4  signatures are cumulative: S_k(v)[l] = #{u != v : d(u,v) <= k, L(u)=l}.
      GenerateSignatures (Alg. 1 l.11-18) is written exactly as the paper's
      incremental ring update: S(v, L(u)) += 1 for u in R_k(v) = N^k \\ N^{k-1},
      applied to a persistent S.
  R5  dominance is per field, on every field.
  R6  levels = L: L = 1 labels only; L >= 2 applies radii 1..L-1 (P:553-560,
      P:1594-1598).
  R7  field table below (LSB-first); unlisted labels pool into "other".
  R8  saturate at 2^w - 1 on overflow.
  R10 bitmap view: u32 words, row = query node, bit j of word w = data node
      32w + j.
  R11 GMCR: drop (q, g) if any node of q has no candidate in g.
"""
from __future__ import annotations

from collections import deque

import numpy as np

# R7: (atomic number, bit width), LSB-first; last entry = pooled "other".
FIELDS = [(6, 8), (7, 6), (8, 6), (16, 5), (9, 5), (17, 5), (35, 4), (53, 4), (15, 4), (1, 7), (5, 3), (14, 3),
          (None, 4)]
NF = len(FIELDS)
WIDTHS = np.array([w for _, w in FIELDS], dtype=np.int64)
SATMAX = (1 << WIDTHS) - 1
OFFSETS = np.concatenate([[0], np.cumsum(WIDTHS)[:-1]])
assert int(WIDTHS.sum()) == 64


def field_of(label: int) -> int:
    for i, (z, _) in enumerate(FIELDS[:-1]):
        if z == label:
            return i
    return NF - 1


def _adjacency(B):
    """Python adjacency lists (global ids) of a GraphBatch."""
    return [B.col_indices[B.row_offsets[v]:B.row_offsets[v + 1]].tolist() for v in range(B.num_nodes)]


def _bfs_dist(adj, src, lo, hi):
    """Distances from src to nodes of its graph [lo, hi) (-1 = unreachable)."""
    dist = np.full(hi - lo, -1, np.int64)
    dist[src - lo] = 0
    dq = deque([src])
    while dq:
        u = dq.popleft()
        for w in adj[u]:
            if dist[w - lo] < 0:
                dist[w - lo] = dist[u - lo] + 1
                dq.append(w)
    return dist


def raw_signatures(B, max_radius: int, graphs=None, skip_wildcards: bool = False):
    """Raw (unsaturated) counts S[k][v, f] for k = 1..max_radius, following
    GenerateSignatures (Alg. 1 l.11-18): for each node v and each k, add one to
    S(v, field(L(u))) for every u in the ring R_k(v) = N^k(v) \\ N^{k-1}(v).
    Returns dict k -> int64 array [V, NF] (rows of nodes outside ``graphs``
    stay zero)."""
    adj = _adjacency(B)
    V = B.num_nodes
    fld = np.array([field_of(int(x)) for x in B.node_labels], np.int64)
    # wildcard mode (R22): a '*' query atom (label 0) has no known label, so it
    # adds to no field of its neighbours' signatures (sound: the data
    # signature then dominates on the known labels only)
    wild = (B.node_labels == 0) if skip_wildcards else np.zeros(V, bool)
    S = np.zeros((V, NF), np.int64)
    out = {}
    dists = {}
    gl = range(B.num_graphs) if graphs is None else graphs
    for g in gl:
        lo, hi = int(B.graph_offsets[g]), int(B.graph_offsets[g + 1])
        for v in range(lo, hi):
            dists[v] = (lo, _bfs_dist(adj, v, lo, hi))
    for k in range(1, max_radius + 1):
        for v, (lo, dist) in dists.items():
            ring = np.nonzero(dist == k)[0] + lo          # R_k(v)
            for u in ring:
                if not wild[u]:
                    S[v, fld[u]] += 1                      # S(v, L(u)) <- S(v, L(u)) + 1
        out[k] = S.copy()
    return out


def saturate(S):
    """R8: a field that would overflow stays at its maximum 2^w - 1."""
    return np.minimum(S, SATMAX[None, :])


def pack(Ssat):
    """Masked-bitset signature (section 4.2): fields LSB-first in one u64."""
    out = np.zeros(Ssat.shape[0], np.uint64)
    for f in range(NF):
        out |= Ssat[:, f].astype(np.uint64) << np.uint64(OFFSETS[f])
    return out


def signatures(B, radius: int, graphs=None):
    """Packed u64 signature at the given radius (>= 1) for every node."""
    return pack(saturate(raw_signatures(B, radius, graphs)[radius]))


def candidates_bool(Q, D, levels: int, data_graphs=None, q_rows=None, wildcard: bool = False):
    """Boolean candidate matrix C_L [VQ, VD] (Alg. 1 Filter):
    C_1 = InitializeCandidates (label equality, l.29-37); then for
    k = 1..L-1 RefineCandidates (l.19-28) keeps v_d in C(v_q) iff it was in
    C_prev(v_q) and sat(S_D(v_d)) >= sat(S_Q(v_q)) on every field (R5).
    ``data_graphs`` restricts the data columns that are evaluated (others
    False); ``q_rows`` restricts the query rows (others False)."""
    VQ, VD = Q.num_nodes, D.num_nodes
    rows = range(VQ) if q_rows is None else q_rows
    SQ = raw_signatures(Q, max(levels - 1, 0), skip_wildcards=wildcard)
    SD = raw_signatures(D, max(levels - 1, 0), data_graphs)
    if data_graphs is None:
        cols = np.ones(VD, bool)
    else:
        cols = np.zeros(VD, bool)
        for g in data_graphs:
            cols[int(D.graph_offsets[g]):int(D.graph_offsets[g + 1])] = True
    C = np.zeros((VQ, VD), bool)
    for vq in rows:
        if wildcard and Q.node_labels[vq] == 0:                       # '*': every atom (R22)
            C[vq] = cols.copy()
        else:
            C[vq] = (D.node_labels == Q.node_labels[vq]) & cols      # InitializeCandidates
    for k in range(1, levels):                                        # k = 1 .. s-1
        sq, sd = saturate(SQ[k]), saturate(SD[k])
        for vq in rows:
            C[vq] &= np.all(sq[vq][None, :] <= sd, axis=1)            # RefineCandidates
    return C


def neighbour_support(Q, D, C, wildcard: bool = False):
    """Greatest fixed point of the neighbour-support rule (north_star; R9):
    remove v_d from C(v_q) if some query edge (v_q, u_q, b) has no data edge
    (v_d, u_d, b) with u_d in C(u_q).  Naive iteration until nothing changes."""
    C = C.copy()
    dsrc = np.repeat(np.arange(D.num_nodes), np.diff(D.row_offsets))
    ddst = D.col_indices.astype(np.int64)
    dlab = D.edge_labels
    qsrc = np.repeat(np.arange(Q.num_nodes), np.diff(Q.row_offsets))
    qdst = Q.col_indices.astype(np.int64)
    qlab = Q.edge_labels
    changed = True
    while changed:
        changed = False
        for e in range(qsrc.shape[0]):
            vq, uq, b = int(qsrc[e]), int(qdst[e]), int(qlab[e])
            m = ((dlab == b) | (wildcard and b == 0)) & C[uq, ddst]  # '~' bond: any label (R22)
            support = np.zeros(D.num_nodes, bool)
            support[dsrc[m]] = True
            new = C[vq] & support
            if not np.array_equal(new, C[vq]):
                C[vq] = new
                changed = True
    return C


def to_bitmap(C):
    """R10 view: [VQ, ceil(VD/32)] uint32, bit j of word w = data node 32w+j."""
    VQ, VD = C.shape
    W = (VD + 31) // 32
    pad = np.zeros((VQ, W * 32), bool)
    pad[:, :VD] = C
    by = np.packbits(pad, axis=1, bitorder="little")
    return np.ascontiguousarray(by).view(np.uint32).reshape(VQ, W) if VQ else np.zeros((0, W), np.uint32)


def candidates(Q, D, levels: int, neighbour: bool = False, wildcard: bool = False):
    C = candidates_bool(Q, D, levels, wildcard=wildcard)
    if neighbour:
        C = neighbour_support(Q, D, C, wildcard=wildcard)
    return to_bitmap(C)


def gmcr(Q, D, C):
    """Mapping rule: pair (q, g) survives iff every node of q
    has at least one candidate among the nodes of g.  Returns bool [NQ, ND]."""
    NQ, ND = Q.num_graphs, D.num_graphs
    out = np.zeros((NQ, ND), bool)
    for g in range(ND):
        lo, hi = int(D.graph_offsets[g]), int(D.graph_offsets[g + 1])
        anyc = C[:, lo:hi].any(axis=1)
        for q in range(NQ):
            a, b = int(Q.graph_offsets[q]), int(Q.graph_offsets[q + 1])
            out[q, g] = bool(anyc[a:b].all())
    return out
