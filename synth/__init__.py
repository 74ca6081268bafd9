"""Seeded synthetic inputs for SIGMo (inputs only -- no method arithmetic).

This is the ONE module shared by the oracle side and the CUDA side
(DESIGN.md "Input recipe").  It produces CSR-GO batches (section 4.1,
P:804-840, Fig. 3): ``graph_offsets`` indexes node ids per graph,
``row_offsets``/``col_indices`` are a standard CSR over the concatenation of
all graphs (global node ids, both directions of every undirected edge),
``node_labels`` are atom labels (atomic numbers, R13 heavy-atom graphs) and
``edge_labels`` bond labels (R14: 1 single, 2 double, 3 triple, 4 aromatic).

Molecules come from ``synth.c`` (counter-based: molecule i is a pure function
of (seed, i, mode)).  Queries are (i) a fixed functional-group library,
(ii) random connected subgraphs of 3-8 atoms BFS-grown inside molecules drawn
with the query seed, (iii) 20-30-atom ring-system patterns cut from ring-rich
molecules.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass
from typing import List, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libsigmo_synth.so")
_lib = None

# element symbols -> atomic number (labels are atomic numbers, R13)
Z = {"H": 1, "B": 5, "C": 6, "N": 7, "O": 8, "F": 9, "Si": 14, "P": 15, "S": 16,
     "Cl": 17, "Br": 35, "I": 53}

DATA_SEED_BASE = 0x51C0_0000
QUERY_SEED_BASE = 0x9E00_0000


def build_lib(force: bool = False) -> str:
    src = os.path.join(_HERE, "synth.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-pthread", src, "-o", _LIB_PATH, "-lm"])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build_lib()
        lib = ctypes.CDLL(_LIB_PATH)
        i64p = ctypes.POINTER(ctypes.c_int64)
        i32p = ctypes.POINTER(ctypes.c_int32)
        u8p = ctypes.POINTER(ctypes.c_uint8)
        lib.synth_sizes.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_int,
                                    i32p, i32p]
        lib.synth_fill.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_int,
                                   i64p, i64p, i64p, i32p, u8p, u8p]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


@dataclass
class GraphBatch:
    """A CSR-GO batch of labelled undirected graphs (host numpy arrays)."""
    graph_offsets: np.ndarray  # int64 [G+1]
    row_offsets: np.ndarray    # int64 [V+1]
    col_indices: np.ndarray    # int32 [E2]
    node_labels: np.ndarray    # uint8 [V]
    edge_labels: np.ndarray    # uint8 [E2]

    def __post_init__(self):
        self.graph_offsets = np.ascontiguousarray(self.graph_offsets, dtype=np.int64)
        self.row_offsets = np.ascontiguousarray(self.row_offsets, dtype=np.int64)
        self.col_indices = np.ascontiguousarray(self.col_indices, dtype=np.int32)
        self.node_labels = np.ascontiguousarray(self.node_labels, dtype=np.uint8)
        self.edge_labels = np.ascontiguousarray(self.edge_labels, dtype=np.uint8)

    @property
    def num_graphs(self) -> int:
        return int(self.graph_offsets.shape[0] - 1)

    @property
    def num_nodes(self) -> int:
        return int(self.graph_offsets[-1])

    @property
    def num_adj(self) -> int:
        return int(self.row_offsets[-1])

    def sizes(self) -> np.ndarray:
        return np.diff(self.graph_offsets)

    @staticmethod
    def empty() -> "GraphBatch":
        return GraphBatch(np.zeros(1, np.int64), np.zeros(1, np.int64), np.zeros(0, np.int32),
                          np.zeros(0, np.uint8), np.zeros(0, np.uint8))

    @staticmethod
    def from_graphs(graphs: Sequence[Tuple[Sequence[int], Sequence[Tuple[int, int, int]]]]) -> "GraphBatch":
        """graphs: list of (node_labels, [(u, v, bond_label), ...]) with local ids."""
        goff = [0]
        roff = [0]
        cols: List[int] = []
        labs: List[int] = []
        elabs: List[int] = []
        for labels, edges in graphs:
            n = len(labels)
            base = goff[-1]
            nbrs: List[List[Tuple[int, int]]] = [[] for _ in range(n)]
            for (u, v, b) in edges:
                nbrs[u].append((v, b))
                nbrs[v].append((u, b))
            for u in range(n):
                for (v, b) in sorted(nbrs[u]):
                    cols.append(base + v)
                    elabs.append(b)
                roff.append(len(cols))
                labs.append(labels[u])
            goff.append(base + n)
        return GraphBatch(np.array(goff), np.array(roff), np.array(cols), np.array(labs), np.array(elabs))

    def graph(self, g: int) -> Tuple[List[int], List[Tuple[int, int, int]]]:
        """(labels, undirected edge list u<v with bond label), local ids."""
        a, b = int(self.graph_offsets[g]), int(self.graph_offsets[g + 1])
        labels = [int(x) for x in self.node_labels[a:b]]
        edges = []
        for u in range(a, b):
            for e in range(int(self.row_offsets[u]), int(self.row_offsets[u + 1])):
                v = int(self.col_indices[e])
                if u < v:
                    edges.append((u - a, v - a, int(self.edge_labels[e])))
        return labels, edges

    def graphs(self):
        return [self.graph(g) for g in range(self.num_graphs)]

    def slice(self, g0: int, g1: int) -> "GraphBatch":
        """Graphs g0..g1-1 as a new batch with renumbered node ids."""
        a, b = int(self.graph_offsets[g0]), int(self.graph_offsets[g1])
        ea, eb = int(self.row_offsets[a]), int(self.row_offsets[b])
        return GraphBatch(self.graph_offsets[g0:g1 + 1] - a, self.row_offsets[a:b + 1] - ea,
                          self.col_indices[ea:eb] - a, self.node_labels[a:b], self.edge_labels[ea:eb])

    @staticmethod
    def concat(batches: Sequence["GraphBatch"]) -> "GraphBatch":
        goff = [np.zeros(1, np.int64)]
        roff = [np.zeros(1, np.int64)]
        cols, labs, elabs = [], [], []
        nb = 0
        eb = 0
        for B in batches:
            goff.append(B.graph_offsets[1:] + nb)
            roff.append(B.row_offsets[1:] + eb)
            cols.append(B.col_indices.astype(np.int64) + nb)
            labs.append(B.node_labels)
            elabs.append(B.edge_labels)
            nb += B.num_nodes
            eb += B.num_adj
        return GraphBatch(np.concatenate(goff), np.concatenate(roff),
                          np.concatenate(cols) if cols else np.zeros(0, np.int32),
                          np.concatenate(labs) if labs else np.zeros(0, np.uint8),
                          np.concatenate(elabs) if elabs else np.zeros(0, np.uint8))

    def nbytes(self) -> int:
        return int(self.graph_offsets.nbytes + self.row_offsets.nbytes + self.col_indices.nbytes
                   + self.node_labels.nbytes + self.edge_labels.nbytes)


# ----------------------------------------------------------------------------
# molecules
# ----------------------------------------------------------------------------

def molecule_sizes(seed: int, first: int, count: int, mode: int = 0, nthreads: int | None = None) -> np.ndarray:
    """Atom counts of molecules first..first+count-1 of the stream (no graphs
    built): what a shard planner needs to balance ranks by atoms."""
    lib = _load()
    nthreads = nthreads or min(32, os.cpu_count() or 1)
    natoms = np.zeros(count, np.int32)
    nadj = np.zeros(count, np.int32)
    if count:
        lib.synth_sizes(seed, first, count, mode, nthreads, _ptr(natoms, ctypes.c_int32), _ptr(nadj, ctypes.c_int32))
    return natoms


def molecules(seed: int, first: int, count: int, mode: int = 0, nthreads: int | None = None) -> GraphBatch:
    """Molecules first..first+count-1 of the stream (seed, mode) as one batch."""
    lib = _load()
    nthreads = nthreads or min(32, os.cpu_count() or 1)
    natoms = np.zeros(count, np.int32)
    nadj = np.zeros(count, np.int32)
    if count == 0:
        return GraphBatch.empty()
    lib.synth_sizes(seed, first, count, mode, nthreads, _ptr(natoms, ctypes.c_int32), _ptr(nadj, ctypes.c_int32))
    goff = np.zeros(count + 1, np.int64)
    aoff = np.zeros(count + 1, np.int64)
    np.cumsum(natoms, out=goff[1:])
    np.cumsum(nadj, out=aoff[1:])
    V, E2 = int(goff[-1]), int(aoff[-1])
    roff = np.zeros(V + 1, np.int64)
    col = np.zeros(E2, np.int32)
    nlab = np.zeros(V, np.uint8)
    elab = np.zeros(E2, np.uint8)
    lib.synth_fill(seed, first, count, mode, nthreads, _ptr(goff, ctypes.c_int64), _ptr(aoff, ctypes.c_int64),
                   _ptr(roff, ctypes.c_int64), _ptr(col, ctypes.c_int32), _ptr(nlab, ctypes.c_uint8),
                   _ptr(elab, ctypes.c_uint8))
    return GraphBatch(goff, roff, col, nlab, elab)


# ----------------------------------------------------------------------------
# queries
# ----------------------------------------------------------------------------

def _ring(symbols, bond):
    n = len(symbols)
    return [Z[s] for s in symbols], [(i, (i + 1) % n, bond) for i in range(n)]


def _with(base, extra_atoms, extra_edges):
    labels, edges = base
    return list(labels) + [Z[s] for s in extra_atoms], list(edges) + list(extra_edges)


def _chain(symbols, bonds, branches=()):
    """linear chain of symbols with bond list, plus branches [(at, symbol, bond)]."""
    labels = [Z[s] for s in symbols]
    edges = [(i, i + 1, b) for i, b in enumerate(bonds)]
    for (at, s, b) in branches:
        labels.append(Z[s])
        edges.append((at, len(labels) - 1, b))
    return labels, edges


BENZENE = _ring("CCCCCC", 4)

# Functional-group library (3-9 heavy atoms; 1 single 2 double 3 triple 4 aromatic).
LIBRARY = {
    "nitrile": _chain("CCN", [1, 3]),
    "ketone": _chain("CCC", [1, 1], [(1, "O", 2)]),
    "carboxylic_acid": _chain("CCO", [1, 1], [(1, "O", 2)]),
    "ester": _chain("CCOC", [1, 1, 1], [(1, "O", 2)]),
    "amide": _chain("CCN", [1, 1], [(1, "O", 2)]),
    "nitro": _chain("CNO", [1, 2], [(1, "O", 2)]),
    "benzene": BENZENE,
    "pyridine": _ring("NCCCCC", 4),
    "phenol": _with(BENZENE, ["O"], [(0, 6, 1)]),
    "thiophene": _ring("SCCCC", 4),
    "aldehyde": _chain("CCO", [1, 2]),
    "urea": _chain("NCN", [1, 1], [(1, "O", 2)]),
    "carbamate": _chain("NCO", [1, 1], [(1, "O", 2)]),
    "sulfonamide": _chain("CSN", [1, 1], [(1, "O", 2), (1, "O", 2)]),
    "sulfone": _chain("CSC", [1, 1], [(1, "O", 2), (1, "O", 2)]),
    "ether": _chain("COC", [1, 1]),
    "thioether": _chain("CSC", [1, 1]),
    "secondary_amine": _chain("CNC", [1, 1]),
    "cf3": _chain("CC", [1], [(1, "F", 1), (1, "F", 1), (1, "F", 1)]),
    "tert_butyl": _chain("CC", [1], [(1, "C", 1), (1, "C", 1), (1, "C", 1)]),
    "furan": _ring("OCCCC", 4),
    "pyrrole": _ring("NCCCC", 4),
    "imidazole": _ring("NCNCC", 4),
    "cyclohexane": _ring("CCCCCC", 1),
    "cyclopentane": _ring("CCCCC", 1),
    "piperidine": _ring("NCCCCC", 1),
    "morpholine": _ring("NCCOCC", 1),
    "aniline": _with(BENZENE, ["N"], [(0, 6, 1)]),
    "chlorobenzene": _with(BENZENE, ["Cl"], [(0, 6, 1)]),
    "bromobenzene": _with(BENZENE, ["Br"], [(0, 6, 1)]),
    "toluene": _with(BENZENE, ["C"], [(0, 6, 1)]),
    "acetophenone_core": _with(BENZENE, ["C", "O"], [(0, 6, 1), (6, 7, 2)]),
    "anisole": _with(BENZENE, ["O", "C"], [(0, 6, 1), (6, 7, 1)]),
    "benzylamine": _with(BENZENE, ["C", "N"], [(0, 6, 1), (6, 7, 1)]),
    "hydroxyl_ethyl": _chain("CCO", [1, 1]),
}

# 10 library functional groups
C1_NAMES = ["nitrile", "ketone", "carboxylic_acid", "ester", "amide", "nitro", "benzene", "pyridine", "phenol",
            "thiophene"]


def library(names: Sequence[str] | None = None):
    names = list(LIBRARY.keys()) if names is None else list(names)
    return [LIBRARY[n] for n in names]


def _grow_subgraph(labels, edges, rng: np.random.Generator, k: int, prefer_ring: bool = False):
    n = len(labels)
    adj = [[] for _ in range(n)]
    for (u, v, b) in edges:
        adj[u].append(v)
        adj[v].append(u)
    if n < k:
        return None
    ring_atoms = None
    if prefer_ring:
        deg = np.array([len(a) for a in adj])
        ring_atoms = set(int(i) for i in np.nonzero(deg >= 2)[0])
    start = int(rng.integers(n))
    chosen = [start]
    cset = {start}
    frontier = set(adj[start])
    while len(chosen) < k and frontier:
        fl = sorted(frontier)
        if ring_atoms is not None:
            pri = [v for v in fl if v in ring_atoms]
            if pri and rng.random() < 0.9:
                fl = pri
        v = fl[int(rng.integers(len(fl)))]
        chosen.append(v)
        cset.add(v)
        frontier.discard(v)
        frontier.update(w for w in adj[v] if w not in cset)
    if len(chosen) < k:
        return None
    idx = {v: i for i, v in enumerate(chosen)}
    sub_edges = [(idx[u], idx[v], b) for (u, v, b) in edges if u in cset and v in cset]
    return [labels[v] for v in chosen], sub_edges


def random_subgraph_queries(seed: int, count: int, kmin: int = 3, kmax: int = 8, mode: int = 0,
                            prefer_ring: bool = False):
    """Random connected subgraphs (BFS-grown, induced edges) of molecules drawn
    with the query seed; every query has >= 1 embedding in its source."""
    rng = np.random.default_rng(seed)
    out = []
    mol_index = 0
    while len(out) < count:
        B = molecules(seed, mol_index, 64, mode=mode, nthreads=1)
        mol_index += 64
        for g in range(B.num_graphs):
            if len(out) >= count:
                break
            labels, edges = B.graph(g)
            k = int(rng.integers(kmin, kmax + 1))
            sub = _grow_subgraph(labels, edges, rng, k, prefer_ring)
            if sub is not None:
                out.append(sub)
    return out


def ring_system_queries(seed: int, count: int):
    """20-30-atom ring-system patterns from ring-rich molecules (mode 1)."""
    return random_subgraph_queries(seed, count, 20, 30, mode=1, prefer_ring=True)


def config_queries(c: int) -> GraphBatch:
    """Query sets of SURVEY.md 8(d) configs 1-5."""
    qseed = QUERY_SEED_BASE + c
    names35 = list(LIBRARY.keys())[:35]
    if c == 1:
        return GraphBatch.from_graphs(library(C1_NAMES))
    if c == 2:
        return GraphBatch.from_graphs(library(names35) + random_subgraph_queries(qseed, 15))
    if c == 3:
        return GraphBatch.from_graphs(library(names35) + random_subgraph_queries(qseed, 65))
    if c == 4:
        return GraphBatch.from_graphs(library(names35) + random_subgraph_queries(qseed, 435)
                                      + ring_system_queries(qseed + 1, 30))
    if c == 5:
        return GraphBatch.from_graphs(library(names35) + random_subgraph_queries(qseed, 935)
                                      + ring_system_queries(qseed + 1, 30))
    raise ValueError(c)


CONFIG_MOLECULES = {1: 200, 2: 100_000, 3: 1_000_000, 4: 1_000_000, 5: 10_000_000}


def config_data(c: int, first: int = 0, count: int | None = None, mode: int = 0) -> GraphBatch:
    n = CONFIG_MOLECULES[c] if count is None else count
    return molecules(DATA_SEED_BASE + c, first, n, mode=mode)


# PAPER.md Fig. 3: G0 = 5-cycle on nodes 0-4, G1 = star centred at 6
FIG3_GRAPHS = [
    ([6] * 5, [(0, 1, 1), (1, 2, 1), (2, 3, 1), (3, 4, 1), (0, 4, 1)]),
    ([6] * 4, [(1, 0, 1), (1, 2, 1), (1, 3, 1)]),
]


def fig3_batch() -> GraphBatch:
    return GraphBatch.from_graphs(FIG3_GRAPHS)


def random_labelled_graph(rng: np.random.Generator, n: int, p: float, labels: Sequence[int] = (6, 7, 8),
                          bonds: Sequence[int] = (1, 2)):
    """Erdos-Renyi labelled graph (tiny random cases for brute-force pins)."""
    lab = [int(labels[int(rng.integers(len(labels)))]) for _ in range(n)]
    edges = []
    for u in range(n):
        for v in range(u + 1, n):
            if rng.random() < p:
                edges.append((u, v, int(bonds[int(rng.integers(len(bonds)))])))
    return lab, edges
