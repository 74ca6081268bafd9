import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth, oracle
from oracle import filter_ref as fr
from synth import GraphBatch
import paper_conf_sc_carocfc25_b200 as sigmo
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from test_gpu_wildcard import wildcarded
torch.cuda.set_device(0)
Q0, D = synth.config_queries(1), synth.config_data(1)
Q = wildcarded(Q0.graphs(), 101)
print("qlabels", Q.node_labels.tolist())
print("qbonds", Q.edge_labels.tolist())
with sigmo.Context(0) as c:
    c.set_wildcards(True)
    c.load_batch(Q, D)
    c.filter(1)
    bm = c.candidates()
    c.join(sigmo.SIGMO_FIND_ALL)
    fa = c.dense_results()
Cb = fr.candidates_bool(Q, D, 1, wildcard=True)
ref = fr.to_bitmap(Cb)
for r in range(Q.num_nodes):
    if not np.array_equal(bm[r], ref[r]):
        nb = np.unpackbits(bm[r].view(np.uint8), bitorder="little")[:D.num_nodes].astype(bool)
        print("row", r, "label", Q.node_labels[r], "gpu bits", nb.sum(), "ref bits", Cb[r].sum(),
              "gpu-only labels", sorted(set(D.node_labels[nb & ~Cb[r]].tolist())), "ref-only labels", sorted(set(D.node_labels[Cb[r] & ~nb].tolist())))
refc = oracle.count_dense(Q, D, oracle.WILDCARD)
bad = np.argwhere(fa != refc)
print("count mismatches", len(bad), bad[:10].tolist())
for q, g in bad[:5]:
    print(q, g, fa[q, g], refc[q, g], Q.graphs()[q])
