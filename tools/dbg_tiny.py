import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import synth, oracle
from synth import GraphBatch
import paper_conf_sc_carocfc25_b200 as sigmo
rng = np.random.default_rng(2024)
ds = [synth.random_labelled_graph(rng, int(rng.integers(0, 12)), float(rng.uniform(0.1, 0.7)), labels=(6, 7), bonds=(1, 2)) for _ in range(400)]
qs = [synth.random_labelled_graph(rng, int(rng.integers(1, 6)), float(rng.uniform(0.3, 1.0)), labels=(6, 7), bonds=(1, 2)) for _ in range(40)]
Q, D = GraphBatch.from_graphs(qs), GraphBatch.from_graphs(ds)
ref = oracle.count_dense(Q, D)
ctx = sigmo.Context(0)
ctx.load_batch(Q, D)
for bk in ("1", "4", "32"):
    os.environ["SIGMO_JOIN_BATCH"] = bk
    ctx.filter(1)
    ctx.join(sigmo.SIGMO_FIND_ALL)
    got = ctx.dense_results()
    bad = np.argwhere(got != ref)
    print("batchK", bk, "mismatches", len(bad))
    for q, g in bad[:10]:
        print(q, g, "nq", len(qs[q][0]), "ng", len(ds[g][0]), "qedges", len(qs[q][1]), "got", got[q, g], "ref", ref[q, g])
