"""Print DFS statistics of the join on configs[1] (debug/perf aid)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
import paper_conf_sc_carocfc25_b200 as sigmo

n = int(sys.argv[1]) if len(sys.argv) > 1 else 100_000
L = int(sys.argv[2]) if len(sys.argv) > 2 else 4
cfg = int(sys.argv[3]) if len(sys.argv) > 3 else 2
torch.cuda.set_device(0)
Q, D = synth.config_queries(cfg), synth.config_data(cfg, count=n)
ctx = sigmo.Context(0)
ctx.load_batch(Q, D)
for mode in (0, 1):
    ctx.filter(L)
    ctx.set_timing(True, count_steps=True)
    tot = ctx.join(mode)
    t = ctx.timings()
    ctx.set_timing(False)
    print({"mode": mode, "total": tot, "pairs": ctx.num_pairs(), **{k: t[k] for k in
           ("filter_ms", "join_ms", "dfs_steps", "dfs_iters", "dfs_tail_iters", "dfs_max_stack")}})
