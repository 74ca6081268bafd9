"""Small driver for ncu: load configs[1] (or N molecules), run W warm-up
steps then S profiled steps of filter + join.  Usage:
    python tools/profile_step.py [molecules] [levels] [steps] [mode] [synth config id]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
import paper_conf_sc_carocfc25_b200 as sigmo

n = int(sys.argv[1]) if len(sys.argv) > 1 else 100_000
L = int(sys.argv[2]) if len(sys.argv) > 2 else 4
S = int(sys.argv[3]) if len(sys.argv) > 3 else 2
mode = int(sys.argv[4]) if len(sys.argv) > 4 else 0
cid = int(sys.argv[5]) if len(sys.argv) > 5 else 2
torch.cuda.set_device(0)
Q, D = synth.config_queries(cid), synth.config_data(cid, count=n)
ctx = sigmo.Context(0)
if os.environ.get("SIGMO_PROFILE_INDUCED") == "1":
    ctx.set_induced(True)
ctx.load_batch(Q, D)
ns = os.environ.get("SIGMO_PROFILE_NS") == "1"  # neighbour-support flag
for _ in range(2 + S):
    ctx.filter(L, neighbor_support=ns)
    ctx.join(mode, total=False)
torch.cuda.synchronize()
print("matches", ctx.join(mode))
