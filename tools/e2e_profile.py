"""Host-side breakdown of the e2e step (sigmo_load_batch phases via
SIGMO_DEBUG_LOAD) on configs[2]."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["SIGMO_DEBUG_LOAD"] = "1"
import torch
import synth
import paper_conf_sc_carocfc25_b200 as sigmo
torch.cuda.set_device(0)
Q, D = synth.config_queries(3), synth.config_data(3)
cq, cd = sigmo.as_c_batch(Q, pinned=True), sigmo.as_c_batch(D, pinned=True)
ctx = sigmo.Context(0)
for i in range(4):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ctx.load_batch(cq, cd)
    t1 = time.perf_counter()
    ctx.filter(2)
    tot = ctx.join(sigmo.SIGMO_FIND_ALL, total=True)
    t2 = time.perf_counter()
    print(f"load {1000*(t1-t0):.1f} ms, filter+join+D2H {1000*(t2-t1):.1f} ms, total {1000*(t2-t0):.1f}", flush=True)
print("threads", os.cpu_count(), len(os.sched_getaffinity(0)))
