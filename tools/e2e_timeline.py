"""Timeline of one e2e step (bench.py's StreamRunner path) from the CUPTI
trace of torch.profiler: per stream, copies and kernels with start/end (ms).
Usage: python tools/e2e_timeline.py [molecules] [batch]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from torch.profiler import ProfilerActivity, profile

import synth
import paper_conf_sc_carocfc25_b200 as sigmo
from paper_conf_sc_carocfc25_b200.stream import StreamRunner

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
bs = int(sys.argv[2]) if len(sys.argv) > 2 else 250_000
torch.cuda.set_device(0)
Q, D = synth.config_queries(3), synth.config_data(3, count=n)
nb = max(1, (n + bs - 1) // bs)
subs = [sigmo.as_c_batch(D.slice(i * n // nb, (i + 1) * n // nb), pinned=True) for i in range(nb)]
r = StreamRunner(Q, 0, levels=2, split=False)
for _ in range(2):
    r.run(subs)
torch.cuda.synchronize()
t0 = time.perf_counter()
r.run(subs)
print("wall ms", (time.perf_counter() - t0) * 1e3)
with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
    r.run(subs)
    torch.cuda.synchronize()
ev = [e for e in prof.events() if e.device_type.name == "CUDA"]
t_min = min(e.time_range.start for e in ev)
rows = sorted(((e.time_range.start - t_min) / 1e3, (e.time_range.end - t_min) / 1e3, e.name[:60]) for e in ev)
for s, e, name in rows:
    if e - s > 0.05 or "Memcpy" in name or "Memset" in name:
        print(f"{s:8.2f} {e:8.2f} {e - s:7.2f}  {name}")
