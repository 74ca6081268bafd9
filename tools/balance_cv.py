"""N2 evidence on one GPU (the paper's
static equal-molecule split leaves a 4-8 % runtime CV across GPUs).

Emulates configs[2] at 8 GPUs (8 x 1M molecules of the same stream): for each
split -- equal count (the paper's static split), equal atoms (bench.py's
default) and equal modelled cost (N2) -- times the 8 per-rank shares one
after another on this GPU (device time of filter + join, median of 3 steps)
and reports the coefficient of variation and max/mean (the job waits for the
slowest rank).  The cost model's pair weight is calibrated first by least
squares of share time on (atoms, GMCR pairs) over the count and atom splits.
Usage: python tools/balance_cv.py [world] [molecules_per_rank] > out.json"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_sc_carocfc25_b200 as sigmo
from paper_conf_sc_carocfc25_b200 import sharded

world = int(sys.argv[1]) if len(sys.argv) > 1 else 8
M = int(sys.argv[2]) if len(sys.argv) > 2 else 1_000_000
# --skewed: a heterogeneous stream -- every 4th block of 50k molecules comes
# from the ring-rich generator mode (larger molecules, more matches), a
# stand-in for real libraries whose composition drifts along the file
SKEW = "--skewed" in sys.argv
BLOCK = next((int(a.split("=")[1]) for a in sys.argv if a.startswith("--block=")), 50_000)
cid, L = 3, 4
torch.cuda.set_device(0)
Q = synth.config_queries(cid)
seed = synth.DATA_SEED_BASE + cid


def mode_of_block(k):
    return 1 if SKEW and k % 4 == 3 else 0


def stream_sizes(n):
    if not SKEW:
        return synth.molecule_sizes(seed, 0, n)
    return np.concatenate([synth.molecule_sizes(seed, k * BLOCK, min(BLOCK, n - k * BLOCK), mode=mode_of_block(k))
                           for k in range((n + BLOCK - 1) // BLOCK)])


def stream_data(g0, g1):
    if not SKEW:
        return synth.config_data(cid, first=g0, count=g1 - g0)
    parts = []
    k = g0 // BLOCK
    while k * BLOCK < g1:
        a, b = max(g0, k * BLOCK), min(g1, (k + 1) * BLOCK)
        parts.append(synth.molecules(seed, a, b - a, mode=mode_of_block(k)))
        k += 1
    return synth.GraphBatch.concat(parts)


sizes = stream_sizes(world * M)
ctx = sigmo.Context(0)
st = torch.cuda.current_stream()


def time_share(b0, b1):
    D = stream_data(int(b0), int(b1))
    ctx.load_batch(Q, D)
    ts = []
    for i in range(4):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(st)
        ctx.filter(L)
        ctx.join(sigmo.SIGMO_FIND_ALL, total=False)
        e.record(st)
        torch.cuda.synchronize()
        if i:
            ts.append(s.elapsed_time(e))
    di = ctx.pair_results()[0]
    return statistics.median(ts), D.num_nodes, len(di), D.graph_offsets.copy(), di


def summarize(ms):
    m = statistics.mean(ms)
    return {"ms": ms, "mean_ms": m, "cv": statistics.pstdev(ms) / m, "max_over_mean": max(ms) / m}


out = {"workload": f"configs[2] x {world} ranks ({M} molecules per rank), L={L}, Find All, shares timed one after "
                   f"another on one B200 (device time of filter + mapping + join, median of 3)"
                   + (f", skewed stream: every 4th block of {BLOCK} molecules ring-rich (synth mode 1)" if SKEW else ""),
       "splits": {}}
rows = []
costs_atoms = None
for bal in ("count", "atoms"):
    b = sharded.stream_shard_bounds(sizes, world, bal)
    ms, pcs = [], []
    for r in range(world):
        t, atoms, npairs, goff, di = time_share(b[r], b[r + 1])
        ms.append(t)
        rows.append((atoms, npairs, t))
        pcs.append((goff, di))
    out["splits"][bal] = summarize(ms) | {"bounds": b.tolist()}
    if bal == "atoms":
        atom_pairs = pcs
# calibrate ms = a * atoms + c * pairs (least squares, no intercept)
A = np.array([[r[0], r[1]] for r in rows], np.float64)
y = np.array([r[2] for r in rows], np.float64)
from scipy.optimize import nnls
(a, c), _ = nnls(A, y)  # non-negative: atoms and pairs are collinear across shards
w_pair = float(c / a) if a > 0 else 4.0
out["cost_model"] = {"ms_per_atom": float(a), "ms_per_pair": float(c), "w_pair": w_pair,
                     "fit": "non-negative least squares of share time on (atoms, GMCR pairs) over the count and atom splits"}
costs = np.concatenate([sharded.molecule_costs(g, di, w_atom=1.0, w_pair=w_pair) for g, di in atom_pairs])
b = sharded.stream_shard_bounds(sizes, world, "cost", costs=costs)
ms = [time_share(b[r], b[r + 1])[0] for r in range(world)]
out["splits"]["cost_model"] = summarize(ms) | {"bounds": b.tolist()}
# feedback: the atom split's measured per-share times spread over its molecules
atom_ms = out["splits"]["atoms"]["ms"]
costs = np.concatenate([sharded.measured_costs(g, t) for (g, _), t in zip(atom_pairs, atom_ms)])
b = sharded.stream_shard_bounds(sizes, world, "cost", costs=costs)
ms = [time_share(b[r], b[r + 1])[0] for r in range(world)]
out["splits"]["cost_measured"] = summarize(ms) | {"bounds": b.tolist()}
ctx.close()
print(json.dumps(out))
