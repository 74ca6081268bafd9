"""Filter-levels sweep (the E1/E2 analogue of PAPER.md Fig. 5/6):
candidate bits, GMCR pairs and device time of filter / mapping / join per
level, Find All and Find First.  Prints one JSON line per level.
Usage: python tools/sweep_levels.py [molecules] [levels,..] [synth config id (2 = configs[1])]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import synth
import paper_conf_sc_carocfc25_b200 as sigmo


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 100_000
    levels = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [1, 2, 3, 4, 5, 6]
    cid = int(sys.argv[3]) if len(sys.argv) > 3 else 2
    reps = 20 if n <= 200_000 else 5
    torch.cuda.set_device(0)
    Q, D = synth.config_queries(cid), synth.config_data(cid, count=n)
    ctx = sigmo.Context(0)
    ctx.load_batch(Q, D)
    for L in levels:
        row = {"levels": L, "config_id": cid, "molecules": n}
        for mode, name in ((sigmo.SIGMO_FIND_ALL, "all"), (sigmo.SIGMO_FIND_FIRST, "first")):
            ctx.filter(L)
            ctx.join(mode)
            ctx.set_timing(True)
            for _ in range(reps):
                ctx.filter(L)
                ctx.join(mode, total=False)
            t = ctx.timings()
            ctx.set_timing(False)
            row[name] = {"filter_ms": t["filter_ms"], "mapping_ms": t["mapping_ms"], "join_ms": t["join_ms"],
                         "total_ms": t["filter_ms"] + t["mapping_ms"] + t["join_ms"], "result": ctx.join(mode)}
        row["gmcr_pairs"] = ctx.num_pairs()
        if n <= 200_000:
            bm = ctx.candidates()
            row["candidate_bits"] = int(np.unpackbits(bm.view(np.uint8)).sum())
        # the neighbour-support flag (R9) at this level, Find All
        ctx.filter(L, neighbor_support=True)
        ctx.join(sigmo.SIGMO_FIND_ALL)
        ctx.set_timing(True)
        for _ in range(max(reps // 4, 2)):
            ctx.filter(L, neighbor_support=True)
            ctx.join(sigmo.SIGMO_FIND_ALL, total=False)
        t = ctx.timings()
        ctx.set_timing(False)
        row["all_ns"] = {"filter_ms": t["filter_ms"], "mapping_ms": t["mapping_ms"], "join_ms": t["join_ms"],
                         "total_ms": t["filter_ms"] + t["mapping_ms"] + t["join_ms"],
                         "result": ctx.join(sigmo.SIGMO_FIND_ALL), "gmcr_pairs": ctx.num_pairs()}
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
