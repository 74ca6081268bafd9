"""compute-sanitizer driver (SURVEY.md section 4 / 7 acceptance check 5):
runs every device kernel of the hot path on small seeded batches so that
memcheck, racecheck and synccheck see each of them once:

  * k_filter molecule tiles (lane path) and dense tiles (neighbour-support
    flag), k_support, k_query_prep, k_sig_counts, k_adjb, k_pairs, k_chunks,
    the CUB scan;
  * k_join_lane narrow (<= 32-atom) and wide (33-64-atom) launches, Find All,
    Find First, induced mode;
  * the general k_join (> 64-atom molecules and ring-system queries), Find All,
    Find First, induced mode.

Results are not checked here (the parity tests do that); the process exits
non-zero only if a call fails.  Usage (under gpurun):
    compute-sanitizer --tool memcheck python tools/sanitize_cases.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth
import paper_conf_sc_carocfc25_b200 as sigmo

torch.cuda.set_device(0)
which = sys.argv[1] if len(sys.argv) > 1 else "all"

Q1, D1 = synth.config_queries(1), synth.config_data(1)          # configs[0]: 10 x 200, lane path
_mols = synth.molecules(synth.DATA_SEED_BASE + 77, 0, 40, mode=2).graphs()  # ring-rich
# plus > 64-atom graphs (multi-word masks): an 80-atom chain and a 70-ring
_mols += [([6] * 80, [(i, i + 1, 1) for i in range(79)]), ([6] * 70, [(i, (i + 1) % 70, 1) for i in range(70)])]
big = synth.GraphBatch.from_graphs(_mols)
Qring = synth.config_queries(4)                                   # includes 20-30-atom ring systems
Qring = synth.GraphBatch.from_graphs(Qring.graphs()[-4:] + Q1.graphs()[:4])

cases = []
if which in ("all", "lane"):
    cases.append(("lane", Q1, D1, False))
if which in ("all", "general"):
    cases.append(("general", Qring, big, False))
if which in ("all", "induced"):
    cases.append(("lane-induced", Q1, D1, True))
    cases.append(("general-induced", Qring, big, True))

for name, Q, D, induced in cases:
    with sigmo.Context(0) as ctx:
        ctx.set_induced(induced)
        ctx.load_batch(Q, D)
        for levels in (1, 4):
            for ns in (False, True):
                if induced and ns:
                    continue
                ctx.filter(levels, neighbor_support=ns)
                a = ctx.join(sigmo.SIGMO_FIND_ALL)
                f = ctx.join(sigmo.SIGMO_FIND_FIRST)
                ctx.pair_results()
                ctx.candidates()
                print(f"{name} L={levels} ns={int(ns)}: matches {a}, positive pairs {f}", flush=True)
        ctx.signatures(1, 2)
torch.cuda.synchronize()
print("sanitize cases done")
