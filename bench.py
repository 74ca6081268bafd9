#!/usr/bin/env python
"""SIGMo B200 benchmark (driver contract: one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl sigmo|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...      (N > 1)

Workload (N=1): BASELINE.json configs[2] -- the configuration the metric is
quoted on at 1/2/4/8 B200 -- = 100 queries (35 library functional groups +
65 random 3-8-atom subgraphs) x 1M synthetic ZINC-like molecules per GPU,
Find All, filter levels 2 = the best of the configs[1] levels sweep (SURVEY.md
8(d) C3 "L = best from C2"; profiles/r2/levels_sweep_c1.jsonl: Find All
L=1..7 -> 1.14/0.74/0.75/0.77/0.78/0.79/0.79 ms, Find First best at L=2 too,
and the same on configs[2] itself, levels_sweep_c2.jsonl); `--config 1` selects configs[1]
(50 queries x 100k molecules, the levels-sweep / Find First config).  Weak
scaling: rank r owns molecules [r*M, (r+1)*M) of the same counter-based
stream; queries are replicated; the only collective is an NCCL all-reduce of
the per-query totals.

A step = one pass of the hot path over the resident batch: sigmo_filter
(signatures + dominance + bitmap + GMCR) -> sigmo_join(Find All) -> per-query
totals (+ all-reduce).  Each timed step is bracketed by CUDA events on the
ctx stream; L2 (126 MB) is flushed by a 256 MiB write before every step,
outside the events.  value = all matches of all ranks / max-over-ranks time.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

BASELINE_METRIC = "matches/sec (Find All) and graph-pairs/sec (Find First) at 1/2/4/8 B200"
# BASELINE.json configs[i] -> synth config id i+1, molecules per rank.
# configs[3]/[4] are 8-GPU configurations: the per-rank default is the 8-GPU
# share (1M / 8 and 10M / 8), so `--gpus 8` processes the whole config.
CONFIGS = {1: (2, 100_000), 2: (3, 1_000_000), 3: (4, 125_000), 4: (5, 1_250_000)}
E2E_BATCH = 250_000  # molecules per host batch of the e2e measurement (StreamRunner)
STREAM_BATCH = 250_000        # configs[4]: molecules per streamed batch per GPU
LEVELS = 2  # best of the configs[1] sweep (profiles/r2/levels_sweep_c1.jsonl)
CPU_SAMPLE_MOLS = 200_000     # cpu_baseline leg: oracle on the first 200k molecules (~100 core-seconds)
REF_STEP_MOLS = 2_000         # --impl reference: molecules per step


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="sigmo", choices=["sigmo", "reference"])
    ap.add_argument("--levels", type=int, default=LEVELS)
    ap.add_argument("--levels-large", type=int, default=4,
                    help="configs[3]/[4]: levels of the 20-30-atom ring-system query group (general join)")
    ap.add_argument("--config", type=int, default=2, choices=sorted(CONFIGS), help="BASELINE.json configs[i]")
    ap.add_argument("--molecules", type=int, default=None, help="molecules per rank (default: the config's)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--balance", default="atoms", choices=["count", "atoms", "cost"],
                    help="molecule shards at N>1: equal count (the paper's static split), equal atoms (default), "
                         "or equal modelled cost (SURVEY 8(f) N2: a first filter pass feeds sharded.molecule_costs)")
    ap.add_argument("--ns", action="store_true",
                    help="neighbour-support fixed point in the filter (SIGMO_FILTER_NEIGHBOR_SUPPORT; DESIGN.md R9)")
    ap.add_argument("--induced", action="store_true",
                    help="induced-subgraph embeddings (sigmo_set_induced; SURVEY 8(f) N4, DESIGN.md R21)")
    a = ap.parse_args()
    a.cid = CONFIGS[a.config][0]
    if a.molecules is None:
        a.molecules = CONFIGS[a.config][1]
    return a


# ----------------------------------------------------------------------------
# clocks during the timed region (NVML)
# ----------------------------------------------------------------------------
REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
           0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
           0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}


class ClockSampler:
    def __init__(self, cuda_index: int):
        self.samples = []
        self.reasons = 0
        self.max_mhz = None
        self.ok = False
        self._stop = threading.Event()
        try:
            import pynvml
            import torch
            pynvml.nvmlInit()
            self.nv = pynvml
            h = None
            try:
                want = str(torch.cuda.get_device_properties(cuda_index).uuid)
                for i in range(pynvml.nvmlDeviceGetCount()):
                    hi = pynvml.nvmlDeviceGetHandleByIndex(i)
                    u = pynvml.nvmlDeviceGetUUID(hi)
                    u = u.decode() if isinstance(u, bytes) else u
                    if want and want in u:
                        h = hi
                        break
            except Exception:
                h = None
            if h is None:
                vis = os.environ.get("CUDA_VISIBLE_DEVICES")
                idx = int(vis.split(",")[cuda_index]) if vis and vis.split(",")[0].isdigit() else cuda_index
                h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self.h = h
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = repr(e)

    def _reasons(self):
        f = getattr(self.nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
            self.nv.nvmlDeviceGetCurrentClocksThrottleReasons
        return int(f(self.h))

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                self.reasons |= self._reasons()
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml_unavailable"]}
        rs = [n for b, n in REASONS.items() if self.reasons & b and n != "gpu_idle"]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": rs, "samples": len(self.samples)}


# ----------------------------------------------------------------------------
def dist_setup(args):
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if torch.cuda.is_available() and args.impl == "sigmo":
            torch.cuda.set_device(local)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    elif torch.cuda.is_available() and args.impl == "sigmo":
        torch.cuda.set_device(0)
    return world, rank, local


def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def run_cpu_baseline(Q, args):
    """The oracle as it stands, on a bounded sample of the same workload."""
    import oracle
    import synth
    nmol = min(CPU_SAMPLE_MOLS, args.molecules)
    D = synth.config_data(args.cid, first=0, count=nmol)
    th = host_cores()
    im = oracle.INDUCED if getattr(args, "induced", False) else 0
    t0 = time.perf_counter()
    res = oracle.count_dense(Q, D, oracle.FIND_ALL | im, nthreads=th)
    dt = time.perf_counter() - t0
    t1 = time.perf_counter()
    oracle.count_dense(Q, D, oracle.FIND_FIRST | im, nthreads=th)
    dt_ff = time.perf_counter() - t1
    # single-thread rate on a 1 % deterministic subsample (every 100th molecule)
    sub = synth.GraphBatch.from_graphs([D.graph(g) for g in range(0, D.num_graphs, 100)])
    t2 = time.perf_counter()
    r1 = oracle.count_dense(Q, sub, oracle.FIND_ALL | im, nthreads=1)
    dt1 = time.perf_counter() - t2
    return {"value": float(res.sum()) / dt, "unit": "matches/s", "cores": th, "kind": "oracle",
            "single_thread": {"value": float(r1.sum()) / dt1, "unit": "matches/s",
                              "sample": f"every 100th of the {nmol} molecules ({sub.num_graphs}), 1 thread"},
            "sample": f"{Q.num_graphs} queries x first {nmol} molecules of configs[{args.config}] (Find All), "
                      f"{dt:.2f} s wall on {th} threads; {int(res.sum())} matches",
            "find_first_pairs_per_s": Q.num_graphs * D.num_graphs / dt_ff, "cpu_model": cpu_model()}


# ----------------------------------------------------------------------------
def run_reference(args, world, rank):
    """--impl reference: the CPU oracle on the same config/metric (rank 0 only)."""
    if rank != 0:
        return
    import oracle
    import synth
    Q = synth.config_queries(args.cid)
    th = host_cores()
    im = oracle.INDUCED if args.induced else 0
    n_total = args.molecules
    step_mols = min(REF_STEP_MOLS, n_total)

    def batch(i):
        first = (i * step_mols) % max(n_total - step_mols + 1, 1)
        return synth.config_data(args.cid, first=first, count=step_mols)

    for i in range(args.warmup):
        oracle.count_dense(Q, batch(i), oracle.FIND_ALL | im, nthreads=th)
    batches = [batch(args.warmup + i) for i in range(args.steps)]
    matches = 0
    t = 0.0
    for D in batches:
        t0 = time.perf_counter()
        r = oracle.count_dense(Q, D, oracle.FIND_ALL | im, nthreads=th)
        t += time.perf_counter() - t0
        matches += int(r.sum())
    value = matches / t
    line = {"impl": "reference", "metric": BASELINE_METRIC, "value": value, "unit": "matches/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * t / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
            "config": config_dict(args, world, oracle_step=step_mols),
            "cpu_baseline": {"value": value, "unit": "matches/s", "cores": th, "kind": "oracle",
                             "sample": f"{Q.num_graphs} queries x {step_mols} molecules of configs[{args.config}] per step, "
                                       f"{args.steps} steps", "cpu_model": cpu_model()},
            "e2e": {"value": value, "unit": "matches/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def config_dict(args, world, oracle_step=None):
    nq = {2: 50, 3: 100, 4: 500, 5: 1000}[args.cid]
    mode = "Find First" if args.cid == 4 else "Find All"
    extra = f", streamed in batches of {STREAM_BATCH}" if args.cid == 5 else ""
    d = {"workload": f"configs[{args.config}]: {nq} queries x {args.molecules} ZINC-like molecules per GPU, "
                     f"{mode}, levels={args.levels}{extra}",
         "queries": nq, "molecules_per_gpu": args.molecules, "molecules_total": args.molecules * world,
         "levels": args.levels, "mode": "find_first" if args.cid == 4 else "find_all", "data_seed": hex(0x51C0_0000 + args.cid),
         "query_seed": hex(0x9E00_0000 + args.cid),
         "l2": ("flushed before every timed step (256 MiB device write, outside the events)" if args.cid in (2, 3)
                else "no flush: per-step inputs and candidate arrays are larger than the 126 MB L2"),
         "parallelism": f"dp{world}: molecule shards, queries replicated, NCCL all-reduce of per-query totals",
         "shards": getattr(args, "balance", "atoms") if world > 1 else "whole batch"}
    if args.cid in (4, 5):
        d["levels_ring_systems"] = args.levels_large
        d["workload"] += f" (ring-system query group: levels={args.levels_large})"
    if getattr(args, "induced", False):
        d["workload"] += ", induced-subgraph mode (N4)"
        d["induced"] = True
    if oracle_step:
        d["oracle_molecules_per_step"] = oracle_step
    return d


# ----------------------------------------------------------------------------
def main():
    args = parse()
    world, rank, local = dist_setup(args)
    if args.impl == "reference":
        run_reference(args, world, rank)
        return
    if args.cid in (4, 5):
        if args.induced:
            raise SystemExit("--induced applies to configs[0..2] (the routed runs use the lane join)")
        run_routed(args, world, rank, local)
        return
    import numpy as np
    import torch

    import synth
    import paper_conf_sc_carocfc25_b200 as sigmo

    dev = torch.device("cuda", local)
    dist = None
    if world > 1:
        import torch.distributed as dist
    from paper_conf_sc_carocfc25_b200 import sharded
    Q = synth.config_queries(args.cid)
    stream = torch.cuda.current_stream(dev)
    ctx = sigmo.Context(local, stream)
    if args.induced:
        ctx.set_induced(True)
    # this rank's molecules of the world x M stream (weak scaling): contiguous
    # shards balanced by atoms (default), count, or modelled cost (N2)
    M_total = args.molecules * world
    if world > 1:
        sizes = synth.molecule_sizes(synth.DATA_SEED_BASE + args.cid, 0, M_total)
        bounds = sharded.stream_shard_bounds(sizes, world, "count" if args.balance == "count" else "atoms")
        if args.balance == "cost":
            # adaptive (N2): a timed first pass on the atom shards; each rank's
            # device time spread over its molecules by atoms, gathered over
            # ranks, split at equal cost (sharded.measured_costs)
            D0 = synth.config_data(args.cid, first=int(bounds[rank]), count=int(bounds[rank + 1] - bounds[rank]))
            ctx.load_batch(Q, D0)
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            for i in range(2):
                ev0.record(stream)
                ctx.filter(args.levels, neighbor_support=args.ns)
                ctx.join(sigmo.SIGMO_FIND_ALL, total=False)
                ev1.record(stream)
            torch.cuda.synchronize(dev)
            costs = sharded.gather_costs(sharded.measured_costs(D0.graph_offsets, ev0.elapsed_time(ev1)))
            bounds = sharded.stream_shard_bounds(sizes, world, "cost", costs=costs)
            del D0
    else:
        bounds = np.array([0, args.molecules], np.int64)
    D = synth.config_data(args.cid, first=int(bounds[rank]), count=int(bounds[rank + 1] - bounds[rank]))
    ctx.load_batch(Q, D)
    totals = torch.zeros(Q.num_graphs, dtype=torch.int64, device=dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)

    def step(mode=sigmo.SIGMO_FIND_ALL):
        ctx.filter(args.levels, neighbor_support=args.ns)
        ctx.join(mode, total=False)
        ctx.query_totals(device_tensor=totals)
        sharded.allreduce_totals(totals)  # the only collective: NCCL sum of per-query totals

    # ---- warm-up (both join modes: the first launch of a kernel instantiation
    # loads its module, which must not land in a timed step) ----
    for _ in range(max(args.warmup, 3)):
        step()
    step(sigmo.SIGMO_FIND_FIRST)
    torch.cuda.synchronize(dev)

    def timed_loop(mode, K, with_timing):
        ctx.set_timing(with_timing)
        starts = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
        ends = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize(dev)
        for i in range(K):
            if not args.no_flush:
                flush.fill_(i)
            starts[i].record(stream)
            step(mode)
            ends[i].record(stream)
        torch.cuda.synchronize(dev)
        if dist is not None:
            dist.barrier()
        ms = sum(s.elapsed_time(e) for s, e in zip(starts, ends))
        tim = ctx.timings() if with_timing else None
        ctx.set_timing(False)
        return ms, tim

    sampler = ClockSampler(local)
    with sampler:
        ms_all, tim = timed_loop(sigmo.SIGMO_FIND_ALL, args.steps, True)
    clocks = sampler.summary()
    # DFS steps of one Find All join (counted by the join's counting instantiation, outside the timed loop)
    ctx.set_timing(False, count_steps=True)
    matches_local = int(ctx.join(sigmo.SIGMO_FIND_ALL))  # identical every step (deterministic)
    dfs_steps = int(ctx.timings()["dfs_steps"])
    ctx.set_timing(False)
    pairs_local = ctx.num_pairs()
    ms_ff, _ = timed_loop(sigmo.SIGMO_FIND_FIRST, args.steps, False)
    positive_local = int(ctx.join(sigmo.SIGMO_FIND_FIRST))

    # ---- e2e through the public API from host buffers ----
    # the inputs sit in page-locked host memory as a loader feeding the GPU holds
    # them: the step's molecules in batches of E2E_BATCH, run by the double-buffered
    # StreamRunner (stream.py; each batch's host-to-device copy overlaps the previous
    # batch's filter + join); the copies and the D2H of the per-query totals are
    # inside the timed region
    from paper_conf_sc_carocfc25_b200.stream import StreamRunner
    n_local = D.num_graphs
    nb_e2e = max(1, (n_local + E2E_BATCH - 1) // E2E_BATCH)
    parts = [D.slice(i * n_local // nb_e2e, (i + 1) * n_local // nb_e2e) for i in range(nb_e2e)]
    h2d = sum(p.nbytes() for p in parts) + nb_e2e * Q.nbytes()  # every batch also loads the (small) queries
    subs = [sigmo.as_c_batch(p, pinned=True) for p in parts]
    del parts
    runner = StreamRunner(Q, local, levels=args.levels, mode=sigmo.SIGMO_FIND_ALL, split=False,
                          induced=args.induced, neighbor_support=args.ns)
    e2e_ms = []
    for i in range(args.e2e_steps + 1):
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        tot = runner.run(subs)  # D2H of the per-query totals
        dt = (time.perf_counter() - t0) * 1000
        if i > 0:
            e2e_ms.append(dt)
        assert int(tot.sum()) == matches_local
    runner.close()

    # ---- reduce over ranks (sharded.rank_reduce: times MAX, counts SUM) ----
    ctx.check()  # the device-pointer totals path never synchronized: check the join's capacities once
    (ms_all, ms_ff, e2e_total), (matches, pairs, positive, all_pairs) = sharded.rank_reduce(
        [ms_all, ms_ff, sum(e2e_ms)], [matches_local, pairs_local, positive_local, Q.num_graphs * D.num_graphs], dev)
    if rank != 0:
        ctx.close()
        if dist is not None:
            dist.destroy_process_group()
        return

    K = args.steps
    value = sharded.throughput(matches, K, ms_all)
    ms_per_step = ms_all / K
    # ---- roofline of the dominant kernel (per-launch CUDA events over the timed region) ----
    import json as _json

    def _load(rel):
        try:
            return _json.load(open(os.path.join(ROOT, rel)))
        except Exception:
            return {}

    peaks = _load("MEASURED_PEAKS.json")
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = "measured (MEASURED_PEAKS.json hbm_gbs)" if "hbm_gbs" in peaks else "fallback 6.65 TB/s"
    # ncu --set full of the same kernels at the bench's levels (profiles/r2/ncu_traffic.json, tools/ncu_traffic.py):
    # DRAM bytes per launch and instruction counts; cold-cache and serialised, so only shares/ratios are used
    ncu = _load("profiles/r2/ncu_traffic.json")
    # the capture is of the default workload only (configs[2], 1M molecules, monomorphic, no neighbour support)
    same = (ncu.get("levels") == args.levels and ncu.get("workload") == f"configs[{args.config}]"
            and args.molecules == 1_000_000 and not args.induced and not args.ns)
    nk = ncu.get("kernels", {}) if same else {}
    VQ, VD, ND, NQ = Q.num_nodes, D.num_nodes, D.num_graphs, Q.num_graphs
    W = (VD + 31) // 32
    # the method must produce C_L -- VQ x VD bits written once -- plus the GMCR bits / counts,
    # reading the packed CSR-GO once (the kernel writes the distinct-row windows instead: fewer DRAM bytes)
    filter_bytes = (4 * VQ * W                       # bitmap written once
                    + 4 * ND * ((NQ + 31) // 32) + 16 * ND  # GMCR bits + counts
                    + 4 * (ND + 1) + 2 * VD + 4 * (VD + 1) + 2 * D.num_adj)  # packed CSR-GO read once
    f_ms, j_ms, m_ms = tim["filter_ms"], tim["join_ms"], tim["mapping_ms"]
    fk = nk.get("sigmo_filter_lane_jit", {})
    f_dram = fk.get("dram_bytes")
    filter_roof = {"bound": "hbm", "achieved": filter_bytes / (f_ms * 1e-3) / 1e9, "peak": hbm_peak,
                   "unit": "GB/s", "frac": filter_bytes / (f_ms * 1e-3) / 1e9 / hbm_peak, "traffic": f_dram,
                   "kernel": "sigmo_filter_lane_jit" if tim.get("filter_jit") else "k_filter_lane", "ms": f_ms,
                   "algorithmic_bytes": filter_bytes, "peak_source": peak_src,
                   "algorithmic_bytes_model": "SURVEY 8(d): VQ*VD/8 candidate bits + GMCR bits/counts + packed CSR-GO",
                   "frac_dram": (f_dram / (f_ms * 1e-3) / 1e9 / hbm_peak) if f_dram else None,
                   "frac_dram_note": "ncu DRAM bytes of one launch (distinct-row windows, profiles/r2/ncu_traffic.json) "
                                     "/ this run's kernel time / peak"}
    # join: integer-issue bound.  Peak = the measured mixed LOP3 + IMAD rate of this
    # B200 model (tools/microbench/int_peak.cu -> profiles/r2/int_peak.json: 122 lanes/SM/clk) at the run's
    # clock; algorithmic work = DFS steps x 12 lane-ops (the minimum a step needs); the measured cost per
    # step (thread-instructions) comes from the ncu capture
    sm_mhz = float(clocks.get("sm_mhz") or peaks.get("sm_max_mhz", 1965.0))
    ip = _load("profiles/r2/int_peak.json")
    lanes = float(ip.get("mixed_lanes_per_sm_per_clk", 128.0))
    steps = dfs_steps
    alu_peak = 148 * lanes * sm_mhz * 1e6 / 1e12
    join_ach = 12.0 * steps / (j_ms * 1e-3) / 1e12 if j_ms > 0 else 0.0
    jn, jw = nk.get("k_join_lane_narrow", {}), nk.get("k_join_lane_wide", {})
    thr_instr = sum(k.get("warp_instructions", 0) * k.get("threads_per_instruction", 0) for k in (jn, jw))
    join_roof = {"bound": "alu", "achieved": join_ach, "peak": alu_peak, "unit": "Tops/s", "frac": join_ach / alu_peak,
                 "traffic": (jn.get("dram_bytes", 0) + jw.get("dram_bytes", 0)) or None,
                 "kernel": "k_join_lane", "ms": j_ms, "dfs_steps_per_launch": steps, "ops_per_step": 12,
                 "peak_source": f"measured: 148 SM x {lanes:.1f} int lanes/clk (mixed LOP3+IMAD, profiles/r2/"
                                f"int_peak.json) x {sm_mhz:.0f} MHz (this run's clock)",
                 "thread_instructions_per_step": (thr_instr / steps) if (steps and thr_instr) else None,
                 "l1_global_sectors_per_step": (sum(k.get("l1_global_ld_sectors", 0) for k in (jn, jw)) / steps)
                 if (steps and jn) else None,
                 "l1_shared_wavefronts_per_step": (sum(k.get("l1_shared_wavefronts", 0) for k in (jn, jw)) / steps)
                 if (steps and jn) else None,
                 "l1_data_pipe_pct_narrow": jn.get("l1_data_pipe_pct"),
                 "issue_utilization": (jn.get("ipc", 0) / 4.0) if jn else None,
                 "pairs_per_launch": pairs_local, "matches_per_launch": matches_local}
    dominant = "join" if j_ms >= f_ms else "filter"
    roofline = dict(join_roof) if dominant == "join" else dict(filter_roof)

    line = {
        "metric": BASELINE_METRIC, "value": value, "unit": "matches/s", "n_gpus": world, "steps": K,
        "warmup": max(args.warmup, 3), "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": config_dict(args, world),
        "find_first": {"value": all_pairs * K / (ms_ff / 1000.0), "unit": "graph-pairs/s",
                       "positive_pairs_per_s": positive * K / (ms_ff / 1000.0), "ms_per_step": ms_ff / K},
        "counts": {"matches": matches, "gmcr_pairs": pairs, "positive_pairs": positive, "all_pairs": all_pairs},
        "stage_ms": {"filter": f_ms, "mapping": m_ms, "join": j_ms},
        "roofline_filter": filter_roof,
        "roofline_join": join_roof,
        "dominant_kernel": dominant,
        "e2e": {"value": matches * args.e2e_steps / (e2e_total / 1000.0), "unit": "matches/s",
                "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": 8 * NQ,
                "ms_per_step": e2e_total / args.e2e_steps,
                "batches_per_step": nb_e2e,
                "note": f"StreamRunner.run over the step's molecules in {nb_e2e} pinned host batches: per batch "
                        "sigmo_load_batch (H2D of the raw CSR-GO arrays, validation + packing on the device) + "
                        "filter + join on one of two double-buffered contexts (the next batch's copy overlaps), "
                        "then the D2H of the per-query totals; wall clock"},
        "gpu_launches": int(K * (tim["filter_launches"] + tim["join_launches"])),
        "clocks": clocks,
        "roofline": roofline,
    }
    if world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = run_cpu_baseline(Q, args)
    print(json.dumps(line), flush=True)
    ctx.close()
    if dist is not None:
        dist.destroy_process_group()


def run_routed(args, world, rank, local):
    """configs[3] (500 queries incl. 20-30-atom ring systems, Find First) and
    configs[4] (1,000 queries, Find All, batches of 250k streamed through two
    double-buffered contexts): queries routed by size (stream.split_queries).
    configs[3]: data resident, a step = filter + join of both query groups,
    device-timed.  configs[4]: a step = the whole stream (host pack + H2D of
    every batch overlapped with the kernels of the previous one), wall clock
    between device synchronisations."""
    import numpy as np
    import torch

    import synth
    import paper_conf_sc_carocfc25_b200 as sigmo
    from paper_conf_sc_carocfc25_b200 import sharded, stream

    dev = torch.device("cuda", local)
    dist = None
    if world > 1:
        import torch.distributed as dist
    Q = synth.config_queries(args.cid)
    first = rank * args.molecules
    ff = args.cid == 4
    mode = sigmo.SIGMO_FIND_FIRST if ff else sigmo.SIGMO_FIND_ALL
    if args.cid == 5:
        nb = (args.molecules + STREAM_BATCH - 1) // STREAM_BATCH
        batches = [sigmo.as_c_batch(synth.config_data(5, first=first + i * STREAM_BATCH,
                                                      count=min(STREAM_BATCH, args.molecules - i * STREAM_BATCH)))
                   for i in range(nb)]
    else:
        batches = [sigmo.as_c_batch(synth.config_data(4, first=first, count=args.molecules))]
    sr = stream.StreamRunner(Q, local, levels=args.levels, mode=mode, levels_large=args.levels_large)
    totals_dev = torch.zeros(Q.num_graphs, dtype=torch.int64, device=dev)
    if args.cid == 4:
        for gi, (_, qb) in enumerate(sr.groups):
            sr.ctx[0][gi].load_batch(qb, batches[0])

    def step():
        if args.cid == 5:
            t = sr.run(batches)
        else:
            with torch.cuda.stream(sr.streams[0]):
                for gi, c in enumerate(sr.ctx[0]):
                    c.filter(sr.group_levels(gi))
                    c.join(mode, total=False)
            t = None
        return t

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize(dev)
    K = args.steps
    if args.cid == 4:  # per-group stage times (the ring-system group runs the general k_join)
        for c in sr.ctx[0]:
            c.set_timing(True)
    sampler = ClockSampler(local)
    if dist is not None:
        dist.barrier()
    torch.cuda.synchronize(dev)
    with sampler:
        if args.cid == 5:
            t0 = time.perf_counter()
            for _ in range(K):
                t = step()
            torch.cuda.synchronize(dev)
            ms = (time.perf_counter() - t0) * 1000
        else:
            s = sr.streams[0]
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(K):
                step()
            e1.record(s)
            torch.cuda.synchronize(dev)
            ms = e0.elapsed_time(e1)
    clocks = sampler.summary()
    if args.cid == 5:
        local_tot = sr.run(batches)
    else:
        local_tot = np.zeros(Q.num_graphs, np.uint64)
        for gi, (idx, _) in enumerate(sr.groups):
            c = sr.ctx[0][gi]
            c.join(mode, total=False)
            local_tot[idx] = c.query_totals()
    totals_dev.copy_(torch.from_numpy(local_tot.astype(np.int64)))
    sharded.allreduce_totals(totals_dev)
    nd_local = sum(b.num_graphs for b in batches)
    vals = torch.tensor([ms], dtype=torch.float64, device=dev)
    cnts = torch.tensor([nd_local], dtype=torch.int64, device=dev)
    if dist is not None:
        dist.all_reduce(vals, op=dist.ReduceOp.MAX)
        dist.all_reduce(cnts)
    ms = float(vals.item())
    nd_all = int(cnts.item())
    total = int(totals_dev.sum().item())
    if rank == 0:
        if ff:
            value, unit = Q.num_graphs * nd_all * K / (ms / 1000.0), "graph-pairs/s"
        else:
            value, unit = total * K / (ms / 1000.0), "matches/s"
        tims = [c.timings() for c in sr.ctx[0]]
        launches = sum(t["filter_launches"] + t["join_launches"] for t in tims)
        line = {
            "metric": BASELINE_METRIC, "value": value, "unit": unit, "n_gpus": world, "steps": K,
            "warmup": max(args.warmup, 3), "ms_per_step": ms / K, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u64", "data": "synthetic", "config": config_dict(args, world),
            "counts": {"matches" if not ff else "positive_pairs": total, "all_pairs": Q.num_graphs * nd_all},
            "query_groups": [int(len(g)) for g, _ in sr.groups],
            "group_stage_ms": ([{"queries": int(len(g)), "join_kernel": "k_join_lane" if len(g) and gi == 0 else "k_join",
                                 "filter": t["filter_ms"], "mapping": t["mapping_ms"], "join": t["join_ms"]}
                                for gi, ((g, _), t) in enumerate(zip(sr.groups, tims))] if args.cid == 4 else None),
            "timing": "wall clock incl. host pack + H2D of every batch" if args.cid == 5 else "device events",
            "gpu_launches": int(K * launches * (len(batches) if args.cid == 5 else 1)),
            "clocks": clocks,
        }
        print(json.dumps(line), flush=True)
    sr.close()
    if dist is not None:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
