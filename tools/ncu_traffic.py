"""Per-kernel evidence from an ncu --set full report -> JSON (bench.py reads
it for roofline.traffic and the join's instruction counts).
Usage: python tools/ncu_traffic.py report.ncu-rep levels > profiles/r2/ncu_traffic.json"""
import csv
import io
import json
import re
import subprocess
import sys

rep, levels = sys.argv[1], int(sys.argv[2])
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, units = rows[0], rows[1]


def val(r, k):
    i = hdr.index(k)
    x = float(r[i].replace(",", ""))
    u = units[i]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-6, "us": 1e-3, "ms": 1.0, "usecond": 1e-3,
             "msecond": 1.0, "nsecond": 1e-6}.get(u, 1)
    return x * scale


res = {"source": rep.rsplit("/", 1)[-1], "levels": levels, "workload": "configs[2]", "kernels": {}}
for r in rows[2:]:
    name = r[hdr.index("Kernel Name")]
    # <MODE, W64, PS>: Find All launches (MODE 0, or 8 = the lean instantiation), narrow / wide masks
    m = re.search(r"k_join_lane<(?:0|8), (\d)", name)
    key = "sigmo_filter_lane_jit" if "filter_lane" in name else (
        ("k_join_lane_wide" if m.group(1) == "1" else "k_join_lane_narrow") if m else name)
    res["kernels"][key] = {
        "ms": val(r, "gpu__time_duration.sum"),
        "dram_bytes": val(r, "dram__bytes_read.sum") + val(r, "dram__bytes_write.sum"),
        "dram_read_bytes": val(r, "dram__bytes_read.sum"), "dram_write_bytes": val(r, "dram__bytes_write.sum"),
        "warp_instructions": val(r, "smsp__inst_executed.sum"),
        "threads_per_instruction": val(r, "smsp__thread_inst_executed_per_inst_executed.ratio"),
        "ipc": val(r, "sm__inst_executed.avg.per_cycle_active"),
        "occupancy_pct": val(r, "sm__warps_active.avg.pct_of_peak_sustained_active"),
        "l2_hit_pct": val(r, "lts__t_sector_hit_rate.pct"),
        "l1_global_ld_sectors": val(r, "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"),
        "l1_global_ld_hit_pct": val(r, "l1tex__t_sector_pipe_lsu_mem_global_op_ld_hit_rate.pct"),
        "l1_shared_wavefronts": val(r, "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
        "l1_data_pipe_pct": val(r, "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed"),
    }
print(json.dumps(res, indent=1))
