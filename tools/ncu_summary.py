"""Summarise an ncu --set full report (per kernel) into markdown lines.
Usage: python tools/ncu_summary.py report.ncu-rep [more.ncu-rep ...]"""
import csv
import io
import subprocess
import sys

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occupancy % (achieved)"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads per warp-instruction (warp exec eff x32)"),
    ("smsp__inst_executed.sum", "warp-instructions executed"),
    ("sm__inst_executed.avg.per_cycle_active", "IPC (per SM, active)"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__shared_mem_per_block_dynamic", "dyn smem/block"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def main():
    for rep in sys.argv[1:]:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(out)))
        hdr, units = rows[0], rows[1]
        print(f"### {rep}\n")
        print("| kernel | " + " | ".join(n for _, n in METRICS) + " |")
        print("|---|" + "---|" * len(METRICS))
        for r in rows[2:]:
            name = r[hdr.index("Kernel Name")].split("(")[0]
            vals = []
            for m, _ in METRICS:
                if m in hdr:
                    i = hdr.index(m)
                    vals.append(f"{r[i]} {units[i]}".strip())
                else:
                    vals.append("n/a")
            print(f"| {name} | " + " | ".join(vals) + " |")
        print()


if __name__ == "__main__":
    main()
