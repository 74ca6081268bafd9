"""Per-CUDA-line hotspots from an ncu source page.
Usage: ncu -i rep --page source --csv --kernel-name regex:K --print-source cuda,sass > x.csv
       python tools/ncu_hotspots.py x.csv [topN]"""
import csv
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
rows = list(csv.reader(open(path)))
hdr = next(r for r in rows if r and r[0] == "Line No")
start = rows.index(hdr) + 1
ie = hdr.index("Instructions Executed")
ws = hdr.index("Warp Stall Sampling (All Samples)")
tie = hdr.index("Thread Instructions Executed")
lines = []
for r in rows[start:]:
    if r and r[0] and len(r) > tie:
        try:
            lines.append((int(r[ws] or 0), int(r[ie] or 0), int(r[tie] or 0), r[0], r[1].strip()[:100]))
        except ValueError:
            pass
ts = sum(x[0] for x in lines)
ti = sum(x[1] for x in lines)
print(f"total warp-instructions {ti:,}  stall samples {ts:,}")
for s, n, tn, ln, src in sorted(lines, reverse=True)[:top]:
    eff = tn / max(n, 1)
    print(f"{100*s/max(ts,1):5.1f}% stall {100*n/max(ti,1):5.1f}% inst  thr/warp {eff:4.1f}  L{ln}: {src}")
