"""Per-CUDA-line hotspots from an ncu source page.
Usage: ncu -i rep --page source --csv --kernel-name regex:K --launch-count 1 --print-source cuda,sass > x.csv
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
has_addr = "Address" in hdr
lines = []
fname = ""
for r in rows:
    if r and r[0] in ("File Path", "File Name"):
        fname = r[1].rsplit("/", 1)[-1]
        continue
    if len(r) <= tie or not r[0] or not r[0].isdigit():
        continue
    if has_addr and r[hdr.index("Address")] not in ("-", ""):
        continue
    try:
        lines.append((int(r[ie] or 0), int(r[ws] or 0), int(r[tie] or 0), fname + ":" + r[0], r[1].strip()[:100]))
    except ValueError:
        pass
ti = sum(x[0] for x in lines)
ts = sum(x[1] for x in lines)
print(f"total warp-instructions {ti:,}  stall samples {ts:,}")
for n, s, tn, ln, src in sorted(lines, reverse=True)[:top]:
    print(f"{100*n/max(ti,1):5.1f}% inst {100*s/max(ts,1):5.1f}% stall  thr/warp {tn/max(n,1):4.1f}  L{ln}: {src}")
