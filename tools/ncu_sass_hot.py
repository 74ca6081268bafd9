"""Hot SASS instructions (with their CUDA line) from an ncu source page
exported with --print-source cuda,sass.
Usage: python tools/ncu_sass_hot.py x.csv [min_millions] [first_line last_line]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
thr = float(sys.argv[2]) * 1e6 if len(sys.argv) > 2 else 2e6
lo, hi = (int(sys.argv[3]), int(sys.argv[4])) if len(sys.argv) > 4 else (0, 10 ** 9)
hdr = None
cur = (0, "")
out = []
for r in rows:
    if r and r[0] == "Line No":
        hdr = r
        ie = hdr.index("Instructions Executed")
        continue
    if not hdr or len(r) < 4:
        continue
    if r[0].isdigit() and r[2] in ("", "-"):
        cur = (int(r[0]), r[1].strip())
        continue
    if r[2].startswith("0x"):
        try:
            n = int(r[ie] or 0)
        except ValueError:
            n = 0
        out.append((cur[0], r[2][-5:], n, r[3].strip(), cur[1]))
tot = sum(x[2] for x in out)
print("total", tot)
for ln, a, n, s, src in out:
    if n >= thr and lo <= ln <= hi:
        print(f"{ln:5d} {a} {n / 1e6:8.1f}M  {s[:60]:60s} | {src[:50]}")
