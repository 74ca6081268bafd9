"""Per-SASS execution counts for a source-line range of an ncu source page
(cuda,sass).  Usage: python tools/ncu_sass_lines.py x.csv L0 L1 [divisor] [min]"""
import csv
import sys

path, l0, l1 = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
div = float(sys.argv[4]) if len(sys.argv) > 4 else 1.0
mn = float(sys.argv[5]) if len(sys.argv) > 5 else 0.0
rows = list(csv.reader(open(path)))
hdr = next(r for r in rows if r and r[0] == "Line No")
i0 = rows.index(hdr) + 1
ie = hdr.index("Instructions Executed")
ad = hdr.index("Address")
cur = None
out = []
fname = ""
for r in rows:
    if r and r[0] in ("File Path", "File Name"):
        fname = r[1]
        continue
    if len(r) <= ie or not fname.endswith("sigmo_kernels.cu"):
        continue
    if r[0]:
        if not r[0].isdigit():
            continue
        cur = int(r[0])
        continue
    if cur is None or not (l0 <= cur <= l1) or not r[ad].startswith("0x"):
        continue
    try:
        n = int(r[ie])
    except ValueError:
        continue
    if n / div >= mn:
        out.append((int(r[ad], 16), n, cur, r[3].strip()))
out.sort()
tot = 0
for a, n, l, s in out:
    tot += n
    print(f"{n / div:9.1f} L{l} {s}")
print(f"total {tot / div:.1f}")
