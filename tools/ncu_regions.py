"""Instructions per code region (by source-line markers) of one kernel in an
ncu source page (cuda,sass).  Usage:
  python tools/ncu_regions.py x.csv DIV 'name1:marker text' 'name2:marker text' ...
Regions run from the first line containing each marker to the next marker."""
import csv
import sys

path, div = sys.argv[1], float(sys.argv[2])
marks = [a.split(":", 1) for a in sys.argv[3:]]
rows = list(csv.reader(open(path)))
hdr = next(r for r in rows if r and r[0] == "Line No")
ie = hdr.index("Instructions Executed")
ad = hdr.index("Address")
src = {}
fname = ""
for r in rows:
    if r and r[0] in ("File Path", "File Name"):
        fname = r[1]
        continue
    if len(r) <= ie or not r[0].isdigit():
        continue
    key = (fname.rsplit("/", 1)[-1], int(r[0]))
    try:
        src[key] = (int(r[ie] or 0) if r[ie] not in ("-", "") else 0, r[1])
    except ValueError:  # source text with unbalanced quotes
        continue
kern = sorted(k for k in src if k[0] == "sigmo_kernels.cu")
pos = []
for name, txt in marks:
    ln = next((k[1] for k in kern if txt in src[k][1]), None)
    if ln is None:
        print("marker not found:", txt)
        sys.exit(1)
    pos.append((ln, name))
pos.sort()
res = {}
tot = sum(v[0] for v in src.values())
for (f, ln), (n, _) in src.items():
    name = "other files" if f != "sigmo_kernels.cu" else "before first marker"
    if f == "sigmo_kernels.cu":
        for p, nm in pos:
            if ln >= p:
                name = nm
    res[name] = res.get(name, 0) + n
for k, v in sorted(res.items(), key=lambda x: -x[1]):
    print(f"{k:24s} {100 * v / tot:5.1f}%  {v / div:10.0f}")
print(f"{'total':24s} {100:5.1f}%  {tot / div:10.0f}")
