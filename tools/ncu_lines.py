"""Instruction share per line range of sigmo_kernels.cu from an ncu source csv.
Usage: python tools/ncu_lines.py x.csv name:a-b name:a-b ..."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = next(r for r in rows if r and r[0] == "Line No")
ie, ad = hdr.index("Instructions Executed"), hdr.index("Address")
fname, src = "", {}
for r in rows:
    if r and r[0] in ("File Path", "File Name"):
        fname = r[1].rsplit("/", 1)[-1]
        continue
    if len(r) <= ie or not r[0].isdigit() or r[ad] not in ("-", ""):
        continue
    try:
        src[(fname, int(r[0]))] = int(r[ie] or 0)
    except ValueError:
        pass
tot = sum(src.values())
regs = [(n, *map(int, ab.split("-"))) for n, ab in (a.split(":") for a in sys.argv[2:])]
res = {}
for (f, ln), v in src.items():
    name = "other:" + f
    if f == "sigmo_kernels.cu":
        name = "other kernels.cu"
        for n, a, b in regs:
            if a <= ln <= b:
                name = n
    res[name] = res.get(name, 0) + v
for k, v in sorted(res.items(), key=lambda x: -x[1]):
    print(f"{k:24s} {100 * v / tot:5.1f}%")
print("total", tot)
