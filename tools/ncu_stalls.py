"""Per-instruction stall samples from an ncu source page exported with
--page source --csv --print-source sass: total stall reasons and the top
instructions.  Usage: python tools/ncu_stalls.py src.csv [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top_n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
h = next(r for r in rows if "Address" in r)
data = [r for r in rows[rows.index(h) + 1:] if len(r) == len(h) and r[0].startswith("0x")]
num = lambda r, c: int(r[h.index(c)] or 0)
iS, iE, iSrc = "Warp Stall Sampling (All Samples)", "Instructions Executed", "Source"
stalls = [c for c in h if c.startswith("stall_")]
tot = sum(num(r, iS) for r in data)
print("samples", tot, "instructions", sum(num(r, iE) for r in data))
agg = {c: sum(num(r, c) for r in data) for c in stalls}
print(" ".join(f"{c[6:]}={v / tot:.1%}" for v, c in sorted(((v, c) for c, v in agg.items()), reverse=True)[:10]))
for r in sorted(sorted(data, key=lambda r: -num(r, iS))[:top_n], key=lambda r: int(r[0], 16)):
    st = sorted(((num(r, c), c[6:]) for c in stalls), reverse=True)[:2]
    print(r[0][-5:], f"{num(r, iS):6d} {num(r, iE) / 1e6:6.1f}M", r[h.index(iSrc)].strip()[:58], st)
