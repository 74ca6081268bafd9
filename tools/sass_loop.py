"""Print the SASS of one kernel between two addresses (compact), for
instruction counting of the join loop.
Usage: python tools/sass_loop.py lib.so mangled_name [from_hex to_hex]"""
import re
import subprocess
import sys

out = subprocess.run(["cuobjdump", "-sass", "-fun", sys.argv[2], sys.argv[1]], capture_output=True, text=True).stdout
lo, hi = (int(sys.argv[3], 16), int(sys.argv[4], 16)) if len(sys.argv) > 4 else (0, 1 << 30)
n = 0
for line in out.splitlines():
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if not m:
        continue
    a = int(m.group(1), 16)
    if lo <= a <= hi:
        print(f"{a:05x} {m.group(2).strip()}")
        n += 1
print("instructions:", n)
