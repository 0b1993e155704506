"""Executed-instruction histogram of an ncu report's SASS source page, split into address ranges.

usage: python tools/ncu_sass_hist.py src.csv [lo:hi ...]   (src.csv from ncu -i rep --page source --csv --print-source sass;
addresses as offsets from the kernel start, hex)"""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ia, isrc, iexe = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed")
ins = []
base = None
for r in rows[2:]:
    a = int(r[ia], 16)
    base = a if base is None else base
    ins.append((a - base, r[isrc].strip(), int(r[iexe] or 0)))
tot = sum(x[2] for x in ins)
print(f"total executed warp instructions {tot:.4g}")
ranges = [tuple(int(v, 16) for v in s.split(":")) for s in sys.argv[2:]] or [(0, 1 << 40)]
for lo, hi in ranges:
    sub = [x for x in ins if lo <= x[0] <= hi]
    n = sum(x[2] for x in sub)
    c = Counter()
    for _, s, e in sub:
        op = s.split()[0] if not s.startswith("@") else s.split()[1]
        c[op.split(".")[0]] += e
    print(f"[{lo:#x}, {hi:#x}]: {n:.4g} ({100 * n / max(tot, 1):.1f}%)  " +
          ", ".join(f"{k} {v / max(n, 1) * 100:.1f}%" for k, v in c.most_common(14)))
# hottest straight-line regions: top 25 instructions by count
top = sorted(ins, key=lambda x: -x[2])[:5]
print("max per-instruction count", top[0][2], "at", hex(top[0][0]))
