"""Per-region instruction counts from an ncu source page (SASS) export.

usage: ncu -i rep --page source --csv --print-source sass > src.csv; python tools/ncu_sass_regions.py src.csv [n]
Prints the total warp instructions executed and the hottest basic blocks (runs of equal execution count) with
their share of executed instructions and of stall samples.
"""
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ia, isrc, iex = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed")
isamp = hdr.index("Warp Stall Sampling (All Samples)")
ins = []
for r in rows[2:]:
    try:
        ins.append((int(r[ia], 16), r[isrc].strip(), int(r[iex] or 0), int(r[isamp] or 0)))
    except (ValueError, IndexError):
        pass
base = ins[0][0]
tot = sum(x[2] for x in ins)
tsamp = sum(x[3] for x in ins)
print(f"total warp instructions {tot:.4e}, samples {tsamp}")
blocks = []
cur = [ins[0]]
for x in ins[1:]:
    if x[2] == cur[-1][2] and not re.search(r"\bBRA\b|EXIT|BSYNC", cur[-1][1]):
        cur.append(x)
    else:
        blocks.append(cur)
        cur = [x]
blocks.append(cur)
blocks.sort(key=lambda b: -sum(x[2] for x in b))
for b in blocks[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    s = sum(x[2] for x in b)
    sp = sum(x[3] for x in b)
    print(f"0x{b[0][0]-base:05x}-0x{b[-1][0]-base:05x} n={len(b):4d} exec/instr={b[0][2]:.3e} "
          f"share={s/tot*100:5.1f}% samples={sp/tsamp*100:5.1f}%  first: {b[0][1][:60]}")
