"""List the loops (backward branches) of one kernel's SASS with opcode histograms.

usage: python tools/sass_loops.py <file.sass> [min_instr]
(file from: cuobjdump -sass -fun <mangled> libfastz.so)
"""
import re
import sys
from collections import Counter

pat = re.compile(r"/\*([0-9a-f]{4,})\*/\s+(@!?U?P[T0-9]\s+)?([A-Z][A-Z0-9_]*)([.A-Z0-9_x]*)\s*([^;]*);")
ins = []
for line in open(sys.argv[1]):
    m = pat.search(line)
    if m:
        ins.append((int(m.group(1), 16), m.group(3), m.group(3) + m.group(4), m.group(5)))
minn = int(sys.argv[2]) if len(sys.argv) > 2 else 40
for k, (addr, op, full, args) in enumerate(ins):
    if op == "BRA":
        t = re.search(r"0x([0-9a-f]+)", args)
        if not t:
            continue
        tgt = int(t.group(1), 16)
        if tgt < addr:
            body = [x for x in ins if tgt <= x[0] <= addr]
            if len(body) < minn:
                continue
            c = Counter(x[2] for x in body)
            print(f"loop 0x{tgt:x}-0x{addr:x}: {len(body)} instr")
            print("   ", ", ".join(f"{n} {o}" for o, n in c.most_common()))
