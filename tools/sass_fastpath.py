"""Opcode histogram of a loop's fast path: skips the bodies guarded by `VOTE.ANY Px` + `@!Px BRA target`
(the rare peak-update slow path).  usage: python tools/sass_fastpath.py file.sass 0xSTART 0xEND [steps]"""
import re
import sys
from collections import Counter

pat = re.compile(r"/\*([0-9a-f]{4,})\*/\s+(@!?U?P[T0-9]\s+)?([A-Z][A-Z0-9_.]*)\s*([^;]*);")
lo, hi = int(sys.argv[2], 16), int(sys.argv[3], 16)
steps = int(sys.argv[4]) if len(sys.argv) > 4 else 1
ins = []
for line in open(sys.argv[1]):
    m = pat.search(line)
    if m and lo <= int(m.group(1), 16) <= hi:
        ins.append((int(m.group(1), 16), (m.group(2) or "").strip(), m.group(3), m.group(4)))
c = Counter()
skip_to = -1
for k, (a, pred, op, args) in enumerate(ins):
    if a < skip_to:
        continue
    c[op] += 1
    if op == "BRA" and pred.startswith("@!P") and any(x[2] == "VOTE.ANY" for x in ins[max(0, k - 12):k]):
        t = re.search(r"0x([0-9a-f]+)", args)
        skip_to = int(t.group(1), 16)
tot = sum(c.values())
print(f"fast path: {tot} instructions, {tot / steps:.1f} per step")
print(", ".join(f"{n} {o}" for o, n in c.most_common()))
