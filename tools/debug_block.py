import os, random, sys, subprocess, json
sys.path.insert(0, os.getcwd())
import numpy as np

def rseq(rng, n): return "".join(rng.choice("ACGT") for _ in range(n))
def mutate(rng, s, sub=0.1, indel=0.02):
    out = []
    for ch in s:
        r = rng.random()
        if r < indel / 2: continue
        if r < indel: out.append(rng.choice("ACGT"))
        out.append(rng.choice([b for b in "ACGT" if b != ch]) if rng.random() < sub else ch)
    return "".join(out)

if len(sys.argv) > 1 and sys.argv[1] == "child":
    from tests.gpu_util import compare
    Y = int(sys.argv[2])
    rng = random.Random(Y)
    T = rseq(rng, 4000); Q = mutate(rng, T, sub=0.15)
    seeds = [(rng.randint(0, 4000), rng.randint(0, len(Q))) for _ in range(40)] + [(k, k) for k in range(100, 4000, 400)]
    bad, g, o, st = compare(T, Q, seeds, census=False, ydrop=Y)
    print(json.dumps({"bad": [(b[0], b[1]) for b in bad], "bins": st["bin_counts"][:7]}))
    sys.exit(0)

for esc, bb in [("0", "7"), ("16", "7"), ("0", "3"), ("16", "3"), ("1", "1")]:
    env = dict(os.environ, FASTZ_ESCALATE_STRIPS=esc, FASTZ_BLOCK_BIN=bb)
    r = subprocess.run([sys.executable, __file__, "child", "1000000"], env=env, capture_output=True, text=True)
    print("esc", esc, "block_bin", bb, r.stdout.strip()[-300:], r.stderr.strip()[-300:])
