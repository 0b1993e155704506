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
    from tests.gpu_util import run_both
    Y = 1000000
    rng = random.Random(Y)
    T = rseq(rng, 4000); Q = mutate(rng, T, sub=0.15)
    seeds = [(rng.randint(0, 4000), rng.randint(0, len(Q))) for _ in range(40)] + [(k, k) for k in range(100, 4000, 400)]
    sel = [seeds[19]] if sys.argv[2] == "one" else seeds
    g, sides, cells, st, o = run_both(T, Q, sel, ydrop=Y)
    k = 0 if sys.argv[2] == "one" else 19
    sc, ti, qj, fl = sides
    gc, oc = g.cigar_of(k), o.cigar_of(k)
    # first differing position
    d = next((i for i in range(min(len(gc), len(oc))) if gc[i] != oc[i]), None)
    print(json.dumps({"seed": list(map(int, seeds[19])), "L": [int(ti[2*k]), int(qj[2*k]), int(fl[2*k])], "R": [int(ti[2*k+1]), int(qj[2*k+1]), int(fl[2*k+1])],
                      "same": gc == oc, "len": [len(gc), len(oc)], "diff_at": d, "g": gc[:80], "o": oc[:80], "gt": gc[-80:], "ot": oc[-80:]}))
    sys.exit(0)

for bb in ["7", "3"]:
    for mode in ["one", "all"]:
        env = dict(os.environ, FASTZ_ESCALATE_STRIPS="0", FASTZ_BLOCK_BIN=bb)
        r = subprocess.run([sys.executable, __file__, "child", mode], env=env, capture_output=True, text=True)
        print("block_bin", bb, mode, r.stdout.strip()[-900:], r.stderr.strip()[-500:])
