"""C2 with N bases (assembly-gap-like runs + isolated N): times the N-aware kernels; prints one JSON line."""
import json, os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from synth import genome
from paper_conf_sc_gundaboluvt21_b200 import fastz
w = genome.make(2)
rng = np.random.default_rng(99)
def add_ns(s):
    a = np.frombuffer(bytearray(s), dtype=np.uint8).copy()
    for p in rng.integers(0, len(a) - 1000, 100):
        a[p:p + 1000] = ord("N")
    a[rng.integers(0, len(a), len(a) // 10000)] = ord("N")
    return a.tobytes()
T, Q = add_ns(w.T), add_ns(w.Q)
seeds = torch.from_numpy(np.ascontiguousarray(w.seeds)).cuda()
al = fastz.Aligner(T, Q, torch_alloc=True)
al.extend_only(seeds)
ms = []
for _ in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter(); al.extend_only(seeds); torch.cuda.synchronize()
    ms.append((time.perf_counter() - t0) * 1e3)
st = al.stats()
print(json.dumps({"workload": "C2 + N runs", "ms": min(ms), "inspect_ms": st["ms_inspect"]}))
