"""Time the phases of a fresh context on C2 (create, first extend, second extend, results)."""
import os, sys, time, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from synth import genome
from paper_conf_sc_gundaboluvt21_b200 import fastz
w = genome.make(2)
seeds = np.ascontiguousarray(w.seeds)
torch.cuda.init(); torch.cuda.synchronize()
out = {}
for rep in range(2):
    t0 = time.perf_counter(); al = fastz.Aligner(w.T, w.Q); torch.cuda.synchronize(); out[f"create{rep}"] = time.perf_counter() - t0
    t0 = time.perf_counter(); al.extend_only(seeds); torch.cuda.synchronize(); out[f"extend1_{rep}"] = time.perf_counter() - t0
    out[f"stats1_{rep}"] = {k: round(v, 1) for k, v in al.stats().items() if k.startswith("ms")}
    t0 = time.perf_counter(); al.extend_only(seeds); torch.cuda.synchronize(); out[f"extend2_{rep}"] = time.perf_counter() - t0
    t0 = time.perf_counter(); r = al.results(); out[f"results_{rep}"] = time.perf_counter() - t0
    al.close()
print(json.dumps(out))
