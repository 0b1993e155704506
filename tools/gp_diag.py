"""Diagnose the genome-pair wall time inside a bench-like process: phases of a second context."""
import os, sys, time, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from synth import genome
from paper_conf_sc_gundaboluvt21_b200 import fastz
w = genome.make(2)
dev = torch.device("cuda", 0); torch.cuda.set_device(0)
stream = torch.cuda.current_stream(dev)
shard = np.ascontiguousarray(w.seeds)
al = fastz.Aligner(w.T, w.Q, device=0, stream=stream.cuda_stream)
sd = torch.from_numpy(shard).to(dev)
al.extend_only(sd); al.extend_only(sd)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
def phases(tag):
    torch.cuda.synchronize()
    t0 = time.perf_counter(); al2 = fastz.Aligner(w.T, w.Q, device=0, stream=stream.cuda_stream); torch.cuda.synchronize(); t1 = time.perf_counter()
    al2.extend_only(shard); torch.cuda.synchronize(); t2 = time.perf_counter()
    st = {k: round(v, 1) for k, v in al2.stats().items() if k.startswith("ms")}
    r = al2.results(); t3 = time.perf_counter()
    al2.close(); t4 = time.perf_counter()
    print(json.dumps({"tag": tag, "create": round(t1 - t0, 3), "extend": round(t2 - t1, 3), "results": round(t3 - t2, 3), "close": round(t4 - t3, 3), "stats": st}), flush=True)
phases("no_pinned")
phases("no_pinned_again")
al.results_pinned()
phases("after_pinned")
al.extend_only(sd); al.results_pinned()
phases("after_pinned_e2e")
