import json, os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from synth import genome
from paper_conf_sc_gundaboluvt21_b200 import fastz as fz
for cfg in [int(c) for c in os.environ.get("CFGS", "2 5 1").split()]:
    w = genome.make(cfg)
    seeds = torch.from_numpy(np.ascontiguousarray(w.seeds)).cuda()
    al = fz.Aligner(w.T, w.Q, stream=torch.cuda.current_stream().cuda_stream)
    for esc in ["0", "8", "16", "32", "64"]:
        os.environ["FASTZ_ESCALATE_STRIPS"] = esc
        al.extend_only(seeds)
        ts = []
        for _ in range(2):
            torch.cuda.synchronize(); t0 = time.perf_counter(); al.extend_only(seeds); torch.cuda.synchronize(); ts.append(time.perf_counter() - t0)
        st = al.stats()
        print(json.dumps({"cfg": cfg, "esc": esc, "ms": round(1e3 * min(ts), 1), "inspect": round(st["ms_inspect"], 1), "escalated": st["n_escalated"], "exec": round(st["ms_execute"], 1)}), flush=True)
    al.close()
