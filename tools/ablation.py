"""Fig. 9 analog on B200: the same C2 batch with FastZ's techniques switched off one at a
time and cumulatively, via FASTZ_OPT_* (results are identical -- checked here -- only the time changes)."""
import json, os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np
import torch
from synth import genome
from paper_conf_sc_gundaboluvt21_b200 import fastz as fz

cfg = int(os.environ.get("CFG", "2"))
w = genome.make(cfg)
dev = torch.device("cuda", 0)
seeds = torch.from_numpy(np.ascontiguousarray(w.seeds)).to(dev)
variants = [("fastz (all techniques)", 0), ("no block-per-side", fz.OPT_NO_BLOCK),
            ("no length binning", fz.OPT_NO_BINNING), ("no executor trimming", fz.OPT_NO_TRIM),
            ("no eager traceback", fz.OPT_NO_EAGER),
            ("none of binning/trim/eager/block", fz.OPT_NO_BLOCK | fz.OPT_NO_BINNING | fz.OPT_NO_TRIM | fz.OPT_NO_EAGER)]
ref = None
out = []
for name, opt in variants:
    al = fz.Aligner(w.T, w.Q, fz.fastz_default_params(options=opt), stream=torch.cuda.current_stream().cuda_stream)
    al.extend_only(seeds)
    ts = []
    for _ in range(3):
        torch.cuda.synchronize(); t0 = time.perf_counter(); al.extend_only(seeds); torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    res = al.results(); st = al.stats()
    same = ref is None or (np.array_equal(res.rec, ref.rec) and res.cigar == ref.cigar)
    if ref is None:
        ref = res
    out.append({"variant": name, "options": opt, "ms": 1e3 * min(ts), "inspect_ms": st["ms_inspect"],
                "execute_ms": st["ms_execute"], "traceback_ms": st["ms_traceback"], "exec_sides": st["n_exec_sides"],
                "exec_words": st["exec_words"], "identical_results": bool(same)})
    al.close()
base = out[0]["ms"]
for r in out:
    r["slowdown_vs_fastz"] = r["ms"] / base
    print(json.dumps(r))
