"""Device-timed step per config (bench launch configuration), one JSON line each.

usage: python tools/config_sweep.py [configs...]   (default 1 2 3 5 6; FASTZ_LIB selects an A/B build)
Per config: 3 warm-up + 3 timed fastz_extend_seeds calls (CUDA events on the stream), stages, explored cells
(census), GCUPS, executor words written / reserved, waves."""
import json
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np
import torch

from paper_conf_sc_gundaboluvt21_b200 import fastz
from synth import genome

cfgs = [int(c) for c in sys.argv[1:]] or [1, 2, 3, 5, 6]
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream(dev)
for cfg in cfgs:
    w = genome.make(cfg)
    al = fastz.Aligner(w.T, w.Q, device=0, stream=stream.cuda_stream, torch_alloc=True)
    sd = torch.from_numpy(np.ascontiguousarray(w.seeds)).to(dev)
    al.extend_only(sd)
    cells = int(al.census().sum())
    for _ in range(3):
        al.extend_only(sd)
    ts, sts = [], []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(stream)
        al.extend_only(sd)
        e1.record(stream)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
        sts.append(al.stats())
    ms = sum(ts) / len(ts)
    st = sts[-1]
    avg = lambda k: round(sum(s[k] for s in sts) / len(sts), 2)  # noqa: E731
    print(json.dumps({"config": w.name, "lib": os.environ.get("FASTZ_LIB", "in-tree"), "seeds": w.n, "ms": round(ms, 2),
                      "GCUPS": cells / ms / 1e6, "cells": cells,
                      "stages_ms": {k: avg(k) for k in ("ms_inspect", "ms_bin", "ms_execute", "ms_traceback", "ms_combine")},
                      "bins": st["bin_counts"][:7], "exec_words": st["exec_words"],
                      "exec_reserved_words": st["exec_reserved_words"],
                      "reserved_over_written": st["exec_reserved_words"] / max(st["exec_words"], 1),
                      "waves": st["n_waves"], "wide": st["n_wide_sides"]}), flush=True)
    al.close()
    del w, sd
    torch.cuda.empty_cache()
