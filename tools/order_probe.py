"""Experiment: does the inspector have a long-side tail?  Times fastz_extend_seeds (ms_inspect) on C2 with the
seeds in their natural (random) order versus the same seeds with the planted long classes first (an oracle-free
upper bound for any LPT-style inspector ordering, using the generator's class labels).
usage: python tools/order_probe.py [config]"""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_sc_gundaboluvt21_b200 import fastz  # noqa: E402
from synth import genome  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
w = genome.make(cfg)
names = w.class_names
print("classes", names, np.bincount(w.klass), flush=True)
# longer planted classes first: rank by class index descending (junk = 0 last)
perm_long = np.argsort(-w.klass, kind="stable")
perm_rev = perm_long[::-1].copy()
out = {}
with fastz.Aligner(w.T, w.Q, torch_alloc=True) as al:
    for name, perm in (("natural", np.arange(w.n)), ("long_first", perm_long), ("long_last", perm_rev),
                       ("natural2", np.arange(w.n)), ("long_first2", perm_long)):
        sd = torch.from_numpy(np.ascontiguousarray(w.seeds[perm])).cuda()
        for _ in range(2):
            al.extend_only(sd)
        ms = []
        for _ in range(3):
            al.extend_only(sd)
            ms.append(al.stats()["ms_inspect"])
        st = al.stats()
        out[name] = ms
        print(name, ms, "execute", round(st["ms_execute"], 1), "total", round(st["ms_total"], 1), flush=True)
print(json.dumps(out))
