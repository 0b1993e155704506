"""Run a config end to end on the GPU (timed), report stages, and check a random seed sample vs the oracle."""
import json, os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np
from synth import genome
from paper_conf_sc_gundaboluvt21_b200 import fastz
from oracle import core

cfg = int(sys.argv[1]); nsample = int(sys.argv[2]) if len(sys.argv) > 2 else 20
t0 = time.time(); w = genome.make(cfg); tg = time.time() - t0
al = fastz.Aligner(w.T, w.Q)
al.extend_only(w.seeds)  # warm
t0 = time.time(); res = al.extend(w.seeds); te = time.time() - t0
st = al.stats()
al.mark_redundant()  # NEXT-3 post-pass (reading R14): warm, then timed
t0 = time.time(); red, nred = al.mark_redundant(); tr = time.time() - t0
nk = int(((res.rec["flags"] & fastz.FLAG_ABOVE_K) != 0).sum())
cells = int(al.census().sum())
rng = np.random.default_rng(cfg)
idx = np.sort(rng.choice(w.n, min(nsample, w.n), replace=False))
t0 = time.time(); o = core.extend(w.T, w.Q, w.seeds[idx]); to = time.time() - t0
ok = all(np.array_equal(res.rec[f][idx].astype(np.int64), o.rec[f]) for f in ("score", "t_start", "t_end", "q_start", "q_end")) \
    and all(res.cigar_of(s) == o.cigar_of(k) for k, s in enumerate(idx))
ocells = int(o.rec["l_explored"].sum() + o.rec["r_explored"].sum())
print(json.dumps({"config": w.name, "seeds": w.n, "tlen": len(w.T), "gen_s": round(tg, 1), "e2e_s": round(te, 3),
                  "stages_ms": {k: round(st[k], 2) for k in ("ms_total", "ms_inspect", "ms_bin", "ms_execute", "ms_traceback", "ms_combine")},
                  "cells": cells, "GCUPS_e2e": cells / te / 1e9, "GCUPS_device": cells / (st["ms_total"] / 1e3) / 1e9,
                  "bins": st["bin_counts"][:7], "exec_words": st["exec_words"], "sample": len(idx), "parity": bool(ok),
                  "dedup": {"above_k": nk, "redundant": int(nred), "ms_host": round(tr * 1e3, 2)},
                  "oracle_s": round(to, 1), "oracle_GCUPS": ocells / to / 1e9}))
