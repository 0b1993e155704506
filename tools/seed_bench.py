"""Seeding + ungapped-filter stage (NEXT-4) on one B200: throughput on the C2 pair and sampled parity.

usage: python tools/seed_bench.py [config_id] [sample_bp]
Times fastz_find_hsps (spaced-seed index of T, hits of every Q word, ungapped x-drop walks, dedup, anchors)
on the full pair, then checks a bounded query window (T x Q[0:sample_bp]) against the C oracle and times the
oracle on it (one host thread; the oracle is never tuned).  Prints one JSON line.
"""
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import core, seeds  # noqa: E402
from paper_conf_sc_gundaboluvt21_b200 import fastz  # noqa: E402
from synth import genome  # noqa: E402


def main():
    cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    sample = int(sys.argv[2]) if len(sys.argv) > 2 else 300_000
    w = genome.make(cfg, n_seeds=1024)
    T, Q = w.T, w.Q
    with fastz.Aligner(T, Q) as al:
        al.find_hsps()  # warm-up (allocations, module load)
        times = []
        for _ in range(3):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            hs, an, hits = al.find_hsps()
            torch.cuda.synchronize()
            times.append(time.perf_counter() - t0)
        t_full = min(times)
        # the pipeline end to end: anchors -> gapped extension
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        al.extend(an)
        torch.cuda.synchronize()
        t_ext = time.perf_counter() - t0
    Qs = Q[:sample]
    with fastz.Aligner(T, Qs) as al:
        g, gan, ghits = al.find_hsps()
    t0 = time.perf_counter()
    o, ohits = seeds.find_hsps(T, Qs, core.HOXD70)
    t_or = time.perf_counter() - t0
    same = ghits == ohits and len(g) == len(o) and all(
        np.array_equal(g[f].astype(np.int64), o[f].astype(np.int64)) for f in ("t_start", "q_start", "length", "score"))
    out = {
        "stage": "seeding+ungapped filter (fastz_find_hsps)", "config": w.name, "target_bp": len(T),
        "query_bp": len(Q), "pattern": seeds.PATTERN_12OF19, "transitions": 1, "xdrop": seeds.XDROP,
        "hspthresh": seeds.HSPTHRESH, "ms": t_full * 1e3, "query_mbp_per_s": len(Q) / t_full / 1e6,
        "hits": hits, "hits_per_s": hits / t_full, "hsps": int(len(hs)), "extend_anchors_ms": t_ext * 1e3,
        "sample": {"query_bp": sample, "parity": bool(same), "hits": ghits, "hsps": int(len(g)),
                   "oracle_s": t_or, "oracle_threads": 1,
                   "oracle_query_mbp_per_s": sample / t_or / 1e6},
    }
    print(json.dumps(out))


if __name__ == "__main__":
    main()
