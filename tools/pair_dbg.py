"""Diagnostics of the mixed inspector (FASTZ_PAIR_DEBUG): per-phase warp clocks and the slowest packed sides.
usage: python tools/pair_dbg.py [small|c<id>] [FASTZ_PAIR_LONG]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["FASTZ_PAIR_DEBUG"] = "1"
from paper_conf_sc_gundaboluvt21_b200 import fastz  # noqa: E402
from synth import genome  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "small"
if len(sys.argv) > 2:
    os.environ["FASTZ_PAIR_LONG"] = sys.argv[2]
w = genome.small_pair(7, length=30000, n_seeds=512) if which == "small" else genome.make(int(which[1:]))
with fastz.Aligner(w.T, w.Q) as al:
    for _ in range(2):
        al.extend_only(w.seeds)
        print("ms_inspect", al.stats()["ms_inspect"], flush=True)
