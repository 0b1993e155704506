"""One extend of a config with the packed inspector (for ncu launch lists / captures).
usage: python tools/pair_prof.py [config_id] [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_gundaboluvt21_b200 import fastz  # noqa: E402
from synth import genome  # noqa: E402

cid = int(sys.argv[1]) if len(sys.argv) > 1 else 2
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
w = genome.make(cid)
with fastz.Aligner(w.T, w.Q) as al:
    for _ in range(reps):
        al.extend_only(w.seeds)
        st = al.stats()
        print({k: st[k] for k in ("ms_inspect", "ms_total", "n_packed_sides", "n_long_sides", "n_redo_sides")},
              flush=True)
