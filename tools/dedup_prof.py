"""Run C5 (the most candidates) once and the redundant-alignment post-pass twice -- for ncu captures of k_rd_*."""
import os
import sys

sys.path.insert(0, os.getcwd())
from paper_conf_sc_gundaboluvt21_b200 import fastz  # noqa: E402
from synth import genome  # noqa: E402

w = genome.make(int(sys.argv[1]) if len(sys.argv) > 1 else 5)
with fastz.Aligner(w.T, w.Q) as al:
    al.extend_only(w.seeds)
    for _ in range(2):
        red, n = al.mark_redundant()
print("redundant", n)
