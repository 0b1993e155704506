"""Full-size parity in the bench launch configuration: the whole C2 batch (2^20 seeds, 10 Mbp pair) and
C1 (2,048 seeds on a 100 kbp pair) run through the C ABI exactly as bench.py runs them; a random sample of
seeds is compared bit-exactly with the CPU oracle, and properties that must hold for every seed are
checked on the whole batch (CIGAR consumes exactly the reported spans; score = left + right; eager flags
match the spans' peak classification)."""
import re

import numpy as np
import pytest

from oracle import core
from paper_conf_sc_gundaboluvt21_b200 import fastz
from synth import genome
from tests.gpu_util import FIELDS

pytestmark = pytest.mark.gpu
_RUN = re.compile(rb"(\d+)([MID])")


def _check_all(w, g, n_sample, rng):
    rec = g.rec
    assert np.array_equal(rec["score"], rec["left_score"] + rec["right_score"])
    assert (rec["t_start"] <= w.seeds[:, 0]).all() and (rec["t_end"] >= w.seeds[:, 0]).all()
    # every CIGAR consumes exactly the reported spans
    for s in range(len(rec)):
        c = g.cigar[rec["cigar_off"][s]: rec["cigar_off"][s] + rec["cigar_len"][s]]
        m = i = d = 0
        for num, op in _RUN.findall(c):
            k = int(num)
            if op == b"M":
                m += k
            elif op == b"I":
                i += k
            else:
                d += k
        assert m + d == rec["t_end"][s] - rec["t_start"][s] and m + i == rec["q_end"][s] - rec["q_start"][s], s
    idx = np.sort(rng.choice(len(rec), n_sample, replace=False))
    o = core.extend(w.T, w.Q, w.seeds[idx])
    for f in FIELDS:
        assert np.array_equal(rec[f][idx].astype(np.int64), o.rec[f]), f
    assert np.array_equal((rec["flags"][idx] & 15).astype(np.int64), o.rec["flags"] & 15)
    for k, s in enumerate(idx):
        assert g.cigar_of(s) == o.cigar_of(k), s


def test_c2_full_batch_sampled_parity():
    w = genome.config2()
    with fastz.Aligner(w.T, w.Q) as al:
        g = al.extend(w.seeds)
        st = al.stats()
    assert len(g.rec) == 1 << 20 and st["n_sides"] == 1 << 21
    _check_all(w, g, 300, np.random.default_rng(2))


def test_c1_full_batch_sampled_parity():
    w = genome.config1()
    with fastz.Aligner(w.T, w.Q) as al:
        g = al.extend(w.seeds)
    _check_all(w, g, 24, np.random.default_rng(1))
