"""Pins of the whole-batch re-scoring check (oracle/rescore.c) used by the full-size GPU parity tests: it must
accept the oracle's own records (every CIGAR walks through the cut point and re-scores to the per-side peaks)
and reject each kind of corruption.  CPU only."""
import json
import os

import numpy as np

from oracle import core, rescore
from synth import genome

HERE = os.path.dirname(os.path.abspath(__file__))
GOLD = json.load(open(os.path.join(HERE, "golden", "worked_examples.json")))


def _records(o):
    rec = np.zeros(len(o.rec), dtype=rescore.RECORD_DTYPE)
    for f in ("score", "left_score", "right_score", "flags", "t_start", "t_end", "q_start", "q_end", "cigar_off",
              "cigar_len"):
        rec[f] = o.rec[f]
    return rec


def test_worked_examples_rescore():
    for ex in GOLD["two_sided"]:
        rec = np.zeros(1, rescore.RECORD_DTYPE)
        for f in ("score", "left_score", "right_score", "t_start", "t_end", "q_start", "q_end"):
            rec[f] = ex[f]
        rec["cigar_len"] = len(ex["cigar"])
        nbad, why = rescore.rescore(ex["T"], ex["Q"], [(ex["tpos"], ex["qpos"])], rec, ex["cigar"].encode())
        assert nbad == 0, (ex["id"], rescore.REASONS[int(why[0])])


def test_oracle_records_rescore_and_corruptions_fail():
    w = genome.small_pair(7, length=20000, n_seeds=300)
    o = core.extend(w.T, w.Q, w.seeds)
    rec = _records(o)
    nbad, why = rescore.rescore(w.T, w.Q, w.seeds, rec, o.cigar)
    assert nbad == 0, [rescore.REASONS[int(x)] for x in why[why != 0][:5]]
    long = np.nonzero(o.rec["cigar_len"] > 8)[0]
    s = int(long[0])
    # a score off by one
    r2 = rec.copy()
    r2["left_score"][s] += 1
    r2["score"][s] += 1
    assert rescore.rescore(w.T, w.Q, w.seeds, r2, o.cigar)[1][s] == 7
    # score != left + right
    r2 = rec.copy()
    r2["score"][s] += 1
    assert rescore.rescore(w.T, w.Q, w.seeds, r2, o.cigar)[1][s] == 2
    # a CIGAR op flipped (M -> I somewhere) changes the walk
    cig = bytearray(o.cigar)
    off = int(rec["cigar_off"][s])
    text = cig[off: off + int(rec["cigar_len"][s])]
    k = text.find(b"M")
    cig[off + k] = ord("I") if text[k + 1:k + 2] != b"I" and (k == 0 or text[k - 1:k] != b"I") else ord("D")
    assert rescore.rescore(w.T, w.Q, w.seeds, rec, bytes(cig))[1][s] != 0
    # endpoints shifted
    r2 = rec.copy()
    r2["t_end"][s] += 1
    assert rescore.rescore(w.T, w.Q, w.seeds, r2, o.cigar)[1][s] != 0
    # a wrong seed (cut point not on the path)
    sd = w.seeds.copy()
    sd[s, 0] += 1
    assert rescore.rescore(w.T, w.Q, sd, rec, o.cigar)[1][s] != 0


def test_gap_run_across_the_cut_pays_two_opens():
    """T = ACGTTACGT, Q = ACGTACGT cut inside the deleted T: the left side ends with 1D and the right side
    starts with ... here a 2-base deletion split 1+1 across the cut costs 2(O + E), merged in the text."""
    T, Q = "ACGTAAACGT", "ACGTACGT"
    rec = np.zeros(1, rescore.RECORD_DTYPE)
    # path 4M 2D 4M; cut after the first D: (tpos, qpos) = (5, 4)
    left = 91 + 100 + 100 + 91 - (400 + 30)
    right = -(400 + 30) + 91 + 100 + 100 + 91
    rec["left_score"], rec["right_score"], rec["score"] = left, right, left + right
    rec["t_start"], rec["t_end"], rec["q_start"], rec["q_end"] = 0, 10, 0, 8
    rec["cigar_len"] = 6
    assert rescore.rescore(T, Q, [(5, 4)], rec, b"4M2D4M")[0] == 0
    rec["left_score"] += 400
    rec["score"] += 400
    assert rescore.rescore(T, Q, [(5, 4)], rec, b"4M2D4M")[0] == 1
