"""Redundant-alignment post-pass oracle -- TEST INFRASTRUCTURE ONLY.

PAPER.md P:110: "LASTZ terminates an ongoing seed extension upon reaching a previously-discovered alignment
because it is not profitable to combine the prior and current alignments; if it were, the prior alignment would
have expanded to include the current one."  P:220: this is "infeasible in *any* parallel implementation", so
FastZ extends every seed and reports "the same or a strict superset" of LASTZ's work.  NEXT-3 applies the
skip after the fact, order-free.  The paper gives no formula; reading R14 fixes it:

  Only records with FASTZ_FLAG_ABOVE_K take part.  Record b DOMINATES record a (a != b) iff
    b.t_start <= a.t_start, a.t_end <= b.t_end, b.q_start <= a.q_start, a.q_end <= b.q_end   (box containment)
    and b.score >= a.score
    and (the boxes differ, or b.score > a.score, or b.index < a.index)            (strict tie-break)
  a is REDUNDANT iff some record dominates it.

Domination is a strict partial order, so every redundant record is dominated by a non-redundant one and the
non-redundant records form an antichain (tests/test_dedup_oracle.py checks both without this module's loop).
This is the definition written out as an all-pairs loop: O(n^2), for the small batches of the tests.
Not imported by the product.
"""
from __future__ import annotations

import numpy as np

FLAG_ABOVE_K = 1


def dominates(b: dict, a: dict, ib: int, ia: int) -> bool:
    """Reading R14 for one ordered pair (b over a); a and b are records with the fastz_alignment fields."""
    if ia == ib:
        return False
    if not (b["t_start"] <= a["t_start"] and a["t_end"] <= b["t_end"]):
        return False
    if not (b["q_start"] <= a["q_start"] and a["q_end"] <= b["q_end"]):
        return False
    if b["score"] < a["score"]:
        return False
    same_box = (b["t_start"] == a["t_start"] and b["t_end"] == a["t_end"] and b["q_start"] == a["q_start"]
                and b["q_end"] == a["q_end"])
    return (not same_box) or b["score"] > a["score"] or ib < ia


def redundant(rec) -> np.ndarray:
    """rec: structured array (or dict of equal-length arrays) with score, flags, t_start, t_end, q_start,
    q_end.  Returns uint8[n]: 1 where the record is redundant (R14), 0 elsewhere (including below-K)."""
    n = len(rec["score"])
    rows = [{k: int(rec[k][s]) for k in ("score", "flags", "t_start", "t_end", "q_start", "q_end")}
            for s in range(n)]
    cand = [s for s in range(n) if rows[s]["flags"] & FLAG_ABOVE_K]
    out = np.zeros(n, dtype=np.uint8)
    for a in cand:
        for b in cand:
            if dominates(rows[b], rows[a], b, a):
                out[a] = 1
                break
    return out
