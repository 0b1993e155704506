"""Pins for the redundant-alignment oracle (``oracle/dedup.py``, reading R14; SURVEY.md
§8(f) NEXT-3) against things other than itself:

* hand-derived examples (tests/golden/dedup_examples.json): identical, nested, crossing, one-axis, below-K,
  equal-box tie rules, transitive chains, inclusive edges, empty boxes, off-by-one boxes;
* order-theoretic invariants on random batches: the kept records form an antichain and every redundant record
  is dominated by a kept one (a strict partial order on a finite set has both properties);
* permutation covariance when no two records tie on (box, score);
* a closed form through the extension oracle: every seed on the diagonal of two identical sequences extends to
  the whole pair (all diagonal scores positive), so all records coincide and only the first is kept.
"""
import json
import os
import random

import numpy as np
import pytest

from oracle import core, dedup

HERE = os.path.dirname(os.path.abspath(__file__))
GOLD = json.load(open(os.path.join(HERE, "golden", "dedup_examples.json")))
KEYS = ("score", "flags", "t_start", "t_end", "q_start", "q_end")


def as_rec(rows):
    a = np.asarray(rows, dtype=np.int64).reshape(-1, 6)
    return {k: a[:, i] for i, k in enumerate(KEYS)}


@pytest.mark.parametrize("case", GOLD["cases"], ids=lambda c: c["id"])
def test_golden(case):
    assert dedup.redundant(as_rec(case["recs"])).tolist() == case["redundant"]


def random_batch(rng, n, span=40):
    rows = []
    for _ in range(n):
        t0 = rng.randrange(span)
        q0 = rng.randrange(span)
        rows.append([rng.choice([3000, 3001, 3002, 3500]), rng.choice([0, 1, 1, 1]), t0, t0 + rng.randrange(12),
                     q0, q0 + rng.randrange(12)])
    # copies and nested copies so that ties and containment occur often
    for _ in range(n // 3):
        r = list(rows[rng.randrange(len(rows))])
        if rng.random() < 0.5:
            r[3] = max(r[2], r[3] - rng.randrange(3))
        rows.append(r)
    rng.shuffle(rows)
    return rows


def contains(b, a):
    """box(b) contains box(a), written on its own (not the oracle's code)."""
    return b[2] <= a[2] and a[3] <= b[3] and b[4] <= a[4] and a[5] <= b[5]


@pytest.mark.parametrize("seed", range(12))
def test_antichain_and_cover(seed):
    rng = random.Random(seed)
    rows = random_batch(rng, 60)
    red = dedup.redundant(as_rec(rows))
    kept = [i for i, r in enumerate(rows) if r[1] & 1 and not red[i]]
    # below-K records are never marked
    assert all(red[i] == 0 for i, r in enumerate(rows) if not r[1] & 1)
    # antichain: no kept record's box contains another kept record's box with a score at least as high,
    # unless they tie exactly (same box, same score) -- which the index rule forbids among kept records
    for a in kept:
        for b in kept:
            if a != b and contains(rows[b], rows[a]) and rows[b][0] >= rows[a][0]:
                raise AssertionError(f"kept {b} still covers kept {a}: {rows[b]} {rows[a]}")
    # cover: every redundant record is inside a kept record that scores at least as high
    for a, r in enumerate(rows):
        if red[a]:
            assert any(contains(rows[b], r) and rows[b][0] >= r[0] for b in kept), (a, r)


@pytest.mark.parametrize("seed", range(6))
def test_permutation_covariance(seed):
    rng = random.Random(100 + seed)
    rows, seen = [], set()
    while len(rows) < 50:
        r = random_batch(rng, 1)[0]
        key = (r[0],) + tuple(r[2:])
        if key not in seen:
            seen.add(key)
            rows.append(r)
    red = dedup.redundant(as_rec(rows))
    perm = list(range(len(rows)))
    rng.shuffle(perm)
    red_p = dedup.redundant(as_rec([rows[i] for i in perm]))
    assert [int(red[i]) for i in perm] == red_p.tolist()


def test_identical_sequences_through_the_extension_oracle():
    rng = random.Random(7)
    T = "".join(rng.choice("ACGT") for _ in range(400))
    seeds = np.array([[p, p] for p in (200, 37, 399, 1, 250, 250)], dtype=np.int64)
    o = core.extend(T, T, seeds, core.Params())
    total = sum(core.Params().s("ACGT".index(c), "ACGT".index(c)) for c in T)
    assert (o.rec["score"] == total).all()
    assert (o.rec["t_start"] == 0).all() and (o.rec["t_end"] == 400).all()
    assert dedup.redundant(o.rec).tolist() == [0, 1, 1, 1, 1, 1]


def test_empty_batch():
    assert dedup.redundant(as_rec([])).tolist() == []
