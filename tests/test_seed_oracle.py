"""Pins of the seeding + ungapped-filter oracle (oracle/seed_oracle.c, readings S1-S6 in DESIGN.md; NEXT-4).

The C oracle is checked against things other than itself: an all-pairs brute force that tests every (t, q)
pair directly (no index, no binary search), closed forms for identical sequences and for an x-drop threshold
crossing, and hand-built transition / transversion / don't-care cases.
"""
import numpy as np
import pytest

from oracle import seeds
from oracle.core import HOXD70

RNG = np.random.default_rng(20211114)


def rand_seq(n, rng=RNG):
    return "".join("ACGT"[i] for i in rng.integers(0, 4, n))


def mutate(s, rng, sub=0.1, indel=0.01):
    out = []
    for c in s:
        u = rng.random()
        if u < indel / 2:
            continue
        if u < indel:
            out.append("ACGT"[rng.integers(0, 4)])
        if rng.random() < sub:
            out.append("ACGT"[(("ACGT".index(c)) + rng.integers(1, 4)) % 4])
        else:
            out.append(c)
    return "".join(out)


def as_tuples(a):
    return [(int(r["t_start"]), int(r["q_start"]), int(r["length"]), int(r["score"])) for r in a]


@pytest.mark.parametrize("pattern", [seeds.PATTERN_12OF19, "1101011", "111"])
@pytest.mark.parametrize("transitions", [True, False])
def test_brute_force_agrees(pattern, transitions):
    rng = np.random.default_rng(7 + len(pattern) + transitions)
    for trial in range(3):
        core = rand_seq(150, rng)
        T = rand_seq(40, rng) + core + rand_seq(30, rng)
        Q = rand_seq(25, rng) + mutate(core, rng) + rand_seq(45, rng)
        thr = [300, 1000, 3000][trial]
        got, hits = seeds.find_hsps(T, Q, HOXD70, pattern, transitions, 910, thr)
        want = seeds.brute_hsps(T, Q, HOXD70, pattern, transitions, 910, thr)
        assert as_tuples(got) == want
        assert hits == len(seeds.brute_hits(T, Q, pattern, transitions))


def test_identical_sequences_closed_form():
    T = rand_seq(400)
    got, hits = seeds.find_hsps(T, T, HOXD70)
    full = (0, 0, 400, sum(HOXD70["ACGT".index(c)]["ACGT".index(c)] for c in T))
    assert full in as_tuples(got)
    # every diagonal word hits itself exactly
    assert hits >= 400 - 19 + 1


def test_xdrop_threshold_crossing():
    # 7 C/A mismatches cost 7 * 114 = 798 <= 910: the extension crosses them; 8 cost 912 > 910: it stops
    for k, crosses in [(7, True), (8, False)]:
        T = "A" * 60 + "C" * k + "A" * 60
        Q = "A" * (120 + k)
        got, _ = seeds.find_hsps(T, Q, HOXD70, "111", False, 910, 0)
        tup = as_tuples(got)
        if crosses:
            assert (0, 0, 120 + k, 120 * 91 - 114 * k) in tup
        else:
            assert (0, 0, 60, 60 * 91) in tup
            assert all(h[2] < 120 + k or h[1] != 0 or h[0] != 0 for h in tup)


def test_transition_transversion_dontcare():
    base = rand_seq(19)
    care = [i for i, c in enumerate(seeds.PATTERN_12OF19) if c == "1"]
    dont = [i for i, c in enumerate(seeds.PATTERN_12OF19) if c == "0"]
    ti = {"A": "G", "G": "A", "C": "T", "T": "C"}
    tv = {"A": "C", "G": "T", "C": "A", "T": "G"}

    def with_change(pos, table):
        return base[:pos] + table[base[pos]] + base[pos + 1:]

    assert (0, 0) in seeds.brute_hits(base, with_change(dont[0], tv), transitions=False)
    assert (0, 0) in seeds.brute_hits(base, with_change(care[3], ti), transitions=True)
    assert (0, 0) not in seeds.brute_hits(base, with_change(care[3], ti), transitions=False)
    assert (0, 0) not in seeds.brute_hits(base, with_change(care[3], tv), transitions=True)
    two = with_change(care[1], ti)
    two = two[:care[5]] + ti[two[care[5]]] + two[care[5] + 1:]
    assert (0, 0) not in seeds.brute_hits(base, two, transitions=True)
    # the C oracle's hit counts agree on the same constructed pairs
    for Q, tr in [(with_change(care[3], ti), True), (with_change(care[3], ti), False), (two, True)]:
        _, hits = seeds.find_hsps(base, Q, HOXD70, seeds.PATTERN_12OF19, tr, 910, 10 ** 9)
        assert hits == len(seeds.brute_hits(base, Q, seeds.PATTERN_12OF19, tr))


def test_anchor_order_and_dedup():
    core = rand_seq(600)
    T = rand_seq(100) + core + rand_seq(100)
    Q = rand_seq(50) + mutate(core, np.random.default_rng(3)) + rand_seq(150)
    got, hits = seeds.find_hsps(T, Q, HOXD70)
    tup = as_tuples(got)
    assert len(set(tup)) == len(tup)                   # S5
    keys = [(h[0] + h[2] // 2, h[1] + h[2] // 2, h[0], h[2]) for h in tup]
    assert keys == sorted(keys)                        # S6
    assert all(h[3] >= seeds.HSPTHRESH for h in tup)   # S4
    assert hits > len(tup)                             # many seeds collapse onto few HSPs


def test_bad_input():
    with pytest.raises(ValueError):
        seeds.find_hsps("ACGX" * 10, "ACGT" * 10, HOXD70)
    with pytest.raises(ValueError):
        seeds.find_hsps("ACGT" * 10, "ACGT" * 10, HOXD70, pattern="0110")


def test_n_bases():
    """S7: words with an N at a care position match nothing; walks score N as n_score.  Brute force agrees."""
    rng = np.random.default_rng(77)
    for trial in range(4):
        core_ = rand_seq(160, rng)
        T = list(rand_seq(30, rng) + core_ + rand_seq(30, rng))
        Q = list(rand_seq(20, rng) + mutate(core_, rng) + rand_seq(40, rng))
        for s_ in (T, Q):
            for p in rng.choice(len(s_), 6, replace=False):
                s_[p] = "N"
        T, Q = "".join(T), "".join(Q)
        for pattern, nsc in ((seeds.PATTERN_12OF19, -100), ("1101011", 0), ("111", -300)):
            got, hits = seeds.find_hsps(T, Q, HOXD70, pattern, True, 910, 300, nsc)
            assert as_tuples(got) == seeds.brute_hsps(T, Q, HOXD70, pattern, True, 910, 300, nsc)
            assert hits == len(seeds.brute_hits(T, Q, pattern, True))
    # an N at a don't-care position does not block a hit; at a care position it does
    base = rand_seq(19, rng)
    dont = seeds.PATTERN_12OF19.index("0")
    care = seeds.PATTERN_12OF19.index("1")
    assert (0, 0) in seeds.brute_hits(base, base[:dont] + "N" + base[dont + 1:])
    assert (0, 0) not in seeds.brute_hits(base, base[:care] + "N" + base[care + 1:])
