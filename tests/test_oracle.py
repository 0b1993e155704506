"""Pins for the CPU oracle (``oracle/``) against things other than itself.

Each pin names the PAPER.md passage (P:<line>) or the mathematical fact it checks.  A plausible mistake
anywhere in the oracle -- a dropped term, a wrong sign, a transposed operand, a wrong tie rule, a wrong
pruning rule or scan region -- fails at least one of these:

* worked examples E1-E8 (tests/golden/worked_examples.json), hand-derived;
* closed forms (row-0 live extent, identical sequences, transversion-only inputs);
* exhaustive enumeration of every alignment path on tiny inputs with y-drop disabled (recurrences and
  gap convention) -- no DP involved on the reference side;
* an independent pure-Python full-matrix evaluation of the same definitions (cone rule, explored cells,
  peak, traceback) with no banding or lazy V;
* invariants: traceback re-scores to the score and consumes (i*, j*); transposition symmetry; left side
  == right side on reversed sequences; two-sided additivity.
"""
import dataclasses
import json
import os
import random

import numpy as np
import pytest

from oracle import brute, core

HERE = os.path.dirname(os.path.abspath(__file__))
GOLD = json.load(open(os.path.join(HERE, "golden", "worked_examples.json")))
P0 = core.Params()
BASES = "ACGT"


def rseq(rng, n):
    return "".join(rng.choice(BASES) for _ in range(n))


def mutate(rng, s, sub=0.1, indel=0.02):
    out = []
    for ch in s:
        r = rng.random()
        if r < indel / 2:
            continue
        if r < indel:
            out.append(rng.choice(BASES))
        if rng.random() < sub:
            out.append(rng.choice([b for b in BASES if b != ch]))
        else:
            out.append(ch)
    return "".join(out)


def rand_params(rng):
    sub = tuple(tuple(rng.randint(-150, 120) for _ in range(4)) for _ in range(4))  # asymmetric on purpose
    return core.Params(sub=sub, gap_open=rng.choice([0, 1, 50, 400]), gap_extend=rng.choice([1, 7, 30, 200]),
                       ydrop=rng.choice([0, 1, 100, 300, 1000, 9400]))


# ---------------------------------------------------------------- worked examples


@pytest.mark.parametrize("ex", GOLD["one_sided"], ids=lambda e: e["id"])
def test_worked_one_sided(ex):
    """E1-E6: e.g. E2 = 564 (GATTAC) - (O+E = 430) + 655 (GATTACA) = 789."""
    p = dataclasses.replace(P0, ydrop=ex.get("ydrop", P0.ydrop), gap_open=ex.get("gap_open", P0.gap_open))
    s = core.one_sided(ex["A"], ex["B"], p)
    assert (s.score, s.i, s.j, s.ops) == (ex["score"], ex["i"], ex["j"], ex["ops"])


@pytest.mark.parametrize("ex", GOLD["two_sided"], ids=lambda e: e["id"])
def test_worked_two_sided(ex):
    """E7, E8: score = S_L + S_R, endpoints tpos-i_L .. tpos+i_R, left ops reversed into forward order."""
    r = core.extend(ex["T"], ex["Q"], [(ex["tpos"], ex["qpos"])], P0, threads=1)
    rec = r.rec[0]
    for k in ("score", "left_score", "right_score", "t_start", "t_end", "q_start", "q_end"):
        assert rec[k] == ex[k], k
    assert r.cigar_of(0) == ex["cigar"]


# ---------------------------------------------------------------- closed forms


@pytest.mark.parametrize("O,E,Y", [(400, 30, 9400), (0, 1, 5), (100, 7, 1000), (400, 30, 399)])
def test_row0_extent(O, E, Y):
    """Row 0 cell (0,j) has S = -(O + jE) and V(0,j-1) = 0, so it is live iff O + jE <= Y.
    With M = 0 the explored cells are the live ones plus the first dead one."""
    p = dataclasses.replace(P0, gap_open=O, gap_extend=E, ydrop=Y)
    N = 2000
    s = core.one_sided("", "A" * N, p)
    jmax = (Y - O) // E if Y >= O + E else 0
    assert (s.score, s.i, s.j, s.ops) == (0, 0, 0, "")
    assert s.explored == min(jmax, N) + 1 + (1 if jmax < N else 0)
    # transposed: column 0
    s2 = core.one_sided("A" * N, "", p)
    assert s2.explored == s.explored and s2.rows == min(jmax, N) + 1


@pytest.mark.parametrize("n", [1, 5, 40, 300])
def test_identical_sequences(n):
    """Identical sequences under HOXD70 (positive diagonal, gaps cost >= 430): S* = sum of sub(a,a)."""
    rng = random.Random(n)
    a = rseq(rng, n)
    s = core.one_sided(a, a)
    want = sum(P0.sub[BASES.index(c)][BASES.index(c)] for c in a)
    assert (s.score, s.i, s.j, s.ops) == (want, n, n, "M" * n)


def test_transversions_only():
    """Every diagonal pair a transversion (A/G vs C/T): every path scores < 0, the origin is the peak."""
    rng = random.Random(7)
    a = "".join(rng.choice("AG") for _ in range(200))
    b = "".join(rng.choice("CT") for _ in range(200))
    s = core.one_sided(a, b)
    assert (s.score, s.i, s.j, s.ops) == (0, 0, 0, "")


# ---------------------------------------------------------------- exhaustive enumeration


def test_exhaustive_paths():
    """With Y large enough that nothing is pruned, the peak score equals the best score of ANY path from
    the origin (enumerated, affine O + kE per gap run).  Pins P:70-74 and P:71-72 independently of DP."""
    rng = random.Random(1234)
    for trial in range(150):
        p = rand_params(rng)
        p = dataclasses.replace(p, ydrop=10 ** 8)
        a, b = rseq(rng, rng.randint(0, 6)), rseq(rng, rng.randint(0, 6))
        s = core.one_sided(a, b, p)
        want = brute.best_path_score(core.encode(a), core.encode(b), p)
        assert s.score == want, (trial, a, b, p)
        sc, i, j = brute.path_score(core.encode(a), core.encode(b), s.ops, p)
        assert (sc, i, j) == (s.score, s.i, s.j)


# ---------------------------------------------------------------- full matrix vs banded oracle


def _cmp_full(a, b, p):
    s = core.one_sided(a, b, p)
    f = brute.full_matrix(core.encode(a), core.encode(b), p)
    assert (s.score, s.i, s.j, s.ops, s.explored, s.rows) == \
        (f["score"], f["i"], f["j"], f["ops"], f["explored"], f["rows"]), (a, b, p)


def test_full_matrix_random():
    rng = random.Random(99)
    for _ in range(60):
        p = rand_params(rng)
        _cmp_full(rseq(rng, rng.randint(0, 40)), rseq(rng, rng.randint(0, 40)), p)
    # small y-drop on larger inputs: regions whose right edge retreats, so V beyond the previous row's
    # scanned columns must come from earlier rows (the C oracle's per-column maximum)
    for _ in range(40):
        p = dataclasses.replace(rand_params(rng), ydrop=rng.choice([60, 150, 250, 400]))
        a = rseq(rng, 70)
        _cmp_full(a, mutate(rng, a, sub=0.3, indel=0.1) if rng.random() < 0.5 else rseq(rng, 70), p)


def test_full_matrix_homologous_defaults():
    rng = random.Random(5)
    for ln in (30, 80, 150):
        a = rseq(rng, ln)
        for Y in (300, 1000, 9400):
            _cmp_full(a, mutate(rng, a), dataclasses.replace(P0, ydrop=Y))


@pytest.mark.parametrize("case", ["homopolymer", "tandem", "dinuc", "endhit", "junk"])
def test_full_matrix_adversarial(case):
    rng = random.Random(sum(map(ord, case)))
    if case == "homopolymer":
        a, b = "A" * 60, "A" * 45
    elif case == "tandem":
        a, b = "ACG" * 25, "ACG" * 20 + "T"
    elif case == "dinuc":
        a, b = "AT" * 30, "TA" * 30
    elif case == "endhit":
        a = rseq(rng, 12)
        b = a[:10]
    else:
        a, b = rseq(rng, 120), rseq(rng, 120)
    for Y in (0, 1, 300, 1000, 9400, 10 ** 6):
        _cmp_full(a, b, dataclasses.replace(P0, ydrop=Y))
        _cmp_full(a, b, dataclasses.replace(P0, ydrop=Y, gap_open=0))


def test_full_matrix_junk_300bp():
    """A default-scoring random 'junk' extension that explores a large region (the bulk of the workload)."""
    rng = random.Random(11)
    _cmp_full(rseq(rng, 300), rseq(rng, 300), P0)


# ---------------------------------------------------------------- invariants


def test_rescore_and_consume():
    rng = random.Random(3)
    for _ in range(40):
        a = rseq(rng, rng.randint(50, 400))
        b = mutate(rng, a) if rng.random() < 0.7 else rseq(rng, rng.randint(50, 400))
        s = core.one_sided(a, b)
        sc, i, j = brute.path_score(core.encode(a), core.encode(b), s.ops, P0)
        assert (sc, i, j) == (s.score, s.i, s.j)


def test_transpose_symmetry():
    """Swapping target and query with the transposed matrix transposes the DP: score and explored cells
    are identical; the peak position swaps when unique; the (I<->D swapped) path re-scores equal."""
    rng = random.Random(8)
    pt = P0.transposed()
    for _ in range(30):
        p = rand_params(rng) if rng.random() < 0.5 else P0
        ptr = p.transposed()
        a = rseq(rng, rng.randint(0, 200))
        b = mutate(rng, a) if rng.random() < 0.5 else rseq(rng, rng.randint(0, 200))
        s1 = core.one_sided(a, b, p)
        s2 = core.one_sided(b, a, ptr)
        assert s1.score == s2.score and s1.explored == s2.explored
        swapped = s2.ops.translate(str.maketrans("ID", "DI"))
        sc, i, j = brute.path_score(core.encode(a), core.encode(b), swapped, p)
        assert (sc, i, j) == (s1.score, s2.j, s2.i)
    del pt


def test_left_equals_right_on_reversed():
    """the left extension is the one-sided extension of the reversed prefixes."""
    rng = random.Random(21)
    T = rseq(rng, 3000)
    Q = mutate(rng, T)
    seeds = [(rng.randint(0, len(T)), rng.randint(0, len(Q))) for _ in range(20)] + [(1500, 1500)]
    r = core.extend(T, Q, seeds, P0, threads=2)
    for k, (tp, qp) in enumerate(seeds):
        L = core.one_sided(T[:tp][::-1], Q[:qp][::-1])
        R = core.one_sided(T[tp:], Q[qp:])
        rec = r.rec[k]
        assert (rec["left_score"], rec["li"], rec["lj"], rec["l_explored"]) == (L.score, L.i, L.j, L.explored)
        assert (rec["right_score"], rec["ri"], rec["rj"], rec["r_explored"]) == (R.score, R.i, R.j, R.explored)
        assert rec["score"] == L.score + R.score
        assert (rec["t_start"], rec["t_end"], rec["q_start"], rec["q_end"]) == (tp - L.i, tp + R.i, qp - L.j, qp + R.j)
        # CIGAR = reversed left path ++ right path, runs merged
        fwd = L.ops[::-1] + R.ops
        runs, cur, cnt = [], None, 0
        for op in fwd:
            if op == cur:
                cnt += 1
            else:
                if cnt:
                    runs.append(f"{cnt}{cur}")
                cur, cnt = op, 1
        if cnt:
            runs.append(f"{cnt}{cur}")
        assert r.cigar_of(k) == "".join(runs)


def test_threads_deterministic():
    rng = random.Random(4)
    T = rseq(rng, 5000)
    Q = mutate(rng, T)
    seeds = [(rng.randint(0, len(T)), rng.randint(0, len(Q))) for _ in range(64)]
    r1 = core.extend(T, Q, seeds, P0, threads=1)
    r8 = core.extend(T, Q, seeds, P0, threads=8)
    assert np.array_equal(r1.rec, r8.rec) and r1.cigar == r8.cigar


def test_flags_and_eager():
    r = core.extend("GATTACAGATTACAGATTACA", "GATTACGATTACAGATTACA", [(14, 13), (0, 0), (21, 20)], P0, threads=1)
    assert r.rec[0]["flags"] & 1 == 0          # 1444 < K = 3000
    assert r.rec[0]["flags"] & 4               # right peak (7,7) within the 16x16 eager window
    assert r.rec[0]["flags"] & 2               # left peak (14,13): max(i*,j*) = 14 <= 16
    assert not r.rec[2]["flags"] & 2 or r.rec[2]["li"] <= 16
    assert r.rec[1]["score"] == r.rec[1]["right_score"]


def test_bad_inputs():
    with pytest.raises(RuntimeError):
        core.extend("ACGX", "ACGT", [(1, 1)])
    with pytest.raises(RuntimeError):
        core.extend("ACGT", "ACGT", [(5, 1)])


# ---------------------------------------------------------------- N bases (reading R13, NEXT-4)


def test_n_closed_form():
    """An N scores n_score against anything: ACNGT vs ACNGT = 91 + 100 + n + 100 + 91, all matches."""
    for n in (-100, 0):
        p = dataclasses.replace(P0, n_score=n)
        s = core.one_sided("ACNGT", "ACNGT", p)
        assert (s.score, s.i, s.j, s.ops) == (382 + n, 5, 5, "M" * 5)
    # n = -1000: crossing the N (191 - 1000 + 191 < 191) loses to stopping before it; skipping it costs two
    # gap opens (-860), so the peak is (191, 2, 2)
    s = core.one_sided("ACNGT", "ACNGT", dataclasses.replace(P0, n_score=-1000))
    assert (s.score, s.i, s.j, s.ops) == (191, 2, 2, "MM")
    # a deep N run breaks the extension exactly like mismatches of the same score would
    p = dataclasses.replace(P0, n_score=-114)
    a = "A" * 20 + "N" * 10 + "A" * 20
    b = "A" * 20 + "C" * 10 + "A" * 20
    assert core.one_sided(a, "A" * 50, p).score == core.one_sided(b, "A" * 50, P0).score  # sub(C, A) = -114


def test_n_full_matrix_and_paths():
    """Random sequences with N on both sides: banded oracle == full matrix; exhaustive paths == peak."""
    rng = random.Random(4242)
    nseq = lambda k: "".join(rng.choice("ACGTN") for _ in range(k))
    for _ in range(60):
        p = dataclasses.replace(rand_params(rng), n_score=rng.choice([-100, -7, 0, 25]))
        _cmp_full(nseq(rng.randint(0, 40)), nseq(rng.randint(0, 40)), p)
    for trial in range(80):
        p = dataclasses.replace(rand_params(rng), ydrop=10 ** 8, n_score=rng.choice([-100, 0, 40]))
        a, b = nseq(rng.randint(0, 6)), nseq(rng.randint(0, 6))
        s = core.one_sided(a, b, p)
        assert s.score == brute.best_path_score(core.encode(a), core.encode(b), p), (trial, a, b)
