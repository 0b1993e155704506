"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element, bit-exact
(all arithmetic is integer).  Compared per seed: score, left/right scores, endpoints, flags, CIGAR; per
side: peak (score, i*, j*); and the explored-cell census (the GCUPS numerator) against the oracle's count.
"""
import json
import os
import random

import numpy as np
import pytest

from synth import genome
from tests.gpu_util import compare, run_both

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))
GOLD = json.load(open(os.path.join(HERE, "golden", "worked_examples.json")))
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
        out.append(rng.choice([b for b in BASES if b != ch]) if rng.random() < sub else ch)
    return "".join(out)


def assert_ok(bad):
    assert not bad, bad


@pytest.mark.parametrize("ex", GOLD["two_sided"], ids=lambda e: e["id"])
def test_worked_two_sided(ex):
    bad, g, o, _ = compare(ex["T"], ex["Q"], [(ex["tpos"], ex["qpos"])])
    assert_ok(bad)
    assert g.cigar_of(0) == ex["cigar"] and int(g.rec[0]["score"]) == ex["score"]


@pytest.mark.parametrize("ex", GOLD["one_sided"], ids=lambda e: e["id"])
def test_worked_one_sided_as_right_side(ex):
    kw = {k: ex[k] for k in ("ydrop", "gap_open") if k in ex}
    bad, g, o, _ = compare(ex["A"], ex["B"], [(0, 0)], **kw)
    assert_ok(bad)
    assert int(g.rec[0]["right_score"]) == ex["score"]


def test_small_mixed_workloads():
    for seed in range(4):
        w = genome.small_pair(seed, length=20000, n_seeds=200)
        bad, *_ = compare(w.T, w.Q, w.seeds)
        assert_ok(bad)


def test_edges_empty_sides_and_sequence_ends():
    rng = random.Random(5)
    T = rseq(rng, 3000)
    Q = mutate(rng, T)
    seeds = [(0, 0), (len(T), len(Q)), (0, len(Q)), (len(T), 0), (1, 1), (len(T) - 1, len(Q) - 1),
             (1500, 1500), (1500, 0), (0, 1500)]
    bad, *_ = compare(T, Q, seeds)
    assert_ok(bad)


def test_empty_batch_and_tiny_sequences():
    g, sides, cells, stats, o = run_both("A", "C", np.zeros((0, 2), np.int64))
    assert len(g.rec) == 0 and g.cigar == b""
    bad, *_ = compare("A", "A", [(0, 0), (1, 1), (0, 1), (1, 0)])
    assert_ok(bad)


@pytest.mark.parametrize("Y", [0, 1, 300, 9400, 10 ** 6])
def test_ydrop_values(Y):
    rng = random.Random(Y)
    T = rseq(rng, 4000)
    Q = mutate(rng, T, sub=0.15)
    seeds = [(rng.randint(0, 4000), rng.randint(0, len(Q))) for _ in range(40)] + \
            [(k, k) for k in range(100, 4000, 400)]
    bad, *_ = compare(T, Q, seeds, ydrop=Y)
    assert_ok(bad)


@pytest.mark.parametrize("O,E", [(0, 30), (400, 1), (50, 200), (0, 1)])
def test_gap_parameters(O, E):
    rng = random.Random(O * 1000 + E)
    T = rseq(rng, 3000)
    Q = mutate(rng, T, sub=0.1, indel=0.05)
    seeds = [(k, min(k, len(Q))) for k in range(0, 3000, 150)]
    bad, *_ = compare(T, Q, seeds, gap_open=O, gap_extend=E, ydrop=min(9400, O + 300 * E))
    assert_ok(bad)


def test_random_scoring_matrices():
    rng = random.Random(77)
    for trial in range(6):
        sub = [[rng.randint(-150, 120) for _ in range(4)] for _ in range(4)]
        T = rseq(rng, 1500)
        Q = mutate(rng, T, sub=0.2)
        seeds = [(rng.randint(0, 1500), rng.randint(0, len(Q))) for _ in range(30)]
        bad, *_ = compare(T, Q, seeds, sub=sub, gap_open=rng.choice([0, 100, 400]),
                          gap_extend=rng.choice([5, 30]), ydrop=rng.choice([200, 1000, 9400]))
        assert_ok(bad)


@pytest.mark.parametrize("kind", ["homopolymer", "tandem", "dinuc"])
def test_adversarial_wide_bands(kind):
    if kind == "homopolymer":
        T, Q = "A" * 3000, "A" * 2500
    elif kind == "tandem":
        T, Q = "ACGTTG" * 500, "ACGTTG" * 450 + "ACG"
    else:
        T, Q = "AT" * 1500, "TA" * 1400
    seeds = [(0, 0), (1000, 1000), (1500, 900), (len(T), len(Q)), (2000, 2400)]
    bad, *_ = compare(T, Q, seeds)
    assert_ok(bad)


def test_long_homologous_multi_strip():
    """Alignments spanning many strips (strip height 32*R rows) and long executor traceback."""
    rng = random.Random(9)
    T = rseq(rng, 12000)
    Q = mutate(rng, T, sub=0.08, indel=0.01)
    seeds = [(6000, int(len(Q) * 0.5)), (0, 0), (12000, len(Q))]
    # exact 12-mer seeds on the diagonal
    w = genome.config1(n_seeds=64)
    bad, *_ = compare(T, Q, seeds)
    assert_ok(bad)
    bad, *_ = compare(w.T, w.Q, w.seeds[:16], census=False)
    assert_ok(bad)


def test_deterministic_repeat():
    w = genome.small_pair(11, length=20000, n_seeds=300)
    g1, *_ = run_both(w.T, w.Q, w.seeds)
    g2, *_ = run_both(w.T, w.Q, w.seeds)
    assert np.array_equal(g1.rec, g2.rec) and g1.cigar == g2.cigar


def test_large_scores():
    """Large scoring parameters (|sub| up to 24k, O + E = 8600, Y = 188000): substitution values with O + E
    folded in stay exact in the kernels' int32 table and all scores stay far inside the int32 range."""
    hox = np.array([[91, -114, -31, -123], [-114, 100, -125, -31], [-31, -125, 100, -114], [-123, -31, -114, 91]])
    rng = random.Random(123)
    T = rseq(rng, 3000)
    Q = mutate(rng, T)
    seeds = [(rng.randint(0, 3000), rng.randint(0, len(Q))) for _ in range(30)] + [(1500, 1500)]
    bad, *_ = compare(T, Q, seeds, sub=hox * 200, gap_open=8000, gap_extend=600, ydrop=8000 + 300 * 600,
                      gapped_threshold=600000)
    assert_ok(bad)


@pytest.fixture
def force_block(monkeypatch):
    """Every side that needs more than one strip escalates to the block-per-side inspector and every executed
    side runs block per side (pipelined strips across the CTA's warps)."""
    monkeypatch.setenv("FASTZ_ESCALATE_STRIPS", "1")
    monkeypatch.setenv("FASTZ_BLOCK_BIN", "1")


def test_block_per_side_mixed(force_block):
    for seed in range(2):
        w = genome.small_pair(40 + seed, length=20000, n_seeds=200)
        bad, *_ = compare(w.T, w.Q, w.seeds, census=False)
        assert_ok(bad)


def test_block_per_side_long_and_adversarial(force_block):
    rng = random.Random(19)
    T = rseq(rng, 9000)
    Q = mutate(rng, T, sub=0.08, indel=0.01)
    seeds = [(4500, int(len(Q) * 0.5)), (0, 0), (9000, len(Q)), (100, 90)]
    bad, *_ = compare(T, Q, seeds, census=False)
    assert_ok(bad)
    for Y in (0, 300, 10 ** 6):
        bad, *_ = compare(T[:3000], Q[:3000], [(1500, 1500), (0, 0), (3000, 3000)], census=False, ydrop=Y)
        assert_ok(bad)
    bad, *_ = compare("A" * 3000, "A" * 2500, [(0, 0), (1000, 1000), (3000, 2500)], census=False)
    assert_ok(bad)


def test_block_inspector_only(monkeypatch):
    """Escalation after 2 strips with the default executor split."""
    monkeypatch.setenv("FASTZ_ESCALATE_STRIPS", "2")
    w = genome.small_pair(50, length=30000, n_seeds=150)
    bad, *_ = compare(w.T, w.Q, w.seeds, census=False)
    assert_ok(bad)


def test_executor_waves_under_pool_budget(monkeypatch):
    """A 1 MiB traceback-code budget forces the executor + traceback into many waves (list ranges)."""
    monkeypatch.setenv("FASTZ_POOL_MB", "1")
    w = genome.small_pair(60, length=30000, n_seeds=200)
    bad, *_ = compare(w.T, w.Q, w.seeds, census=False)
    assert_ok(bad)
    rng = random.Random(61)
    T = rseq(rng, 6000)
    Q = mutate(rng, T, sub=0.08, indel=0.01)
    bad, *_ = compare(T, Q, [(3000, int(len(Q) * 0.5)), (0, 0), (6000, len(Q)), (10, 10)], census=False)
    assert_ok(bad)


@pytest.mark.parametrize("opt", [1, 2, 4, 8, 1 | 2 | 4 | 8])
def test_ablation_options_do_not_change_results(opt):
    """FASTZ_OPT_NO_EAGER / NO_TRIM / NO_BINNING / NO_BLOCK (the paper's Fig. 9 variants) change
    only the work, never the alignments."""
    w = genome.small_pair(70, length=30000, n_seeds=200)
    rng = random.Random(71)
    T = rseq(rng, 5000)
    Q = mutate(rng, T, sub=0.08, indel=0.01)
    for TT, QQ, seeds in ((w.T, w.Q, w.seeds), (T, Q, [(2500, int(len(Q) * 0.5)), (0, 0), (5000, len(Q))])):
        bad, *_ = compare(TT, QQ, seeds, census=False, options=opt)
        assert_ok(bad)


def test_traceback_above_k_only():
    """FASTZ_OPT_TRACEBACK_ABOVE_K (NEXT-3): seeds below K keep score and endpoints but get no CIGAR."""
    from paper_conf_sc_gundaboluvt21_b200 import fastz as fz
    w = genome.small_pair(72, length=30000, n_seeds=300)
    g0, *_ = run_both(w.T, w.Q, w.seeds)
    with fz.Aligner(w.T, w.Q, fz.fastz_default_params(options=fz.OPT_TRACEBACK_ABOVE_K)) as al:
        g1 = al.extend(w.seeds)
    for f in ("score", "t_start", "t_end", "q_start", "q_end"):
        assert np.array_equal(g0.rec[f], g1.rec[f])
    above = g0.rec["score"] >= 3000
    assert above.any() and (~above).any()
    for s in range(len(w.seeds)):
        if above[s]:
            assert g1.cigar_of(s) == g0.cigar_of(s)
        else:
            assert g1.rec["cigar_len"][s] == 0 and g1.rec["flags"][s] & fz.FLAG_NO_CIGAR


@pytest.mark.parametrize("n_score", [-100, 0, 60])
def test_n_bases(n_score):
    """N bases (reading R13: any pair with an N scores n_score) in both sequences, isolated and in runs, on a
    mixed workload: bit-exact per seed and per side, explored-cell census included."""
    rng = np.random.default_rng(500 + n_score)
    w = genome.small_pair(21, length=20000, n_seeds=300)
    def with_ns(s, k, run):
        s = bytearray(s)
        for p in rng.choice(len(s) - run, k, replace=False):
            s[p:p + run] = b"N" * run
        return bytes(s)
    T = with_ns(with_ns(w.T, 200, 1), 5, 30)
    Q = with_ns(with_ns(w.Q, 200, 1), 5, 30).lower()
    assert_ok(compare(T, Q, w.seeds, census=True, n_score=n_score)[0])
