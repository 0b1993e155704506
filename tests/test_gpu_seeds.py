"""GPU parity of the seeding + ungapped filter stage (NEXT-4, readings S1-S6; include/fastz.h
fastz_find_hsps) against the C oracle (oracle/seed_oracle.c), through the C ABI.  Integer work: the HSP
lists (t_start, q_start, length, score, in anchor order) and the raw hit counts must be identical."""
import numpy as np
import pytest

from oracle import core, seeds
from paper_conf_sc_gundaboluvt21_b200 import fastz
from synth import genome
from tests.gpu_util import compare

pytestmark = pytest.mark.gpu


def both(T, Q, pattern=seeds.PATTERN_12OF19, transitions=True, xdrop=910, hspthresh=3000, sub=core.HOXD70):
    with fastz.Aligner(T, Q, fastz.fastz_default_params(sub=np.asarray(sub).reshape(16))) as al:
        g, an, gh = al.find_hsps(pattern=pattern, transitions=transitions, xdrop=xdrop, hspthresh=hspthresh)
    o, oh = seeds.find_hsps(T, Q, sub, pattern, transitions, xdrop, hspthresh)
    return g, an, gh, o, oh


def assert_same(g, an, gh, o, oh):
    assert gh == oh
    assert len(g) == len(o)
    for f in ("t_start", "q_start", "length", "score"):
        assert np.array_equal(g[f].astype(np.int64), o[f].astype(np.int64)), f
    assert np.array_equal(an[:, 0], o["t_start"] + o["length"] // 2)
    assert np.array_equal(an[:, 1], o["q_start"] + o["length"] // 2)


@pytest.mark.parametrize("pattern,transitions,thr", [
    (seeds.PATTERN_12OF19, True, 3000), (seeds.PATTERN_12OF19, False, 3000), (seeds.PATTERN_12OF19, True, 500),
    ("111", False, 300), ("1101011", True, 400),
    ("11111111111111", True, 1000),                     # w = 14: binary-search bucket path
    ("1" + "01" * 14 + "001", True, 2000),               # span 32, 16 care positions
])
def test_small_pair(pattern, transitions, thr):
    w = genome.small_pair(3, length=30000, n_seeds=8)
    assert_same(*both(w.T, w.Q, pattern, transitions, 910, thr))


def test_c1_pair_and_chunking(monkeypatch):
    w = genome.config1(n_seeds=16)
    ref = both(w.T, w.Q)
    assert_same(*ref)
    assert len(ref[0]) > 100
    # tiny hit buffer: many query chunks (and chunk halving), identical result
    monkeypatch.setenv("FASTZ_SEED_HIT_CAP", "3000")
    assert_same(*both(w.T, w.Q))


def test_edges():
    # sequences shorter than the span, no hits at all, an asymmetric matrix
    assert_same(*both("ACGTACGTAC", "ACGTACGTAC"))
    assert_same(*both("A" * 5000, "C" * 5000))
    rng = np.random.default_rng(5)
    sub = rng.integers(-150, 120, (4, 4))
    w = genome.small_pair(4, length=20000, n_seeds=8)
    assert_same(*both(w.T, w.Q, "1101011", True, 300, 200, sub))


def test_homopolymer_repeats():
    # long exact repeats: huge buckets and many hits collapsing onto few HSPs
    T = "ACGT" * 500 + "A" * 300 + "GATTACA" * 100
    Q = "A" * 200 + "ACGT" * 300 + "GATTACA" * 50
    assert_same(*both(T, Q, "111", True, 910, 300))


def test_pipeline_seeds_to_alignments():
    """find_hsps -> anchors -> extend: the gapped results on the GPU's anchors equal the oracle's."""
    w = genome.small_pair(6, length=40000, n_seeds=8)
    with fastz.Aligner(w.T, w.Q) as al:
        hs, an, _ = al.find_hsps()
    assert len(an) > 5
    bad, g, o, stats = compare(w.T, w.Q, an, census=False)
    assert not bad, bad


def revcomp(s: str) -> str:
    return s.translate(str.maketrans("ACGTacgt", "TGCAtgca"))[::-1]


def test_minus_strand():
    """FASTZ_OPT_QUERY_REVCOMP (32): the context aligns against the reverse complement of the query; HSPs and
    gapped alignments equal the oracle's on the explicitly reverse-complemented string."""
    w = genome.small_pair(7, length=30000, n_seeds=8)
    T = w.T.decode() if isinstance(w.T, bytes) else w.T
    Q = w.Q.decode() if isinstance(w.Q, bytes) else w.Q
    Qm = revcomp(T[5000:9000]) + Q[4000:20000] + revcomp(T[15000:17000])  # minus-strand homology
    rc = revcomp(Qm)
    with fastz.Aligner(T, Qm, fastz.fastz_default_params(options=32)) as al:
        g, an, gh = al.find_hsps()
        ga = al.extend(an)
    o, oh = seeds.find_hsps(T, rc, core.HOXD70)
    assert_same(g, an, gh, o, oh)
    assert len(o) >= 2
    orr = core.extend(T, rc, an, core.Params())
    for f in ("score", "t_start", "t_end", "q_start", "q_end"):
        assert np.array_equal(ga.rec[f].astype(np.int64), orr.rec[f]), f
    assert all(ga.cigar_of(s) == orr.cigar_of(s) for s in range(len(an)))
    # invalid character reported at its index in the caller's string
    with pytest.raises(fastz.FastzError, match="index"):
        fastz.Aligner(T, Qm[:100] + "X" + Qm[101:], fastz.fastz_default_params(options=32))


def with_ns(s: str, rng, k: int, run: int = 1) -> str:
    s = list(s)
    for p in rng.choice(len(s) - run, k, replace=False):
        for d in range(run):
            s[p + d] = "N"
    return "".join(s)


@pytest.mark.parametrize("n_score", [-100, 0])
def test_n_bases_seeding_and_pipeline(n_score):
    """N (reading R13 / S7) on both sequences, both strands: HSPs equal the oracle's; anchors -> gapped parity."""
    rng = np.random.default_rng(11)
    w = genome.small_pair(9, length=30000, n_seeds=8)
    T = with_ns(w.T.decode(), rng, 60) ; T = with_ns(T, rng, 3, run=40)
    Q = with_ns(w.Q.decode(), rng, 60)
    for opts, Qo in ((0, Q), (32, revcomp(Q))):
        with fastz.Aligner(T, Q, fastz.fastz_default_params(options=opts, n_score=n_score)) as al:
            g, an, gh = al.find_hsps()
            ga = al.extend(an)
        o, oh = seeds.find_hsps(T, Qo, core.HOXD70, n_score=n_score)
        assert_same(g, an, gh, o, oh)
        orr = core.extend(T, Qo, an, core.Params(n_score=n_score))
        for f in ("score", "t_start", "t_end", "q_start", "q_end"):
            assert np.array_equal(ga.rec[f].astype(np.int64), orr.rec[f]), f
        assert all(ga.cigar_of(s) == orr.cigar_of(s) for s in range(len(an)))
