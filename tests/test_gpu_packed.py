"""GPU parity of the packed inspector (csrc/pair.cuh: two one-sided extensions per warp in 16-bit halves, run by
k_inspect_mixed) against the CPU oracle, bit-exact, on the same workloads as test_gpu_parity.  FASTZ_PAIR=2 forces
the packed path on batches too small to choose it by themselves; the knobs exercise each of its branches: the
predicted-long head run by the concurrent 32-bit k_inspect (FASTZ_PAIR_LONG), packed sides abandoned at the value
cap or after FASTZ_PAIR_ESCAPE strips and redone by the 32-bit path, seed order vs predicted order, and parameters
the packed arithmetic cannot hold (the whole batch then falls back to the 32-bit inspector)."""
import random

import numpy as np
import pytest

from synth import genome
from tests.gpu_util import compare, run_both
from tests.test_gpu_parity import mutate, rseq

pytestmark = pytest.mark.gpu


@pytest.fixture
def packed(monkeypatch):
    monkeypatch.setenv("FASTZ_PAIR", "2")
    return monkeypatch


def assert_ok(bad):
    assert not bad, bad


def test_packed_small_mixed(packed):
    seen = {"packed": 0, "long": 0, "redo": 0}
    for seed in range(4):
        w = genome.small_pair(seed, length=20000, n_seeds=200)
        bad, g, o, st = compare(w.T, w.Q, w.seeds)
        assert_ok(bad)
        seen["packed"] += st["n_packed_sides"]
        seen["long"] += st["n_long_sides"]
        seen["redo"] += st["n_redo_sides"]
    # every branch ran: packed sides, the 32-bit predicted-long head, and sides redone in 32 bits
    assert seen["packed"] > 0 and seen["long"] > 0 and seen["redo"] > 0, seen


@pytest.mark.parametrize("knobs", [{"FASTZ_PAIR_LONG": "100000"}, {"FASTZ_INSPECT_ORDER": "0"},
                                   {"FASTZ_PAIR_ESCAPE": "1"}, {"FASTZ_PAIR_ESCAPE": "3", "FASTZ_PAIR_LONG": "0"}],
                         ids=["all-packed", "seed-order", "escape-1", "escape-3-all-long"])
def test_packed_knobs(packed, knobs):
    for k, v in knobs.items():
        packed.setenv(k, v)
    w = genome.small_pair(21, length=20000, n_seeds=256)
    bad, g, o, st = compare(w.T, w.Q, w.seeds)
    assert_ok(bad)
    if knobs.get("FASTZ_PAIR_LONG") == "100000" or "FASTZ_INSPECT_ORDER" in knobs:
        assert st["n_long_sides"] == 0 and st["n_packed_sides"] == 2 * len(w.seeds)


def test_packed_equals_32bit(packed):
    """Per-side peaks, flags, executor bounds are the same whichever inspector ran a side."""
    w = genome.small_pair(5, length=40000, n_seeds=1024)
    g1, s1, _, st1, _ = run_both(w.T, w.Q, w.seeds)
    packed.setenv("FASTZ_PAIR", "0")
    g0, s0, _, st0, _ = run_both(w.T, w.Q, w.seeds)
    assert st1["n_packed_sides"] > 0 and st0["n_packed_sides"] == 0
    for a, b in zip(s0, s1):
        assert np.array_equal(a, b)
    assert np.array_equal(g0.rec, g1.rec) and bytes(g0.cigar) == bytes(g1.cigar)
    # the packed path sizes its sides' executor storage exactly from the strip history; the executor writes
    # the same codes either way and its self-check keeps every store inside the reservation
    assert st0["exec_words"] == st1["exec_words"]
    assert st1["exec_words"] <= st1["exec_reserved_words"] <= st0["exec_reserved_words"]


@pytest.mark.parametrize("Y", [0, 1, 50, 1000, 9400, 20000, 32000, 40000])
def test_packed_ydrop_values(packed, Y):
    rng = random.Random(Y + 3)
    T = rseq(rng, 2000)
    Q = mutate(rng, T)
    seeds = [(rng.randint(0, 2000), rng.randint(0, len(Q))) for _ in range(40)]
    bad, *_ = compare(T, Q, seeds, ydrop=Y)
    assert_ok(bad)


@pytest.mark.parametrize("O,E", [(0, 1), (0, 30), (400, 1), (400, 30), (3000, 1)])
def test_packed_gap_parameters(packed, O, E):
    rng = random.Random(O * 7 + E)
    T = rseq(rng, 1500)
    Q = mutate(rng, T, sub=0.15, indel=0.05)
    seeds = [(rng.randint(0, 1500), rng.randint(0, len(Q))) for _ in range(40)]
    bad, *_ = compare(T, Q, seeds, gap_open=O, gap_extend=E)
    assert_ok(bad)


def test_packed_random_scoring_matrices(packed):
    rng = random.Random(78)
    for trial in range(6):
        sub = [[rng.randint(-150, 120) for _ in range(4)] for _ in range(4)]
        T = rseq(rng, 1500)
        Q = mutate(rng, T, sub=0.2)
        seeds = [(rng.randint(0, 1500), rng.randint(0, len(Q))) for _ in range(30)]
        bad, *_ = compare(T, Q, seeds, sub=sub, gap_open=rng.choice([0, 100, 400]),
                          gap_extend=rng.choice([5, 30]), ydrop=rng.choice([200, 1000, 9400]))
        assert_ok(bad)


@pytest.mark.parametrize("kind", ["homopolymer", "tandem", "dinuc"])
def test_packed_adversarial_wide_bands(packed, kind):
    if kind == "homopolymer":
        T, Q = "A" * 3000, "A" * 2500
    elif kind == "tandem":
        T, Q = "ACGTTG" * 500, "ACGTTG" * 450 + "ACG"
    else:
        T, Q = "AT" * 1500, "TA" * 1400
    seeds = [(0, 0), (1000, 1000), (1500, 900), (len(T), len(Q)), (2000, 2400)]
    bad, *_ = compare(T, Q, seeds)
    assert_ok(bad)


def test_packed_long_homologous(packed):
    """Long alignments reach the 16-bit value cap inside the packed inspector and are redone in 32 bits."""
    packed.setenv("FASTZ_PAIR_LONG", "100000")
    rng = random.Random(9)
    T = rseq(rng, 12000)
    Q = mutate(rng, T, sub=0.08, indel=0.01)
    seeds = [(6000, int(len(Q) * 0.5)), (0, 0), (12000, len(Q)), (3000, int(len(Q) * 0.25))]
    bad, g, o, st = compare(T, Q, seeds)
    assert_ok(bad)
    assert st["n_redo_sides"] >= 4, st


def test_packed_edges(packed):
    T, Q = "ACGT" * 50, "ACGA" * 50
    seeds = [(0, 0), (200, 200), (0, 200), (200, 0), (100, 100), (1, 199), (199, 1)]
    bad, *_ = compare(T, Q, seeds)
    assert_ok(bad)
    bad, *_ = compare("A", "A", [(0, 0), (1, 1), (0, 1), (1, 0)])
    assert_ok(bad)


@pytest.mark.parametrize("entries", ["64", "256"])
def test_packed_ring_overflow_goes_wide(packed, entries):
    """Packed sides whose band outgrows a small boundary ring are flagged (SF_RING) like 32-bit ones and
    re-inspected with the wide ring by the 32-bit inspector; the batch stays exact."""
    packed.setenv("FASTZ_RING_ENTRIES", entries)
    packed.setenv("FASTZ_PAIR_LONG", "100000")  # every side starts packed
    w = genome.small_pair(91, length=20000, n_seeds=200)
    bad, g, o, st = compare(w.T, w.Q, w.seeds, census=True)
    assert_ok(bad)
    assert st["n_wide_sides"] > 0 and st["n_packed_sides"] == 2 * len(w.seeds)


def test_packed_ydrop_1e4_low_identity(packed):
    """Y just above the default (10^4) on a low-identity pair: wide y-drop blobs, many strips per packed side."""
    rng = random.Random(10 ** 4)
    T = rseq(rng, 4000)
    Q = mutate(rng, T, sub=0.3, indel=0.05)
    seeds = [(rng.randint(0, 4000), rng.randint(0, len(Q))) for _ in range(60)]
    bad, *_ = compare(T, Q, seeds, ydrop=10000)
    assert_ok(bad)
