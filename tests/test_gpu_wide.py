"""Explored bands wider than the per-warp boundary ring (the y-drop rule, has no width limit): such
sides are re-inspected and executed with a wider ring (csrc/api.cu).  Bit-exact against the oracle, census
included; plus out-of-range seeds far outside the sequences (ERANGE without touching foreign memory)."""
import random

import numpy as np
import pytest
import torch

from paper_conf_sc_gundaboluvt21_b200 import fastz
from synth import genome
from tests.gpu_util import compare

pytestmark = pytest.mark.gpu
BASES = "ACGT"


def _mut(rng, s, sub=0.1, indel=0.01):
    out = []
    for ch in s:
        r = rng.random()
        if r < indel / 2:
            continue
        if r < indel:
            out.append(rng.choice(BASES))
        out.append(rng.choice([b for b in BASES if b != ch]) if rng.random() < sub else ch)
    return "".join(out)


def test_ydrop_1e6_on_100kbp_mutated_pair():
    """Y = 10^6: row 0 alone stays live for (Y - O) / E = 33,320 columns, beyond the 2^15-entry ring of a
    100 kbp pair.  Target = a 2 kbp piece of the source (so the oracle's full-width region stays small), query =
    the mutated 100 kbp copy; seeds on and off the true diagonal."""
    rng = random.Random(1000000)
    src = "".join(rng.choice(BASES) for _ in range(100_000))
    Q = _mut(rng, src)
    T = src[40_000:42_000]
    seeds = [(0, 40_000), (1000, 40_990), (2000, 42_010), (500, 90_000), (1500, 3_000), (2000, 100_000 - 5000)]
    bad, g, o, st = compare(T, Q, seeds, census=True, ydrop=10 ** 6)
    assert not bad, bad
    assert st["n_wide_sides"] > 0


@pytest.mark.parametrize("entries", ["64", "256"])
def test_forced_small_ring_mixed_workload(monkeypatch, entries):
    """A 64/256-entry ring makes most non-trivial sides overflow: the wide path (repeated 4x growth, wide
    executor launch, wide census) must reproduce the oracle exactly, including multi-wave execution."""
    monkeypatch.setenv("FASTZ_RING_ENTRIES", entries)
    w = genome.small_pair(90, length=20000, n_seeds=200)
    bad, g, o, st = compare(w.T, w.Q, w.seeds, census=True)
    assert not bad, bad
    assert st["n_wide_sides"] > 0
    monkeypatch.setenv("FASTZ_POOL_MB", "1")
    bad, *_ = compare(w.T, w.Q, w.seeds, census=False)
    assert not bad, bad


def test_seeds_far_outside_sequences_are_rejected_safely():
    """Seeds far beyond the sequences: ERANGE, no out-of-bounds reads, and the context and the
    CUDA context stay usable (a following valid batch is exact)."""
    w = genome.small_pair(91, length=12000, n_seeds=60)
    bad_seeds = np.array([[1 << 40, 5], [5, -(1 << 40)], [-7, -7], [w.seeds[0, 0], len(w.Q) + 10 ** 9]], np.int64)
    with fastz.Aligner(w.T, w.Q) as al:
        for k in range(len(bad_seeds)):
            batch = np.concatenate([w.seeds[:20], bad_seeds[k:k + 1], w.seeds[20:]])
            with pytest.raises(fastz.FastzError) as e:
                al.extend(batch)
            assert e.value.status == fastz.FASTZ_ERANGE and "seed 20" in str(e.value)
        torch.cuda.synchronize()
        good = al.extend(w.seeds)
    bad, g, o, _ = compare(w.T, w.Q, w.seeds, census=False)
    assert not bad, bad
    assert np.array_equal(good.rec, g.rec) and good.cigar == g.cigar


def test_executor_self_check_fires(monkeypatch):
    """The executor's self-check (recomputed S(i*, j*) == the inspector's peak) is live: with a
    deliberately wrong expectation (test hook) every executed side fails it and the call returns FASTZ_ECUDA
    naming the count; without the hook the same batch passes and the stats report no failure."""
    w = genome.small_pair(92, length=20000, n_seeds=120)
    with fastz.Aligner(w.T, w.Q) as al:
        al.extend(w.seeds)
        st = al.stats()
        assert st["n_exec_sides"] > 0 and st["n_selfcheck_fail"] == 0
        assert st["exec_words"] <= st["exec_reserved_words"]
        monkeypatch.setenv("FASTZ_TEST_SELFCHECK", "1")
        with pytest.raises(fastz.FastzError) as e:
            al.extend(w.seeds)
        assert e.value.status == fastz.FASTZ_ECUDA and "self-check" in str(e.value)
        assert f"on {st['n_exec_sides']} sides" in str(e.value)
        monkeypatch.delenv("FASTZ_TEST_SELFCHECK")
        al.extend(w.seeds)
