"""GPU parity of the redundant-alignment post-pass (``fastz_mark_redundant``, csrc/dedup.cu; NEXT-3, reading
R14) through the C ABI.

Small mixed workloads: the CUDA marks equal, element by element, those of ``oracle/dedup.py`` applied to the
extension ORACLE's records for the same seeds (no oracle input comes from the CUDA path).  Full-size C2 (the
bench batch): the marks are checked against the defining property at any size -- a candidate is marked iff
some candidate dominates it -- evaluated independently in numpy over a t_start-sorted window."""
import numpy as np
import pytest

from oracle import core, dedup
from paper_conf_sc_gundaboluvt21_b200 import fastz
from synth import genome
from tests.gpu_util import gparams, oparams

pytestmark = pytest.mark.gpu


def gpu_marks(T, Q, seeds, **kw):
    with fastz.Aligner(T, Q, gparams(**kw)) as al:
        al.extend_only(seeds)
        red, cnt = al.mark_redundant()
        rec = al.results().rec
        red2, cnt2 = al.mark_redundant()   # idempotent
    assert np.array_equal(red, red2) and cnt == cnt2
    assert cnt == int(red.sum())
    assert np.array_equal((rec["flags"] & fastz.FLAG_REDUNDANT) != 0, red.astype(bool))
    return red, rec


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("K", [3000, 0])
def test_small_pairs_match_oracle(seed, K):
    w = genome.small_pair(seed, length=20_000, n_seeds=400)
    red, rec = gpu_marks(w.T, w.Q, w.seeds, gapped_threshold=K)
    o = core.extend(w.T, w.Q, w.seeds, oparams(gapped_threshold=K))
    exp = dedup.redundant(o.rec)
    bad = np.nonzero(red != exp)[0]
    assert len(bad) == 0, (bad[:10].tolist(), red[bad[:10]].tolist(), exp[bad[:10]].tolist())
    if K == 0:
        assert exp.sum() > 0   # the case exercises marking


def test_identical_sequences_keep_the_first_seed():
    rng = np.random.default_rng(5)
    T = genome.to_ascii(genome.random_codes(rng, 3000))
    pos = [1500, 10, 2999, 700, 700, 1]
    seeds = np.array([[p, p] for p in pos], dtype=np.int64)
    red, rec = gpu_marks(T, T, seeds)
    assert (rec["t_start"] == 0).all() and (rec["t_end"] == 3000).all()
    assert red.tolist() == [0, 1, 1, 1, 1, 1]


def test_marks_reset_by_the_next_extend():
    w = genome.small_pair(9, n_seeds=300)
    with fastz.Aligner(w.T, w.Q, gparams(gapped_threshold=0)) as al:
        al.extend_only(w.seeds)
        _, cnt = al.mark_redundant()
        assert cnt > 0
        rec = al.extend(w.seeds).rec
        assert not (rec["flags"] & fastz.FLAG_REDUNDANT).any()


def test_empty_batch_and_state_errors():
    T = b"ACGT" * 100
    with fastz.Aligner(T, T) as al:
        with pytest.raises(fastz.FastzError) as e:
            al.mark_redundant()
        assert e.value.status == fastz.FASTZ_ESTATE
        al.extend_only(np.zeros((0, 2), np.int64))
        red, cnt = al.mark_redundant()
        assert len(red) == 0 and cnt == 0


def maximal_marks(rec):
    """Independent numpy evaluation: candidate a is marked iff some candidate dominates it (R14)."""
    cand = np.nonzero(rec["flags"] & fastz.FLAG_ABOVE_K)[0]
    t0, t1 = rec["t_start"][cand], rec["t_end"][cand]
    q0, q1, sc = rec["q_start"][cand], rec["q_end"][cand], rec["score"][cand]
    order = np.argsort(t0, kind="stable")
    t0s = t0[order]
    maxlen = int((t1 - t0).max()) if len(cand) else 0
    out = np.zeros(len(rec), np.uint8)
    for k in range(len(cand)):
        lo, hi = np.searchsorted(t0s, t0[k] - maxlen, "left"), np.searchsorted(t0s, t0[k], "right")
        j = order[lo:hi]
        j = j[j != k]
        box = (t0[j] <= t0[k]) & (t1[j] >= t1[k]) & (q0[j] <= q0[k]) & (q1[j] >= q1[k]) & (sc[j] >= sc[k])
        same = (t0[j] == t0[k]) & (t1[j] == t1[k]) & (q0[j] == q0[k]) & (q1[j] == q1[k])
        tie_ok = ~same | (sc[j] > sc[k]) | (cand[j] < cand[k])
        out[cand[k]] = np.any(box & tie_ok)
    return out


def test_c2_full_batch_maximality():
    w = genome.config2()
    with fastz.Aligner(w.T, w.Q) as al:
        al.extend_only(w.seeds)
        red, cnt = al.mark_redundant()
        rec = al.results().rec
    assert cnt == int(red.sum()) and cnt > 0
    assert np.array_equal(red, maximal_marks(rec))


def oracle_records(o):
    rec = np.zeros(len(o.rec), dtype=fastz.ALIGN_DTYPE)
    for f in ("score", "left_score", "right_score", "flags", "t_start", "t_end", "q_start", "q_end"):
        rec[f] = o.rec[f]
    return rec


@pytest.mark.parametrize("seed", range(3))
def test_context_free_records_match_oracle(seed):
    """fastz_mark_redundant_records on ORACLE records held on the host (gathered-set use, dist.py)."""
    w = genome.small_pair(40 + seed, length=20_000, n_seeds=300)
    o = core.extend(w.T, w.Q, w.seeds, oparams(gapped_threshold=1000))
    rec = oracle_records(o)
    rec["flags"] |= fastz.FLAG_REDUNDANT * (np.arange(len(rec)) % 2).astype(np.uint32)  # stale bits are recomputed
    red, cnt = fastz.fastz_mark_redundant_records(rec)
    exp = dedup.redundant(o.rec)
    assert np.array_equal(red, exp) and cnt == int(exp.sum()) and cnt > 0
    assert np.array_equal((rec["flags"] & fastz.FLAG_REDUNDANT) != 0, exp.astype(bool))
    assert np.array_equal(rec["flags"] & ~np.uint32(fastz.FLAG_REDUNDANT), o.rec["flags"].astype(np.uint32))


def test_context_free_empty_and_bad_args():
    rec = np.zeros(0, dtype=fastz.ALIGN_DTYPE)
    red, cnt = fastz.fastz_mark_redundant_records(rec)
    assert len(red) == 0 and cnt == 0
    with pytest.raises(ValueError):
        fastz.fastz_mark_redundant_records(np.zeros(3, np.int64))


def test_context_free_device_records():
    """recs_on_device = 1: records in device memory (a torch buffer), flags recomputed in place on the GPU."""
    import ctypes

    import torch
    w = genome.small_pair(50, length=20_000, n_seeds=300)
    o = core.extend(w.T, w.Q, w.seeds, oparams(gapped_threshold=0))
    rec = oracle_records(o)
    buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
    red = np.zeros(len(rec), np.uint8)
    cnt = ctypes.c_int64()
    st = fastz.lib().fastz_mark_redundant_records(buf.data_ptr(), len(rec), 1, red.ctypes.data, ctypes.byref(cnt), 0)
    assert st == 0
    exp = dedup.redundant(o.rec)
    assert np.array_equal(red, exp) and cnt.value == int(exp.sum()) > 0
    back = buf.cpu().numpy().view(fastz.ALIGN_DTYPE)
    assert np.array_equal((back["flags"] & fastz.FLAG_REDUNDANT) != 0, exp.astype(bool))
