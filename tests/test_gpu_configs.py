"""Bit-exact parity on every BASELINE config at full size, in the launch configuration bench.py times
(PyTorch stream, PyTorch caching allocator, device-resident seeds, the whole batch in one
fastz_extend_seeds call).

Per config the whole batch is checked for properties that hold at any size (every CIGAR is well formed, walks
through its seed's cut point, and its left/right parts re-score to the reported per-side scores:
oracle/rescore.c), and a stratified sample is compared with the CPU oracle field by field and CIGAR by CIGAR
(score, left/right scores, endpoints, flags, per-side peaks i*/j*):

* C1 (2,048 seeds): every seed;
* C2, C3, C5, C6: every seed with a side in bin >= 2 (max(i*, j*) > 512; the bins come from the GPU's
  per-side peaks, which are themselves compared) plus 2,000 random seeds;
* C4 (2^23 seeds): >= 5,000 seeds stratified by bin (all bins >= 3, up to 2,000 of bin 2, 1,500 of bin 1,
  1,000 eager seeds).

The oracle (the paper's method written out plainly) runs on all host cores.
"""
import os
import time

import numpy as np
import pytest
import torch

from oracle import core, rescore
from paper_conf_sc_gundaboluvt21_b200 import fastz
from synth import genome
from tests.gpu_util import FIELDS

pytestmark = pytest.mark.gpu
BIN_EDGES = np.array([16, 512, 2048, 8192, 32768, 131072])  # bin 0 = eager (<= 16), then P:211's bins


def run_bench_config(w):
    """One fastz_extend_seeds over the whole batch exactly as bench.py launches it."""
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream(dev)
    al = fastz.Aligner(w.T, w.Q, device=0, stream=stream.cuda_stream, torch_alloc=True)
    try:
        al.extend_only(torch.from_numpy(np.ascontiguousarray(w.seeds)).to(dev))
        g = al.results()
        sides = al.sides()
        st = al.stats()
    finally:
        al.close()
        torch.cuda.empty_cache()  # the context's pool came from PyTorch's cache: give it back to the driver
    return g, sides, st


def seed_bins(ti, qj):
    m = np.maximum(ti, qj).reshape(-1, 2).max(axis=1)
    return np.searchsorted(BIN_EDGES, m, side="left")


def stratified(bins, rng, n_random=2000, per_bin=None):
    if per_bin is None:  # every seed in bins >= 2 plus random ones
        long = np.nonzero(bins >= 2)[0]
        rest = np.setdiff1d(np.arange(len(bins)), long)
        pick = rng.choice(rest, min(n_random, len(rest)), replace=False)
        return np.sort(np.concatenate([long, pick]))
    out = []
    for b in range(bins.max() + 1):
        idx = np.nonzero(bins == b)[0]
        k = per_bin.get(b, len(idx))
        out.append(idx if k >= len(idx) else rng.choice(idx, k, replace=False))
    return np.sort(np.concatenate(out))


def check_config(w, sample_fn, min_sample=0):
    t0 = time.time()
    g, (sc, ti, qj, fl), st = run_bench_config(w)
    rec = g.rec
    n = len(w.seeds)
    assert len(rec) == n and st["n_sides"] == 2 * n
    # whole batch: score = left + right, CIGARs re-score per side and pass through the cut points
    nbad, why = rescore.rescore(w.T, w.Q, w.seeds, rec, g.cigar)
    assert nbad == 0, (nbad, [(int(s), rescore.REASONS[int(why[s])]) for s in np.nonzero(why)[0][:5]])
    assert np.array_equal(rec["left_score"], sc[0::2]) and np.array_equal(rec["right_score"], sc[1::2])
    # stratified oracle sample
    bins = seed_bins(ti, qj)
    idx = sample_fn(bins)
    assert len(idx) >= min_sample
    t1 = time.time()
    o = core.extend(w.T, w.Q, w.seeds[idx], threads=os.cpu_count())
    t2 = time.time()
    bad = []
    for f in FIELDS:
        d = np.nonzero(rec[f][idx].astype(np.int64) != o.rec[f])[0]
        if len(d):
            bad.append((f, idx[d[:3]].tolist(), rec[f][idx[d[:3]]].tolist(), o.rec[f][d[:3]].tolist()))
    for nm, gv, ov in (("li", ti[0::2], o.rec["li"]), ("lj", qj[0::2], o.rec["lj"]), ("ri", ti[1::2], o.rec["ri"]),
                       ("rj", qj[1::2], o.rec["rj"])):
        d = np.nonzero(gv[idx].astype(np.int64) != ov)[0]
        if len(d):
            bad.append((nm, idx[d[:3]].tolist(), gv[idx[d[:3]]].tolist(), ov[d[:3]].tolist()))
    d = np.nonzero((rec["flags"][idx] & 15).astype(np.int64) != (o.rec["flags"] & 15))[0]
    if len(d):
        bad.append(("flags", idx[d[:3]].tolist()))
    cig_bad = [int(s) for k, s in enumerate(idx) if g.cigar_of(s) != o.cigar_of(k)]
    if cig_bad:
        bad.append(("cigar", cig_bad[:3]))
    assert not bad, bad
    hist = np.bincount(bins[idx], minlength=7).tolist()
    print(f"{w.name}: {n} seeds, sample {len(idx)} by bin {hist}; gpu+rescore {t1 - t0:.1f} s, "
          f"oracle {t2 - t1:.1f} s")
    return bins, idx


def test_c1_every_seed():
    w = genome.config1()
    check_config(w, lambda bins: np.arange(len(bins)), min_sample=2048)


@pytest.mark.parametrize("cfg", [2, 3, 5, 6])
def test_long_bins_and_random_sample(cfg):
    w = genome.make(cfg)
    rng = np.random.default_rng(100 + cfg)
    bins, idx = check_config(w, lambda b: stratified(b, rng), min_sample=2000)
    assert set(np.nonzero(bins >= 2)[0].tolist()) <= set(idx.tolist())


def test_c4_stratified_by_bin():
    w = genome.config4()
    rng = np.random.default_rng(104)
    per_bin = {0: 1000, 1: 1500, 2: 2000}
    bins, idx = check_config(w, lambda b: stratified(b, rng, per_bin=per_bin), min_sample=5000)
    assert (bins >= 3).sum() == np.isin(np.nonzero(bins >= 3)[0], idx).sum()
