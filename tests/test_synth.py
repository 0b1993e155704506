"""Workload generator checks (validates the generator, not the kernels)."""
import numpy as np

from oracle import core
from synth import genome


def test_mut_mapping_is_exact():
    rng = genome.rng_for(77)
    src = genome.random_codes(rng, 5000)
    cp, mapping, clean = genome.mut(rng, src)
    keep = mapping >= 0
    assert np.all(np.diff(mapping[keep]) > 0)
    assert np.array_equal(cp[mapping[clean]], src[clean])
    ks = genome.exact_kmer_starts(mapping, clean)
    for s in ks[:200]:
        q = mapping[s]
        assert np.array_equal(cp[q:q + genome.K], src[s:s + genome.K])
    # rates: ~0.5% deletions, ~0.5% insertions, ~10% substitutions
    assert abs((~keep).mean() - 0.005) < 0.003
    assert abs(len(cp) - len(src)) < 60


def test_seeds_are_exact_12mer_matches():
    w = genome.small_pair(3)
    for tpos, qpos in w.seeds[:100]:
        assert w.T[tpos - 6:tpos + 6] == w.Q[qpos - 6:qpos + 6]


def test_deterministic():
    a, b = genome.small_pair(5), genome.small_pair(5)
    assert a.T == b.T and a.Q == b.Q and np.array_equal(a.seeds, b.seeds)


def test_c2_shape_matches_table2():
    """C2's per-seed bin histogram on a 600-seed sample, measured with the ORACLE, falls in Table 2's
    ranges: eager 75-83%, bin 1 17-25%, bins 2-4 small; > 97% of alignments <= 128 bp."""
    w = genome.config2(n_seeds=1 << 14, scale=0.1)
    idx = np.random.default_rng(0).choice(w.n, 600, replace=False)
    r = core.extend(w.T, w.Q, w.seeds[idx])
    rec = r.rec
    mx = np.maximum(np.maximum(rec["li"], rec["lj"]), np.maximum(rec["ri"], rec["rj"]))
    eager = (mx <= 16).mean()
    bin1 = ((mx > 16) & (mx <= 512)).mean()
    assert 0.72 <= eager <= 0.86, eager
    assert 0.13 <= bin1 <= 0.28, bin1
    length = (rec["t_end"] - rec["t_start"])
    assert (length <= 128).mean() > 0.95
