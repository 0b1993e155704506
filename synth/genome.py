"""Seeded synthetic genome pairs and seed lists shaped like FastZ's workloads.

This module generates INPUTS only; it contains none of the method's arithmetic (no scoring, no DP, no
pruning) and is the one module both the CPU oracle tests and the CUDA path may use ("Input
recipe").  Every array comes from ``numpy.random.Generator(PCG64(20211114 + config_id))``.

Shape targets from PAPER.md: > 97% of alignments <= 128 bp; per-seed length histogram of Table 2
(P:283-296): ~76-82% eager (<= 16 bp), ~18-24% in bin 1 (<= 512), a thin tail in bins 2-4 (up to 32 kbp);
1M seeds per benchmark.  Recipe:

* ``mut``: per source base, deletion p=0.005, one random base inserted before it p=0.005, otherwise a
  substitution p=0.10 (uniform over the other three bases).  The true alignment (source -> copy) is kept.
* "junk" seeds: exact 12-mer chance matches between unrelated positions (12-mers stand in for LASTZ's
  12of19 spaced seeds [ext]), anchored at the 12-mer midpoint (t+6, q+6).
* "homologous" seeds: exact 12-mers on a planted block's true alignment, anchored at the midpoint.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

ASCII = np.frombuffer(b"ACGT", dtype=np.uint8)
K = 12          # seed word length
BASE_SEED = 20211114


def rng_for(config_id: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(BASE_SEED + config_id))


def random_codes(rng, n: int, packed: bool = False) -> np.ndarray:
    """n iid uniform base codes.  packed=True draws raw random bytes and splits each into 4 codes (same
    distribution, a different stream; used by the 1 Gbp config, where it is ~4x faster)."""
    if not packed:
        return rng.integers(0, 4, size=n, dtype=np.uint8)
    b = np.frombuffer(rng.bytes((n + 3) // 4), dtype=np.uint8)
    out = np.empty((len(b), 4), dtype=np.uint8)
    for k in range(4):
        np.bitwise_and(b >> np.uint8(2 * k), np.uint8(3), out=out[:, k])
    return out.reshape(-1)[:n]


# ASCII of 4 consecutive codes packed into one byte (code k in bits 2k+1:2k) as one little-endian uint32
_LUT4 = (ASCII[np.arange(256) & 3].astype(np.uint32) | (ASCII[(np.arange(256) >> 2) & 3].astype(np.uint32) << 8)
         | (ASCII[(np.arange(256) >> 4) & 3].astype(np.uint32) << 16)
         | (ASCII[(np.arange(256) >> 6) & 3].astype(np.uint32) << 24))


def to_ascii(codes: np.ndarray) -> bytes:
    n = len(codes)
    m = n // 4
    q = codes[:4 * m].reshape(m, 4)
    p = q[:, 0] | (q[:, 1] << np.uint8(2)) | (q[:, 2] << np.uint8(4)) | (q[:, 3] << np.uint8(6))
    return _LUT4[p].view(np.uint8).tobytes() + ASCII[codes[4 * m:]].tobytes()


def mut(rng, src: np.ndarray, p_del=0.005, p_ins=0.005, p_sub=0.10, return_starts=False):
    """Mutated copy of ``src`` and the map source index -> copy index (-1 if deleted) and a mask of
    source bases that survive unsubstituted with no insertion in front of them (and, optionally, the copy
    position where each source base's contribution starts)."""
    n = len(src)
    u = rng.random(n)
    dele = u < p_del
    ins = (u >= p_del) & (u < p_del + p_ins)
    subs = (~dele) & (~ins) & (rng.random(n) < p_sub)
    val = np.where(subs, (src + rng.integers(1, 4, n, dtype=np.uint8)) % 4, src).astype(np.uint8)
    counts = np.where(dele, 0, np.where(ins, 2, 1))
    ends = np.cumsum(counts)
    starts = ends - counts
    out = np.empty(int(ends[-1]) if n else 0, dtype=np.uint8)
    out[starts[ins]] = rng.integers(0, 4, int(ins.sum()), dtype=np.uint8)
    keep = ~dele
    pos = starts + ins.astype(np.int64)
    out[pos[keep]] = val[keep]
    mapping = np.where(keep, pos, -1)
    clean = keep & ~subs & ~ins
    if return_starts:
        return out, mapping, clean, starts
    return out, mapping, clean


def exact_kmer_starts(mapping: np.ndarray, clean: np.ndarray, k: int = K) -> np.ndarray:
    """Source offsets s such that source[s:s+k] appears verbatim and contiguously in the copy."""
    n = len(mapping)
    if n < k:
        return np.zeros(0, dtype=np.int64)
    # linked[t]: base t is clean and directly follows base t-1 in the copy (t >= 1)
    linked = np.zeros(n, dtype=bool)
    np.equal(mapping[1:], mapping[:-1] + 1, out=linked[1:])
    linked &= clean
    linked[1:] &= mapping[1:] >= 0
    c = np.zeros(n + 1, dtype=np.int32)
    np.cumsum(linked, dtype=np.int32, out=c[1:])
    # s is a start iff base s is clean and bases s+1 .. s+k-1 are all linked
    full = clean[:n - k + 1] & ((c[k:] - c[1:n - k + 2]) == k - 1)
    return np.flatnonzero(full)


def kmer_codes(codes: np.ndarray, k: int = K) -> np.ndarray:
    """2-bit packed k-mer value at every start position (k <= 16, so uint32 holds it)."""
    n = len(codes) - k + 1
    if n <= 0:
        return np.zeros(0, dtype=np.uint32)
    out = np.zeros(n, dtype=np.uint32)
    for t in range(k):
        out <<= np.uint32(2)
        out |= codes[t:t + n]
    return out


@dataclass
class Workload:
    name: str
    T: bytes
    Q: bytes
    seeds: np.ndarray                     # (n, 2) int64 cut points (tpos, qpos)
    klass: np.ndarray                     # per seed: 0 junk, 1.. planted class index
    class_names: list = field(default_factory=list)
    note: str = ""

    @property
    def n(self):
        return len(self.seeds)


def _layout(rng, total: int, lengths: np.ndarray) -> np.ndarray:
    """Random non-overlapping start positions for blocks of the given lengths inside [0, total)."""
    free = total - int(lengths.sum())
    assert free > 0, "blocks do not fit"
    order = rng.permutation(len(lengths))
    cuts = np.sort(rng.integers(0, free, len(lengths)))
    lo = lengths[order]
    starts = np.empty(len(lengths), dtype=np.int64)
    starts[order] = cuts + np.concatenate([[0], np.cumsum(lo)[:-1]]).astype(np.int64)
    return starts


def _ranges(starts: np.ndarray, lens: np.ndarray) -> np.ndarray:
    """Concatenation of [starts[b], starts[b] + lens[b]) for all b (vectorised)."""
    tot = int(lens.sum())
    base = np.repeat(starts - np.concatenate([[0], np.cumsum(lens)[:-1]]), lens)
    return base + np.arange(tot, dtype=np.int64)


def _loguniform(rng, lo, hi, n):
    return np.exp(rng.uniform(np.log(lo), np.log(hi), n)).astype(np.int64)


def _kmers_at(codes: np.ndarray, pos: np.ndarray) -> np.ndarray:
    """2-bit packed K-mer (first base most significant) starting at each pos: two aligned 8-byte gathers
    per position instead of K scattered byte gathers."""
    pad = np.zeros(((len(codes) + 7) // 8 + 2) * 8, dtype=np.uint8)
    pad[:len(codes)] = codes
    w = pad.view(np.uint64)
    pos = np.asarray(pos, dtype=np.int64)
    q, sh = pos >> 3, (pos & 7).astype(np.uint64) * np.uint64(8)
    w0, w1, w2 = w[q], w[q + 1], w[q + 2]
    # bytes [pos, pos + 16) as lo | hi << 64
    nz = sh != 0
    inv = np.where(nz, np.uint64(64) - sh, np.uint64(0))
    lo = (w0 >> sh) | np.where(nz, w1 << inv, np.uint64(0))
    hi = (w1 >> sh) | np.where(nz, w2 << inv, np.uint64(0))
    out = np.zeros(len(pos), dtype=np.int64)
    for t in range(K):
        byte = (lo >> np.uint64(8 * t)) if t < 8 else (hi >> np.uint64(8 * (t - 8)))
        out = (out << 2) | (byte & np.uint64(3)).astype(np.int64)
    return out


class KmerIndex:
    """Occurrences of every target 12-mer, sorted by (k-mer, position), with bucket starts from a histogram
    over all 4^12 k-mers (a counting index; built once per target)."""

    def __init__(self, Tc: np.ndarray, index_limit: int | None = None):
        tk = kmer_codes(Tc[:index_limit] if index_limit else Tc)
        packed = (tk.astype(np.uint64) << np.uint64(32)) | np.arange(len(tk), dtype=np.uint64)
        packed.sort()
        self.tpos = (packed & np.uint64(0xFFFFFFFF)).astype(np.int64)
        del packed
        self.cnt = np.bincount(tk, minlength=1 << (2 * K)).astype(np.int64)
        self.bstart = np.cumsum(self.cnt) - self.cnt


def _junk_seeds(rng, Tc, Qc, n, homologous_q: np.ndarray | None, index_limit: int | None = None,
                index: KmerIndex | None = None):
    """Chance exact 12-mer matches: random query positions (outside planted homology) looked up in an
    index of target 12-mers; a uniformly random occurrence is taken; anchored at the midpoint."""
    ix = index if index is not None else KmerIndex(Tc, index_limit)
    seeds = []
    need = n
    qmax = len(Qc) - K
    while need > 0:
        qs = rng.integers(0, qmax + 1, size=max(4 * need, 1024))
        if homologous_q is not None:
            qs = qs[~homologous_q[qs] & ~homologous_q[np.minimum(qs + K - 1, len(Qc) - 1)]]
        qk = _kmers_at(Qc, qs)
        c = ix.cnt[qk]
        hit = c > 0
        qs, lo, c = qs[hit], ix.bstart[qk[hit]], c[hit]
        pick = lo + (rng.random(len(lo)) * c).astype(np.int64)
        ts = ix.tpos[pick]
        take = min(need, len(qs))
        seeds.append(np.stack([ts[:take] + K // 2, qs[:take] + K // 2], axis=1))
        need -= take
    return np.concatenate(seeds).astype(np.int64) if seeds else np.zeros((0, 2), np.int64)


def planted_pair(config_id: int, length: int, classes: list, quotas: dict, n_seeds: int,
                 index_limit: int | None = None, name: str = "", mut_kw: dict | None = None,
                 packed_random: bool = False) -> Workload:
    """Random T, Q of ``length`` bp with planted mutated copies T -> Q.

    classes: list of (class_name, lo_len, hi_len, count); quotas: class_name -> fraction of seeds
    ("junk" -> chance matches)."""
    rng = rng_for(config_id)
    Tc = random_codes(rng, length, packed_random)
    Qc = random_codes(rng, length, packed_random)
    lens, cls = [], []
    for ci, (nm, lo, hi, cnt) in enumerate(classes):
        lens.append(_loguniform(rng, lo, hi, cnt))
        cls.append(np.full(cnt, ci + 1))
    lens = np.concatenate(lens)
    cls = np.concatenate(cls)
    tstart = _layout(rng, length, lens + 64)
    qstart = _layout(rng, length, lens + 64)
    # mutate every block in one pass (mut is per-base independent), then split by block
    bsrc = np.concatenate([[0], np.cumsum(lens)[:-1]]).astype(np.int64)  # block start in the concatenation
    src = Tc[_ranges(tstart, lens)]
    copy, mapping, clean, ostart = mut(rng, src, return_starts=True, **(mut_kw or {}))
    ostart = np.append(ostart, len(copy))
    ob = ostart[bsrc]                                   # block's first position in `copy`
    olen = ostart[bsrc + lens] - ob                     # block's copy length
    qpos = _ranges(qstart, olen)
    keep = qpos < length
    Qc[qpos[keep]] = copy[keep]
    hom_q = np.zeros(length, dtype=bool)
    hom_q[qpos[keep]] = True
    # exact 12-mers on each block's true alignment (not crossing block boundaries, inside the sequence)
    ks = exact_kmer_starts(mapping, clean)
    blk = np.searchsorted(bsrc, ks, side="right") - 1
    inside = (ks + K <= bsrc[blk] + lens[blk]) & (mapping[ks] + K <= ob[blk] + olen[blk])
    ks, blk = ks[inside], blk[inside]
    tcoord = tstart[blk] + (ks - bsrc[blk]) + K // 2
    qcoord = qstart[blk] + (mapping[ks] - ob[blk]) + K // 2
    okq = qcoord + K // 2 <= length
    ks, blk, tcoord, qcoord = ks[okq], blk[okq], tcoord[okq], qcoord[okq]
    per_class = {ci + 1: [] for ci in range(len(classes))}
    for ci in range(len(classes)):
        m = cls[blk] == ci + 1
        if m.any():
            per_class[ci + 1].append(np.stack([tcoord[m], qcoord[m]], axis=1))
    seeds, klass = [], []
    counts = {nm: int(round(quotas.get(nm, 0.0) * n_seeds)) for nm in ["junk"] + [c[0] for c in classes]}
    counts["junk"] += n_seeds - sum(counts.values())
    for ci, (nm, *_rest) in enumerate(classes):
        c = counts[nm]
        if c == 0 or not per_class[ci + 1]:
            counts["junk"] += c
            continue
        cand = np.concatenate(per_class[ci + 1])
        pick = rng.integers(0, len(cand), c)
        seeds.append(cand[pick])
        klass.append(np.full(c, ci + 1))
    js = _junk_seeds(rng, Tc, Qc, counts["junk"], hom_q, index_limit)
    seeds.append(js)
    klass.append(np.zeros(len(js), dtype=np.int64))
    seeds = np.concatenate(seeds).astype(np.int64)
    klass = np.concatenate(klass).astype(np.int64)
    perm = rng.permutation(len(seeds))
    return Workload(name or f"cfg{config_id}", to_ascii(Tc), to_ascii(Qc), seeds[perm], klass[perm],
                    ["junk"] + [c[0] for c in classes])


# ----------------------------------------------------------------------------- configurations

C2_CLASSES = [("S1", 24, 128, 20000), ("S2", 128, 512, 1000), ("M", 1000, 8000, 60), ("L", 8000, 32000, 6)]
# Junk (chance 12-mer) seeds come out ~80% eager per seed under the defaults (both sides' peaks within the
# 16x16 window), so ~96% junk reproduces Table 2's ~76-82% eager / ~18-24% bin-1 split.
C2_QUOTAS = {"junk": 0.958, "S1": 0.031, "S2": 0.0098, "M": 0.0012, "L": 0.00004}


def config1(n_seeds: int = 2048) -> Workload:
    """C1: 100 kbp target vs its mutated copy (~10% subs, 1% indels), ~2k seeds: 1/4 chance 12-mer
    matches off the true diagonal, 3/4 exact 12-mers on it (extensions span the whole pair)."""
    rng = rng_for(1)
    Tc = random_codes(rng, 100_000)
    Qc, mapping, clean = mut(rng, Tc)
    ks = exact_kmer_starts(mapping, clean)
    n_true = (3 * n_seeds) // 4
    pick = ks[rng.integers(0, len(ks), n_true)]
    true = np.stack([pick + K // 2, mapping[pick] + K // 2], axis=1)
    # off-diagonal chance matches: junk search, rejecting hits on the true diagonal
    junk = []
    need = n_seeds - n_true
    ix = KmerIndex(Tc)
    while need > 0:
        js = _junk_seeds(rng, Tc, Qc, need * 4, None, index=ix)
        src_of_q = np.full(len(Qc), -1, dtype=np.int64)
        src_of_q[mapping[mapping >= 0]] = np.nonzero(mapping >= 0)[0]
        off = np.abs(src_of_q[js[:, 1] - K // 2] - (js[:, 0] - K // 2)) > 64
        js = js[off][:need]
        junk.append(js)
        need -= len(js)
    seeds = np.concatenate([true, np.concatenate(junk)]).astype(np.int64)
    klass = np.concatenate([np.ones(n_true, np.int64), np.zeros(n_seeds - n_true, np.int64)])
    perm = rng.permutation(n_seeds)
    return Workload("C1-100kbp-pair", to_ascii(Tc), to_ascii(Qc), seeds[perm], klass[perm], ["junk", "diag"])


def config2(n_seeds: int = 1 << 20, scale: float = 1.0) -> Workload:
    """C2: 10 Mbp chromosome pair, 2^20 seeds, skewed lengths (> 97% <= 128 bp; Table 2 shape)."""
    length = int(10_000_000 * scale)
    classes = [(nm, lo, hi, max(1, int(cnt * scale))) for nm, lo, hi, cnt in C2_CLASSES]
    return planted_pair(2, length, classes, C2_QUOTAS, n_seeds, name="C2-10Mbp-pair")


def config3(n_seeds: int = 1 << 21) -> Workload:
    """C3: 100 Mbp pair with long (16-64 kbp) high-scoring alignments."""
    classes = [(nm, lo, hi, cnt * 10) for nm, lo, hi, cnt in C2_CLASSES] + [("XL", 16000, 64000, 40)]
    quotas = {"junk": 0.88, "S1": 0.09, "S2": 0.02, "M": 0.008, "L": 0.0015, "XL": 0.0005}
    return planted_pair(3, 100_000_000, classes, quotas, n_seeds, index_limit=64_000_000, name="C3-100Mbp-pair")


def config4(n_seeds: int = 1 << 23, length: int = 1 << 30) -> Workload:
    """C4: ~1 Gbp whole-genome pair (C2 block mix scaled x100), seeds meant to be sharded over 8 GPUs."""
    f = length / 10_000_000
    classes = [(nm, lo, hi, int(cnt * f)) for nm, lo, hi, cnt in C2_CLASSES]
    return planted_pair(4, length, classes, C2_QUOTAS, n_seeds, index_limit=64_000_000, name="C4-1Gbp-pair",
                        packed_random=True)


def config5(n_seeds: int = 1 << 20, runs_per_octave: int = 1024, spacer: int = 2048) -> Workload:
    """C5: extension-length stress, 12 octaves l_k = 32 * 2^k (32 bp .. 64 kbp); n_k proportional to 1/l_k
    (equal DP work per octave); each run is a mutated copy whose first 12 bp are kept exact."""
    rng = rng_for(5)
    octs = [32 << k for k in range(12)]
    tparts, qparts, runs = [], [], []
    tlen = qlen = 0
    for k, ln in enumerate(octs):
        for _ in range(runs_per_octave):
            src = random_codes(rng, ln)
            cp, _m, _c = mut(rng, src)
            cp = np.concatenate([src[:K], cp[K:]]) if len(cp) >= K else src[:K].copy()
            runs.append((k, tlen, qlen))
            sp_t, sp_q = random_codes(rng, spacer), random_codes(rng, spacer)
            tparts += [src, sp_t]
            qparts += [cp, sp_q]
            tlen += ln + spacer
            qlen += len(cp) + spacer
    Tc = np.concatenate(tparts)
    Qc = np.concatenate(qparts)
    w = np.array([1.0 / ln for ln in octs])
    n_k = np.floor(w / w.sum() * n_seeds).astype(np.int64)
    n_k[0] += n_seeds - n_k.sum()
    runs = np.array(runs, dtype=np.int64)
    seeds, klass = [], []
    for k in range(12):
        rk = runs[runs[:, 0] == k]
        pick = rk[rng.integers(0, len(rk), n_k[k])]
        seeds.append(np.stack([pick[:, 1] + K // 2, pick[:, 2] + K // 2], axis=1))
        klass.append(np.full(n_k[k], k))
    seeds = np.concatenate(seeds)
    klass = np.concatenate(klass)
    perm = rng.permutation(len(seeds))
    return Workload("C5-length-stress", to_ascii(Tc), to_ascii(Qc), seeds[perm], klass[perm],
                    [f"oct{ln}" for ln in octs])


def small_pair(seed: int, length: int = 20_000, n_seeds: int = 256, homology: float = 0.3) -> Workload:
    """Small mixed workload for parity tests: planted blocks of 24 bp .. 2 kbp plus junk seeds."""
    classes = [("S1", 24, 128, max(1, int(60 * length / 20000))), ("S2", 128, 512, max(1, int(8 * length / 20000))),
               ("M", 800, 2000, max(1, int(2 * length / 20000)))]
    quotas = {"junk": 1 - homology, "S1": homology * 0.7, "S2": homology * 0.2, "M": homology * 0.1}
    return planted_pair(1000 + seed, length, classes, quotas, n_seeds, name=f"small{seed}")


def config6(n_seeds: int = 1 << 20) -> Workload:
    """Dissimilar (cross-genus-like) 10 Mbp pair (NEXT-2; PAPER.md 5.4: "no alignment falls in the two
    largest size bins"): planted blocks are diverged copies (25% substitutions, 3% indels) of at most 2 kbp,
    so the seed mix is almost all chance matches and short, low-identity homology."""
    rng_len = 10_000_000
    classes = [("S1", 24, 128, 20000), ("S2", 128, 512, 1000), ("M", 512, 2000, 200)]
    quotas = {"junk": 0.97, "S1": 0.022, "S2": 0.006, "M": 0.002}
    w = planted_pair(6, rng_len, classes, quotas, n_seeds, name="C6-dissimilar-10Mbp", mut_kw=dict(p_sub=0.25, p_del=0.015, p_ins=0.015))
    return w


CONFIGS = {1: config1, 2: config2, 3: config3, 4: config4, 5: config5, 6: config6}


def make(config_id: int, **kw) -> Workload:
    return CONFIGS[config_id](**kw)
