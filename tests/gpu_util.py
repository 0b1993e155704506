"""Shared helpers for the GPU parity tests: run the CUDA path (through the C ABI) and the CPU oracle on the
same seeded inputs and compare element by element.  Everything is integer: the bar is bit-exact."""
import numpy as np

from oracle import core
from paper_conf_sc_gundaboluvt21_b200 import fastz

FIELDS = ["score", "left_score", "right_score", "t_start", "t_end", "q_start", "q_end"]


def oparams(**kw) -> core.Params:
    p = core.Params()
    for k, v in kw.items():
        if k == "sub":
            v = tuple(tuple(int(x) for x in row) for row in np.asarray(v).reshape(4, 4))
        setattr(p, k, v)
    return p


def gparams(**kw):
    kw2 = dict(kw)
    if "sub" in kw2:
        kw2["sub"] = np.asarray(kw2["sub"]).reshape(16)
    return fastz.fastz_default_params(**kw2)


def run_both(T, Q, seeds, census=False, **kw):
    seeds = np.asarray(seeds, dtype=np.int64).reshape(-1, 2)
    with fastz.Aligner(T, Q, gparams(**kw)) as al:
        g = al.extend(seeds)
        sides = al.sides()
        cells = al.census() if census else None
        stats = al.stats()
    o = core.extend(T, Q, seeds, oparams(**kw))
    return g, sides, cells, stats, o


def compare(T, Q, seeds, census=True, **kw):
    g, (sc, ti, qj, fl), cells, stats, o = run_both(T, Q, seeds, census=census, **kw)
    n = len(seeds)
    orec = o.rec
    bad = []
    for f in FIELDS:
        d = np.nonzero(g.rec[f].astype(np.int64) != orec[f])[0]
        if len(d):
            bad.append((f, d[:5].tolist(), g.rec[f][d[:5]].tolist(), orec[f][d[:5]].tolist()))
    # per side peaks
    for nm, gv, ov in (("ti_L", ti[0::2], orec["li"]), ("qj_L", qj[0::2], orec["lj"]),
                       ("ti_R", ti[1::2], orec["ri"]), ("qj_R", qj[1::2], orec["rj"]),
                       ("sc_L", sc[0::2], orec["left_score"]), ("sc_R", sc[1::2], orec["right_score"])):
        d = np.nonzero(gv.astype(np.int64) != ov)[0]
        if len(d):
            bad.append((nm, d[:5].tolist(), gv[d[:5]].tolist(), ov[d[:5]].tolist()))
    # flags: ABOVE_K, eager L/R, overflow -- same bit assignment in both
    d = np.nonzero((g.rec["flags"] & 15).astype(np.int64) != (orec["flags"] & 15))[0]
    if len(d):
        bad.append(("flags", d[:5].tolist(), g.rec["flags"][d[:5]].tolist(), orec["flags"][d[:5]].tolist()))
    cig_bad = [s for s in range(n) if g.cigar_of(s) != o.cigar_of(s)]
    if cig_bad:
        s = cig_bad[0]
        bad.append(("cigar", cig_bad[:5], g.cigar_of(s)[:200], o.cigar_of(s)[:200]))
    if census:
        d = np.nonzero(cells[0::2] != orec["l_explored"])[0]
        if len(d):
            bad.append(("cells_L", d[:5].tolist(), cells[0::2][d[:5]].tolist(), orec["l_explored"][d[:5]].tolist()))
        d = np.nonzero(cells[1::2] != orec["r_explored"])[0]
        if len(d):
            bad.append(("cells_R", d[:5].tolist(), cells[1::2][d[:5]].tolist(), orec["r_explored"][d[:5]].tolist()))
    return bad, g, o, stats
