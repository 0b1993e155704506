"""Packed inspector vs the 32-bit inspector on the same batch: per-side peaks / flags and the records + CIGARs must be
identical (FASTZ_PAIR=0 forces the 32-bit kernel for every side).  Prints timings and the packed/long/redo counts.

usage: python tools/pair_check.py [small|c1|c2|c3|c5|c6 ...]   (GPU)
"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_gundaboluvt21_b200 import fastz  # noqa: E402
from synth import genome  # noqa: E402


def run(w, pair, **env):
    os.environ["FASTZ_PAIR"] = os.environ.get("PAIR_MODE", "2") if pair else "0"
    for k, v in env.items():
        os.environ[k] = str(v)
    with fastz.Aligner(w.T, w.Q) as al:
        al.extend(w.seeds)  # warm
        t0 = time.perf_counter()
        res = al.extend(w.seeds)
        dt = time.perf_counter() - t0
        sides = al.sides()
        st = al.stats()
    for k in env:
        del os.environ[k]
    return res, sides, st, dt


def compare(name, w, **env):
    g0, s0, st0, dt0 = run(w, False, **env)
    g1, s1, st1, dt1 = run(w, True, **env)
    bad = []
    for nm, a, b in zip(("score", "ti", "qj", "flags"), s0, s1):
        d = np.nonzero(a != b)[0]
        if len(d):
            bad.append((nm, len(d), d[:4].tolist(), a[d[:4]].tolist(), b[d[:4]].tolist()))
    for f in g0.rec.dtype.names:
        d = np.nonzero(g0.rec[f] != g1.rec[f])[0]
        if len(d):
            bad.append(("rec." + f, len(d), d[:4].tolist()))
    if bytes(g0.cigar) != bytes(g1.cigar):
        bad.append(("cigar text", 1))
    print(f"{name}: sides {st1['n_sides']} packed {st1['n_packed_sides']} long {st1['n_long_sides']} "
          f"redo {st1['n_redo_sides']} | inspect 32-bit {st0['ms_inspect']:.2f} ms, packed path "
          f"{st1['ms_inspect']:.2f} ms ({st0['ms_inspect'] / max(st1['ms_inspect'], 1e-9):.2f}x) | total "
          f"{st0['ms_total']:.1f} -> {st1['ms_total']:.1f} ms | reserved/written "
          f"{st0['exec_reserved_words'] / max(st0['exec_words'], 1):.3f} -> "
          f"{st1['exec_reserved_words'] / max(st1['exec_words'], 1):.3f} | {'OK' if not bad else 'MISMATCH ' + str(bad)}",
          flush=True)
    return not bad


def main():
    which = sys.argv[1:] or ["small"]
    ok = True
    for wname in which:
        if wname == "small":
            for s in range(4):
                w = genome.small_pair(s, length=30000, n_seeds=512)
                ok &= compare(f"small{s}", w)
            w = genome.small_pair(7, length=30000, n_seeds=512)
            ok &= compare("small7-alllong", w, FASTZ_PAIR_LONG=0)
            ok &= compare("small7-nolong", w, FASTZ_PAIR_LONG=100000)
            ok &= compare("small7-unordered", w, FASTZ_INSPECT_ORDER=0)
        else:
            cid = int(wname[1:])
            t0 = time.perf_counter()
            w = genome.make(cid)
            print(f"{wname}: generated in {time.perf_counter() - t0:.1f} s", flush=True)
            ok &= compare(wname, w)
    print("ALL OK" if ok else "FAILURES")
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main())
