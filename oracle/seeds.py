"""Seeding + ungapped filter oracle -- TEST INFRASTRUCTURE ONLY.

``find_hsps`` binds the plain C reference ``oracle/seed_oracle.c`` (readings S1-S6; PAPER.md P:93
fixes the 19-bp seed span and the seed -> filter -> gapped-extension pipeline; pattern, transitions, X and the
HSP threshold are LASTZ's documented defaults [ext]).  ``brute_hsps`` is an independent all-pairs Python
evaluation of the same definitions for tiny inputs (it checks every (t, q) pair directly against S2 instead
of building an index).  Neither is imported by the product.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "seed_oracle.c")
_LIB = os.path.join(_HERE, "libfzseedoracle.so")

PATTERN_12OF19 = "1110100110010101111"   # LASTZ default spaced seed [ext]
XDROP = 910                              # LASTZ default ungapped x-drop = 10 * sub(A, A) [ext]
HSPTHRESH = 3000                         # LASTZ default HSP threshold [ext]

HSP_DTYPE = np.dtype([("t_start", "<i8"), ("q_start", "<i8"), ("length", "<i4"), ("score", "<i4")])


class _Hsp(ctypes.Structure):
    _fields_ = [("t_start", ctypes.c_int64), ("q_start", ctypes.c_int64), ("length", ctypes.c_int32),
                ("score", ctypes.c_int32)]


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.fzs_find.restype = ctypes.c_int
        _lib.fzs_find.argtypes = [ctypes.c_char_p, ctypes.c_int64, ctypes.c_char_p, ctypes.c_int64, ctypes.c_char_p,
                                  ctypes.c_int, ctypes.POINTER(ctypes.c_int32), ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                  ctypes.c_void_p, ctypes.c_int64, ctypes.POINTER(ctypes.c_int64),
                                  ctypes.POINTER(ctypes.c_int64)]
    return _lib


def _sub16(sub) -> ctypes.Array:
    return (ctypes.c_int32 * 16)(*[int(sub[a][b]) for a in range(4) for b in range(4)])


def find_hsps(T, Q, sub, pattern: str = PATTERN_12OF19, transitions: bool = True, xdrop: int = XDROP,
              hspthresh: int = HSPTHRESH, n_score: int = -100):
    """HSPs (structured array, HSP_DTYPE) in anchor order, and the raw hit count."""
    T = T.encode() if isinstance(T, str) else bytes(T)
    Q = Q.encode() if isinstance(Q, str) else bytes(Q)
    L = lib()
    cap = 1024
    while True:
        out = np.zeros(cap, dtype=HSP_DTYPE)
        n = ctypes.c_int64(0)
        hits = ctypes.c_int64(0)
        rc = L.fzs_find(T, len(T), Q, len(Q), pattern.encode(), int(transitions), _sub16(sub), n_score, xdrop, hspthresh,
                        out.ctypes.data, cap, ctypes.byref(n), ctypes.byref(hits))
        if rc == -6:
            cap = int(n.value)
            continue
        if rc != 0:
            raise ValueError(f"fzs_find failed: {rc}")
        return out[: n.value].copy(), int(hits.value)


_CODE = {"A": 0, "C": 1, "G": 2, "T": 3, "N": 4}
_TRANSITION = {("A", "G"), ("G", "A"), ("C", "T"), ("T", "C")}


def brute_hits(T: str, Q: str, pattern: str = PATTERN_12OF19, transitions: bool = True):
    """All (t, q) pairs satisfying S2, by direct comparison at the care positions (no index)."""
    T, Q = T.upper(), Q.upper()
    care = [i for i, c in enumerate(pattern) if c == "1"]
    L = len(pattern)
    hits = []
    for t in range(len(T) - L + 1):
        for q in range(len(Q) - L + 1):
            if any(T[t + c] == "N" or Q[q + c] == "N" for c in care):  # S7
                continue
            diff = [(T[t + c], Q[q + c]) for c in care if T[t + c] != Q[q + c]]
            if not diff or (transitions and len(diff) == 1 and diff[0] in _TRANSITION):
                hits.append((t, q))
    return hits


def ungapped(T: str, Q: str, t: int, q: int, sub, xdrop: int = XDROP, n_score: int = -100):
    """S3 for one hit: (t_start, q_start, length, score); an N scores n_score (S7)."""
    T, Q = T.upper(), Q.upper()
    def walk(pairs):
        s = best = ext = 0
        for d, (a, b) in enumerate(pairs, 1):
            s += n_score if "N" in (a, b) else sub[_CODE[a]][_CODE[b]]
            if s > best:
                best, ext = s, d
            if s < best - xdrop:
                break
        return best, ext
    br, r = walk(zip(T[t:], Q[q:]))
    bl, l = walk(zip(T[:t][::-1], Q[:q][::-1]))
    return t - l, q - l, l + r, bl + br


def brute_hsps(T: str, Q: str, sub, pattern: str = PATTERN_12OF19, transitions: bool = True, xdrop: int = XDROP,
               hspthresh: int = HSPTHRESH, n_score: int = -100):
    """S2-S6 by brute force: every hit extended, filtered, deduplicated, sorted by anchor."""
    hs = {ungapped(T, Q, t, q, sub, xdrop, n_score) for t, q in brute_hits(T, Q, pattern, transitions)}
    hs = [h for h in hs if h[3] >= hspthresh]
    hs.sort(key=lambda h: (h[0] + h[2] // 2, h[1] + h[2] // 2, h[0], h[2]))
    return hs
