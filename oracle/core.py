"""ctypes binding of the C oracle (``oracle/fastz_oracle.c``) -- TEST INFRASTRUCTURE ONLY.

The oracle's scoring defaults are LASTZ's documented defaults (SURVEY.md c.2 [ext]; the paper states
none): HOXD70, O = 400, E = 30, Y = O + 300E = 9400, K = 3000.  Gap cost convention O + k*E follows
PAPER.md P:71-72 (s_o + s_e on the first gap base).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "fastz_oracle.c")
_LIB = os.path.join(_HERE, "libfzoracle.so")

# HOXD70, rows = target base, columns = query base, order A C G T (LASTZ default scoring [ext]).
HOXD70 = (
    (91, -114, -31, -123),
    (-114, 100, -125, -31),
    (-31, -125, 100, -114),
    (-123, -31, -114, 91),
)


@dataclass
class Params:
    sub: tuple = HOXD70
    gap_open: int = 400
    gap_extend: int = 30
    ydrop: int = 9400
    gapped_threshold: int = 3000
    eager_max: int = 16
    n_score: int = -100   # reading R13: any pair with an N scores n_score (the paper is silent)

    def s(self, a: int, b: int) -> int:
        """Score of target code a against query code b (A0 C1 G2 T3, N4; reading R13)."""
        return self.n_score if a == 4 or b == 4 else self.sub[a][b]

    def transposed(self) -> "Params":
        return Params(tuple(tuple(self.sub[b][a] for b in range(4)) for a in range(4)),
                      self.gap_open, self.gap_extend, self.ydrop, self.gapped_threshold, self.eager_max, self.n_score)


class _CParams(ctypes.Structure):
    _fields_ = [("sub", ctypes.c_int32 * 16), ("gap_open", ctypes.c_int32), ("gap_extend", ctypes.c_int32),
                ("ydrop", ctypes.c_int32), ("gapped_threshold", ctypes.c_int32), ("eager_max", ctypes.c_int32),
                ("n_score", ctypes.c_int32)]


class _CSide(ctypes.Structure):
    _fields_ = [("score", ctypes.c_int64), ("i", ctypes.c_int64), ("j", ctypes.c_int64),
                ("explored", ctypes.c_int64), ("rows", ctypes.c_int64), ("nops", ctypes.c_int64),
                ("overflow", ctypes.c_int32), ("pad", ctypes.c_int32)]


ALIGN_DTYPE = np.dtype([
    ("score", "<i8"), ("left_score", "<i8"), ("right_score", "<i8"),
    ("t_start", "<i8"), ("t_end", "<i8"), ("q_start", "<i8"), ("q_end", "<i8"),
    ("li", "<i8"), ("lj", "<i8"), ("ri", "<i8"), ("rj", "<i8"),
    ("l_explored", "<i8"), ("r_explored", "<i8"),
    ("cigar_off", "<i8"), ("cigar_len", "<i8"), ("flags", "<i4"), ("pad", "<i4"),
])


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain -O2; the oracle is never tuned)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC", "-pthread",
                               "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.fzo_one_sided.restype = ctypes.c_int
        _lib.fzo_one_sided.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64,
                                       ctypes.POINTER(_CParams), ctypes.POINTER(_CSide), ctypes.c_char_p,
                                       ctypes.c_int64]
        _lib.fzo_extend.restype = ctypes.c_int
        _lib.fzo_extend.argtypes = [ctypes.c_char_p, ctypes.c_int64, ctypes.c_char_p, ctypes.c_int64,
                                    ctypes.c_void_p, ctypes.c_int64, ctypes.POINTER(_CParams), ctypes.c_int,
                                    ctypes.c_void_p, ctypes.POINTER(ctypes.c_void_p),
                                    ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]
        _lib.fzo_free.restype = None
        _lib.fzo_free.argtypes = [ctypes.c_void_p]
    return _lib


def _cparams(p: Params) -> _CParams:
    c = _CParams()
    for a in range(4):
        for b in range(4):
            c.sub[4 * a + b] = int(p.sub[a][b])
    c.gap_open, c.gap_extend, c.ydrop = int(p.gap_open), int(p.gap_extend), int(p.ydrop)
    c.gapped_threshold, c.eager_max = int(p.gapped_threshold), int(p.eager_max)
    c.n_score = int(p.n_score)
    return c


_CODE = {"A": 0, "C": 1, "G": 2, "T": 3, "N": 4, "a": 0, "c": 1, "g": 2, "t": 3, "n": 4}


def encode(seq: str) -> np.ndarray:
    return np.array([_CODE[ch] for ch in seq], dtype=np.uint8)


@dataclass
class Side:
    score: int
    i: int
    j: int
    explored: int
    rows: int
    ops: str           # origin-outward
    overflow: bool = False


def one_sided(A: str, B: str, p: Params | None = None) -> Side:
    """One-sided extension of A (rows, target) against B (columns, query) from the origin."""
    p = p or Params()
    a = encode(A) if isinstance(A, str) else np.ascontiguousarray(A, dtype=np.uint8)
    b = encode(B) if isinstance(B, str) else np.ascontiguousarray(B, dtype=np.uint8)
    side = _CSide()
    cap = len(a) + len(b) + 1
    buf = ctypes.create_string_buffer(cap)
    rc = lib().fzo_one_sided(a.ctypes.data, len(a), b.ctypes.data, len(b), ctypes.byref(_cparams(p)),
                             ctypes.byref(side), buf, cap)
    if rc != 0:
        raise RuntimeError(f"fzo_one_sided failed: {rc}")
    return Side(side.score, side.i, side.j, side.explored, side.rows, buf.raw[:side.nops].decode(),
                bool(side.overflow))


@dataclass
class Result:
    rec: np.ndarray                  # ALIGN_DTYPE per seed, seed order
    cigar: bytes = field(repr=False)

    def cigar_of(self, s: int) -> str:
        r = self.rec[s]
        return self.cigar[r["cigar_off"]: r["cigar_off"] + r["cigar_len"]].decode()


def extend(T: str | bytes, Q: str | bytes, seeds, p: Params | None = None, threads: int | None = None) -> Result:
    """Two-sided extension of every seed (tpos, qpos); results in seed order."""
    p = p or Params()
    T = T.encode() if isinstance(T, str) else bytes(T)
    Q = Q.encode() if isinstance(Q, str) else bytes(Q)
    sd = np.ascontiguousarray(np.asarray(seeds, dtype=np.int64).reshape(-1, 2))
    n = sd.shape[0]
    out = np.zeros(max(n, 1), dtype=ALIGN_DTYPE)
    cig = ctypes.c_void_p()
    nbytes = ctypes.c_int64()
    bad = ctypes.c_int64()
    threads = threads or os.cpu_count() or 1
    rc = lib().fzo_extend(T, len(T), Q, len(Q), sd.ctypes.data, n, ctypes.byref(_cparams(p)), int(threads),
                          out.ctypes.data, ctypes.byref(cig), ctypes.byref(nbytes), ctypes.byref(bad))
    if rc != 0:
        raise RuntimeError(f"fzo_extend failed rc={rc} at {bad.value}")
    text = ctypes.string_at(cig, nbytes.value) if nbytes.value else b""
    lib().fzo_free(cig)
    return Result(out[:n], text)
