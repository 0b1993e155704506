"""Binding of ``oracle/rescore.c`` -- TEST INFRASTRUCTURE ONLY.

Whole-batch property check for alignment records in the C-ABI layout (``fastz_alignment``, 64 bytes): every
CIGAR is well formed, walks from (t_start, q_start) through the seed's cut point to (t_end, q_end), and its
left and right parts re-score (sum of sub over M columns, O + k*E per gap run, each side paying its own
opens -- P:70-74) to the record's left_score / right_score.  No DP is run, so it applies at any
size; it shares nothing with the product.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "rescore.c")
_LIB = os.path.join(_HERE, "libfzrescore.so")

# fastz_alignment restated (include/fastz.h), 64 bytes
RECORD_DTYPE = np.dtype([("score", "<i4"), ("left_score", "<i4"), ("right_score", "<i4"), ("flags", "<u4"),
                         ("t_start", "<i8"), ("t_end", "<i8"), ("q_start", "<i8"), ("q_end", "<i8"),
                         ("cigar_off", "<i8"), ("cigar_len", "<i4"), ("reserved", "<i4")])
assert RECORD_DTYPE.itemsize == 64

REASONS = {0: "ok", 1: "endpoints", 2: "score != left + right", 3: "malformed CIGAR", 4: "walks off the sequences",
           5: "misses the cut point", 6: "does not end at (t_end, q_end)", 7: "re-score mismatch",
           8: "CIGAR outside the text"}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
        L.fzr_rescore.restype = i64
        L.fzr_rescore.argtypes = [ctypes.c_char_p, i64, ctypes.c_char_p, i64, vp, i64, vp, vp, i64, vp, i32, i32, i32,
                                  vp, ctypes.POINTER(i64)]
        _lib = L
    return _lib


def rescore(T: bytes, Q: bytes, seeds, rec: np.ndarray, cigar: bytes, sub=None, gap_open: int = 400,
            gap_extend: int = 30, n_score: int = -100):
    """(number of failing records, per-record reason codes).  ``sub`` is 4x4 (target row, query column)."""
    from oracle.core import HOXD70
    T = T.encode() if isinstance(T, str) else bytes(T)
    Q = Q.encode() if isinstance(Q, str) else bytes(Q)
    sd = np.ascontiguousarray(np.asarray(seeds, dtype=np.int64).reshape(-1, 2))
    r = np.ascontiguousarray(rec)
    if r.dtype != RECORD_DTYPE:
        r = r.astype(RECORD_DTYPE) if r.dtype.names else r.view(RECORD_DTYPE)
    sub = np.ascontiguousarray(np.asarray(HOXD70 if sub is None else sub, dtype=np.int32).reshape(16))
    cig = np.frombuffer(bytes(cigar) if not isinstance(cigar, np.ndarray) else cigar.tobytes(), dtype=np.uint8)
    cig = np.ascontiguousarray(cig) if len(cig) else np.zeros(1, np.uint8)
    reason = np.zeros(max(len(r), 1), np.int32)
    first = ctypes.c_int64()
    nbad = lib().fzr_rescore(T, len(T), Q, len(Q), sd.ctypes.data, len(r), r.ctypes.data, cig.ctypes.data,
                             len(cigar), sub.ctypes.data, int(gap_open), int(gap_extend), int(n_score),
                             reason.ctypes.data, ctypes.byref(first))
    return int(nbad), reason[:len(r)]
