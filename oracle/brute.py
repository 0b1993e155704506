"""Brute-force references for tiny inputs -- TEST INFRASTRUCTURE ONLY.

Two independent restatements used to pin the C oracle (``oracle/fastz_oracle.c``):

* :func:`full_matrix` evaluates the definitions of SURVEY.md 8(c) / DESIGN.md "Readings" on the WHOLE
  (M+1)x(N+1) matrix in row-major order with ``-inf`` as the dead value: the recurrences of PAPER.md Fig. 1
  (P:70-74), the y-drop cone rule with V(i,j) computed literally as the 2-D prefix maximum
  over live cells, the peak and the traceback over 2+1+1 bit codes.  It has no
  banding, no scan-region logic and no lazy V, which are exactly the parts of the C oracle it checks.
* :func:`best_path_score` enumerates every alignment path that starts at the cut point (one-sided,
  global-start / free-end) and scores it with affine gaps O + k*E.  With y-drop disabled
  its maximum must equal the DP's peak score: this pins the recurrences and the gap convention without
  reference to any DP at all.
"""
from __future__ import annotations

import math

NEG = -math.inf


def full_matrix(A, B, p):
    """Return dict(score, i, j, ops (origin-outward), explored, rows) for codes A (rows), B (cols)."""
    M, N = len(A), len(B)
    O, E, Y = p.gap_open, p.gap_extend, p.ydrop
    S = [[NEG] * (N + 1) for _ in range(M + 1)]
    D = [[NEG] * (N + 1) for _ in range(M + 1)]
    I = [[NEG] * (N + 1) for _ in range(M + 1)]
    V = [[NEG] * (N + 1) for _ in range(M + 1)]
    live = [[False] * (N + 1) for _ in range(M + 1)]
    code = [[0] * (N + 1) for _ in range(M + 1)]
    explored = 0
    best, bi, bj = 0, 0, 0
    for i in range(M + 1):
        for j in range(N + 1):
            pred_live = (i >= 1 and j >= 1 and live[i - 1][j - 1]) or (i >= 1 and live[i - 1][j]) or \
                        (j >= 1 and live[i][j - 1])
            if (i == 0 and j == 0) or pred_live:
                explored += 1
            vu = V[i - 1][j] if i >= 1 else NEG
            vl = V[i][j - 1] if j >= 1 else NEG
            if i == 0 and j == 0:
                s, d, ii, c, lv = 0, NEG, NEG, 0, True
            else:
                h = S[i - 1][j - 1] + p.s(A[i - 1], B[j - 1]) if (i >= 1 and j >= 1) else NEG
                d, dbit = NEG, 0
                if i >= 1:
                    ext, opn = D[i - 1][j] - E, S[i - 1][j] - O - E
                    d, dbit = (ext, 1) if ext > opn else (opn, 0)
                ii, ibit = NEG, 0
                if j >= 1:
                    ext, opn = I[i][j - 1] - E, S[i][j - 1] - O - E
                    ii, ibit = (ext, 1) if ext > opn else (opn, 0)
                src, m = 0, h
                if d > m:
                    src, m = 1, d
                if ii > m:
                    src, m = 2, ii
                lv = m != NEG and m >= max(vu, vl) - Y
                s = m if lv else NEG
                if not lv:
                    d = ii = NEG
                c = src | (dbit << 2) | (ibit << 3)
            S[i][j], D[i][j], I[i][j], live[i][j], code[i][j] = s, d, ii, lv, c
            V[i][j] = max(vu, vl, s if lv else NEG)
            if lv and s > best:
                best, bi, bj = s, i, j
    rows = 0
    for i in range(M + 1):
        if any(live[i]):
            rows = i + 1
    ops = []
    i, j, state = bi, bj, 0
    while i > 0 or j > 0:
        c = code[i][j]
        if state == 0:
            src = c & 3
            if src == 0:
                ops.append("M")
                i, j = i - 1, j - 1
                continue
            state = src
        if state == 1:
            ops.append("D")
            state = 1 if (c >> 2) & 1 else 0
            i -= 1
        else:
            ops.append("I")
            state = 2 if (c >> 3) & 1 else 0
            j -= 1
    return dict(score=int(best), i=bi, j=bj, ops="".join(reversed(ops)), explored=explored, rows=rows)


def path_score(A, B, ops, p):
    """Score of an alignment path (origin-outward ops) with affine gaps O + k*E."""
    i = j = 0
    total = 0
    prev = None
    for op in ops:
        if op == "M":
            total += p.s(A[i], B[j])
            i += 1
            j += 1
        elif op == "D":
            total -= p.gap_extend + (p.gap_open if prev != "D" else 0)
            i += 1
        elif op == "I":
            total -= p.gap_extend + (p.gap_open if prev != "I" else 0)
            j += 1
        else:
            raise ValueError(op)
        prev = op
    return total, i, j


def best_path_score(A, B, p):
    """Max over ALL paths from the origin (ending anywhere) of the affine path score; no pruning."""
    M, N = len(A), len(B)
    best = 0  # the empty path

    def rec(i, j, prev, score):
        nonlocal best
        if score > best:
            best = score
        if i < M and j < N:
            rec(i + 1, j + 1, "M", score + p.s(A[i], B[j]))
        if i < M:
            rec(i + 1, j, "D", score - p.gap_extend - (p.gap_open if prev != "D" else 0))
        if j < N:
            rec(i, j + 1, "I", score - p.gap_extend - (p.gap_open if prev != "I" else 0))

    rec(0, 0, None, 0)
    return best
