"""Brute-force Smith-Waterman scores for tiny inputs (test pins for oracle/sw_oracle.c).

TEST INFRASTRUCTURE ONLY. No recurrence: every path of Eq. 5's moves (PAPER.md L16@3413)
is enumerated explicitly. A path starts at any cell (i0, j0) with value 0 and is a
sequence of moves -- diagonal (+s(a_i, b_j)), down by k >= 1 (+W_k), right by l >= 1
(+W_l) -- that stays inside the (M+1) x (N+1) matrix; H(i, j) is the maximum of 0 and the
scores of all paths ending at (i, j). Exponential: M, N <= 4.
"""
from __future__ import annotations

import numpy as np


def sw_brute_H(a: bytes, b: bytes, params) -> np.ndarray:
    match, mismatch, gopen, gext = params
    M, N = len(a), len(b)
    W = lambda k: gopen + (k - 1) * gext  # noqa: E731
    best = np.zeros((M + 1, N + 1), dtype=np.int64)  # the 0 term

    def walk(i, j, s):
        if s > best[i, j]:
            best[i, j] = s
        if i < M and j < N:
            walk(i + 1, j + 1, s + (match if a[i] == b[j] else mismatch))
        for k in range(1, M - i + 1):
            walk(i + k, j, s + W(k))
        for l in range(1, N - j + 1):
            walk(i, j + l, s + W(l))

    for i0 in range(M + 1):
        for j0 in range(N + 1):
            walk(i0, j0, 0)
    # row 0 and column 0 are the boundary (0), not reachable cells of Eq. 5
    best[0, :] = 0
    best[:, 0] = 0
    return best
