"""Independent textbook routines used to PIN the oracle (tests only).

None of these calls oracle/; each is the standard definition of a quantity
that the Smith-Waterman score reduces to in a special case (DESIGN.md,
"Oracle pins").
"""
from __future__ import annotations

import numpy as np


def lcs_len(a, b) -> int:
    """Longest common subsequence length (textbook DP, Cormen et al. 15.4)."""
    a, b = list(a), list(b)
    prev = [0] * (len(b) + 1)
    for x in a:
        cur = [0]
        for j, y in enumerate(b):
            cur.append(prev[j] + 1 if x == y else max(prev[j + 1], cur[j]))
        prev = cur
    return prev[-1]


def longest_common_substring(a, b) -> int:
    """Length of the longest common contiguous substring, by brute force."""
    a, b = list(a), list(b)
    best = 0
    for i in range(len(a)):
        for j in range(len(b)):
            k = 0
            while i + k < len(a) and j + k < len(b) and a[i + k] == b[j + k]:
                k += 1
            best = max(best, k)
    return best


def kadane(vals) -> int:
    """Maximum sum of a (possibly empty) contiguous subarray."""
    best = cur = 0
    for v in vals:
        cur = max(0, cur + v)
        best = max(best, cur)
    return best


def best_diagonal_kadane(a, b, match: int, mismatch: int) -> int:
    """Max over all diagonals of Kadane on the +match/mismatch scores: the
    local score when gaps are never worth taking."""
    a, b = list(a), list(b)
    m, n = len(a), len(b)
    best = 0
    for off in range(-(m - 1), n):
        vals = []
        for i in range(m):
            j = i + off
            if 0 <= j < n:
                vals.append(match if a[i] == b[j] else mismatch)
        best = max(best, kadane(vals))
    return best


def bits_to_word(s: str) -> int:
    """'0101' printed MSB first -> int."""
    return int(s, 2)


def planes_from_scores(vals, s: int) -> np.ndarray:
    """Bit-slice 32 scores into s words (bit k of word b = bit b of vals[k])."""
    out = np.zeros(s, dtype=np.uint32)
    for k, v in enumerate(vals):
        for b in range(s):
            if (int(v) >> b) & 1:
                out[b] |= np.uint32(1 << k)
    return out
