"""Exact-rational Gauss-Jordan inverse used ONLY to pin the C oracle's GETRI
(test helper; the inversion-based variant, PAPER.md P:206-214 / P:265-278).

``fractions.Fraction`` arithmetic, no rounding.  Two independent things:
  * ``inverse_exact``: the textbook inverse by Gauss-Jordan on [A | I] with
    explicit row swaps and scaled pivot rows -- a different algorithm from the
    oracle's; pins the result mathematically (A * X == I exactly);
  * ``gje_implicit``: the oracle's reading R23-R26 step by step, recording every
    intermediate value, so that when all of them are exactly representable in
    binary64 the floating-point oracle must reproduce it bit for bit.
"""
from __future__ import annotations

from fractions import Fraction


def inverse_exact(A):
    """Textbook Gauss-Jordan with explicit partial pivoting (largest |a|)."""
    m = len(A)
    M = [list(map(Fraction, row)) + [Fraction(int(i == j)) for j in range(m)] for i, row in enumerate(A)]
    for k in range(m):
        p = max(range(k, m), key=lambda i: abs(M[i][k]))
        if M[p][k] == 0:
            return None
        M[k], M[p] = M[p], M[k]
        d = M[k][k]
        M[k] = [v / d for v in M[k]]
        for i in range(m):
            if i != k and M[i][k] != 0:
                f = M[i][k]
                M[i] = [a - f * b for a, b in zip(M[i], M[k])]
    return [row[m:] for row in M]


def gje_implicit(A):
    """R23-R26: in-place GJE on [A | I] with implicit pivoting (first maximal
    |a| among unpivoted rows), unscaled pivot rows, final row division.
    Returns (Dinv rows, perm, info, intermediates)."""
    m = len(A)
    W = [list(map(Fraction, row)) for row in A]
    tag = [0] * m
    perm = [0] * m
    pos = [0] * m
    dp = [Fraction(0)] * m
    info = 0
    inter = []
    for k in range(m):
        p = -1
        for i in range(m):
            if tag[i]:
                continue
            if p < 0 or abs(W[i][k]) > abs(W[p][k]):
                p = i
        tag[p] = k + 1
        perm[k] = p
        pos[p] = k
        d = W[p][k]
        dp[p] = d
        if d == 0:
            if info == 0:
                info = k + 1
            continue
        for i in range(m):
            if i == p:
                continue
            f = W[i][k] / d
            inter.append(f)
            for j in range(m):
                if j != k:
                    W[i][j] = W[i][j] - f * W[p][j]
                    inter.append(W[i][j])
            W[i][k] = -f
        W[p][k] = Fraction(1)
    if info:
        return None, perm, info, inter
    X = [[W[i][j] / dp[i] for j in range(m)] for i in range(m)]
    inter += [v for row in X for v in row]
    Dinv = [[X[perm[a]][pos[b]] for b in range(m)] for a in range(m)]
    return Dinv, perm, info, inter
