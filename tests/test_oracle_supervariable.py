"""Pins of the supervariable-blocking oracle (oracle/supervariable.py,
P:186-193, readings R20-R22) against things other than itself:

* closed form: on a 3-dof-per-node FEM pattern every node is one supervariable
  of 3 rows, so bound b gives blocks of 3*floor(b/3) rows (8/12/16/24/32 ->
  6/12/15/24/30) plus one remainder block;
* brute force on tiny patterns: among ALL cuts at unit boundaries whose blocks
  have <= bound rows, the greedy partition has the fewest blocks and, among
  those, the lexicographically largest boundary list (each block as long as
  possible, left to right);
* invariants on skewed (hub-row) FEM patterns.
"""
import itertools

import numpy as np
import pytest

import bj_synth as S
from oracle.supervariable import supervariable_blocking


def _csr_from_patterns(pats):
    rp = np.zeros(len(pats) + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(p) for p in pats])
    ci = np.asarray([c for p in pats for c in p], dtype=np.int32)
    return rp, ci


@pytest.mark.parametrize("bound,blk", [(8, 6), (12, 12), (16, 15), (24, 24), (32, 30), (3, 3), (2, 2), (1, 1)])
def test_fem_3dof_closed_form(bound, blk):
    g = S.FemGrid(5, 4, 3, skew=False)
    rp, ci, _ = g.csr()
    bp = supervariable_blocking(rp, ci, bound)
    n = g.n
    if bound >= 3:
        expect = list(range(0, n, blk)) + [n]
    else:   # supervariables of 3 rows cut into pieces of `bound` + remainder (R22)
        expect = [0]
        for node in range(n // 3):
            for piece in ([1, 1, 1] if bound == 1 else [2, 1]):
                expect.append(expect[-1] + piece)
    assert bp.tolist() == expect


def _unit_boundaries(pats, bound):
    """Independent restatement of R20/R22: a block may start at row i iff
    i == 0, row i's pattern differs from row i-1's, or i lies a multiple of
    `bound` rows after the start of its supervariable."""
    cuts, sv = [], 0
    for i, p in enumerate(pats):
        if i == 0 or tuple(p) != tuple(pats[i - 1]):
            sv = i
        if (i - sv) % bound == 0:
            cuts.append(i)
    return cuts


def _brute(pats, bound):
    n = len(pats)
    cand = _unit_boundaries(pats, bound)[1:]
    best = None
    for r in range(len(cand) + 1):
        for sub in itertools.combinations(cand, r):
            edges = [0, *sub, n]
            if any(b - a > bound for a, b in zip(edges[:-1], edges[1:])):
                continue
            key = (len(edges), [-e for e in edges])
            if best is None or key < best[0]:
                best = (key, edges)
        if best is not None:
            break                      # fewest blocks found
    return best[1]


def test_brute_force_tiny():
    rng = np.random.default_rng(20170814)
    templates = [[0], [0, 1], [1, 2], [], [0, 2], [3]]
    for trial in range(300):
        n = int(rng.integers(0, 11))
        pats, i = [], 0
        while i < n:
            run = int(rng.integers(1, 6))
            t = templates[int(rng.integers(0, len(templates)))]
            pats.extend([t] * min(run, n - i))
            i += run
        bound = int(rng.integers(1, 7))
        rp, ci = _csr_from_patterns(pats)
        got = supervariable_blocking(rp, ci, bound).tolist()
        assert got == (_brute(pats, bound) if n else [0]), (pats, bound)


def test_order_sensitive_pattern():
    # R20: identical column SETS stored in a different order are different patterns
    rp, ci = _csr_from_patterns([[0, 1], [1, 0], [1, 0]])
    assert supervariable_blocking(rp, ci, 32).tolist() == [0, 3]
    assert supervariable_blocking(rp, ci, 2).tolist() == [0, 1, 3]


@pytest.mark.parametrize("bound", [8, 24, 32])
def test_invariants_skewed_fem(bound):
    g = S.FemGrid(6, 5, 4, skew=True)
    rp, ci, _ = g.csr()
    bp = supervariable_blocking(rp, ci, bound)
    sizes = np.diff(bp)
    assert bp[0] == 0 and bp[-1] == g.n and np.all(sizes >= 1) and np.all(sizes <= bound)
    pats = [tuple(ci[rp[i]:rp[i + 1]]) for i in range(g.n)]
    cuts = set(_unit_boundaries(pats, bound))
    assert set(bp[:-1].tolist()) <= cuts
    # greedy maximality: the next unit never fits into the previous block
    cl = sorted(cuts) + [g.n]
    for a, b in zip(bp[:-1], bp[1:]):
        if b < g.n:
            nxt = cl[cl.index(int(b)) + 1]
            assert nxt - a > bound
