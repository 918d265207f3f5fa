"""CPU oracle for supervariable blocking -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this module.  The
product path never imports it and shares no code with it.

Follows PAPER.md section II.A: "Supervariable blocking aims to
identify variables sharing the same column-nonzero-pattern ... Depending on
the pre-defined upper bound for the size of the diagonal blocks, multiple
supervariables adjacent in the coefficient matrix can be clustered within the
same diagonal block".  The paper does not state the clustering rule; the
readings (R20-R22) are:

* R20  a supervariable is a maximal run of CONSECUTIVE rows whose column
       index sequences are identical as stored (same length, same ids in the
       same order); an empty row has the empty pattern.
* R21  clustering is greedy in row order: walk the supervariables, add the
       next one to the open block while the block stays <= bound rows,
       otherwise close the block and open a new one.
* R22  a supervariable longer than the bound is cut into pieces of exactly
       `bound` rows plus a remainder (remainder last); the pieces then enter
       the greedy walk of R21 like supervariables.

Written row by row in plain Python/numpy, in the order above.  Pinned by
``tests/test_oracle_supervariable.py``: the 3-dof FEM closed form
(bound 8/12/16/24/32 -> blocks of 6/12/15/24/30 rows), brute-force
search for the greedy partition on tiny patterns, and the invariants
(every block <= bound, blocks are unions of pieces, no two adjacent blocks
could be merged).
"""
from __future__ import annotations

import numpy as np


def supervariables(row_ptr, col_idx):
    """Start rows of the supervariables (R20), int64[], first entry 0."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    col_idx = np.asarray(col_idx)
    n = row_ptr.shape[0] - 1
    starts = []
    prev = None
    for i in range(n):
        pat = col_idx[row_ptr[i]:row_ptr[i + 1]]
        if prev is None or pat.shape[0] != prev.shape[0] or not np.array_equal(pat, prev):
            starts.append(i)
        prev = pat
    return np.asarray(starts, dtype=np.int64)


def pieces(sv_starts, n: int, bound: int):
    """Row counts of the units of the greedy walk (R22), in row order."""
    out = []
    edges = list(sv_starts) + [n]
    for a, b in zip(edges[:-1], edges[1:]):
        s = int(b - a)
        while s > bound:
            out.append(bound)
            s -= bound
        out.append(s)
    return out


def supervariable_blocking(row_ptr, col_idx, bound: int):
    """block_ptr int32[nb+1] of the greedy clustering (R20-R22)."""
    if not 1 <= bound <= 32:
        raise ValueError("bound must lie in 1..32 (P:115-117, P:395-396)")
    n = int(np.asarray(row_ptr).shape[0] - 1)
    bp = [0]
    cur = 0
    for s in pieces(supervariables(row_ptr, col_idx), n, bound):
        if cur + s > bound:            # R21: close the open block
            bp.append(bp[-1] + cur)
            cur = 0
        cur += s
    if cur > 0:
        bp.append(bp[-1] + cur)
    return np.asarray(bp, dtype=np.int32)
