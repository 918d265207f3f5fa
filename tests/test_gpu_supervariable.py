"""GPU parity of supervariable blocking (NEXT(2), R20-R22):
bj_supervariable_blocking through the C ABI vs oracle/supervariable.py,
bit-exact (integer work)."""
import numpy as np
import pytest
import torch

import bj_synth as S
from oracle.supervariable import supervariable_blocking as ref_blocking
from paper_conf_icpp_anztdfq17_b200 import bj

pytestmark = pytest.mark.gpu


def _dev(rp, ci, bound):
    A = bj.Csr(torch.from_numpy(np.ascontiguousarray(rp, dtype=np.int64)).cuda(),
               torch.from_numpy(np.ascontiguousarray(ci, dtype=np.int32)).cuda(),
               torch.zeros(max(len(ci), 1), dtype=torch.float64, device="cuda"))
    return bj.supervariable_blocking(A, bound).cpu().numpy()


def _pats_csr(pats):
    rp = np.zeros(len(pats) + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(p) for p in pats])
    ci = np.asarray([c for p in pats for c in p], dtype=np.int32)
    return rp, ci


@pytest.mark.parametrize("skew", [False, True])
@pytest.mark.parametrize("bound", [1, 2, 8, 12, 16, 24, 32])
def test_fem(skew, bound):
    g = S.FemGrid(12, 10, 8, skew=skew)        # 2,880 rows: several 512-row segments + ragged tail
    rp, ci, _ = g.csr()
    assert np.array_equal(_dev(rp, ci, bound), ref_blocking(rp, ci, bound))


def test_random_runs():
    rng = np.random.default_rng(7)
    for trial in range(20):
        n = int(rng.integers(1, 5000))
        pats, i = [], 0
        while i < n:
            run = int(rng.choice([1, 2, 3, 5, 31, 32, 33, 70, 700]))
            k = int(rng.integers(0, 40))
            t = sorted(rng.choice(10000, size=k, replace=False).tolist())
            pats.extend([t] * min(run, n - i))
            i += run
        rp, ci = _pats_csr(pats)
        bound = int(rng.integers(1, 33))
        assert np.array_equal(_dev(rp, ci, bound), ref_blocking(rp, ci, bound)), (trial, bound)


def test_edge_cases():
    rp, ci = _pats_csr([])
    assert _dev(rp, ci, 8).tolist() == [0]
    rp, ci = _pats_csr([[]] * 1000)                      # all rows empty: one long supervariable
    assert np.array_equal(_dev(rp, ci, 24), ref_blocking(rp, ci, 24))
    rp, ci = _pats_csr([[5, 1]] * 1537)                  # one supervariable across 4 segments
    for b in (1, 7, 32):
        assert np.array_equal(_dev(rp, ci, b), ref_blocking(rp, ci, b))
    rp, ci = _pats_csr([[i] for i in range(2049)])       # every row its own supervariable
    assert np.array_equal(_dev(rp, ci, 5), ref_blocking(rp, ci, 5))
    A = bj.Csr(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), torch.zeros(1, dtype=torch.float64,
                                                                                      device="cuda"))
    for bad in (0, 33):
        with pytest.raises(bj.BJError):
            bj.supervariable_blocking(A, bad)


def test_feeds_extraction():
    """The produced block_ptr drives the setup path (extract + getrf) unchanged."""
    g = S.FemGrid(8, 6, 5, skew=False)
    rp, ci, va = g.csr()
    A = bj.Csr(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), torch.from_numpy(va).cuda())
    bp = bj.supervariable_blocking(A, 24)
    sizes = torch.diff(bp).cpu().numpy()
    assert np.all(sizes[:-1] == 24) and 0 < sizes[-1] <= 24


def test_c4_full_size_sampled():
    """C4's full-size pattern (174x174x22 grid, 1,998,216 rows, skewed hubs),
    bound 24, in the bench's launch configuration: 40 windows of 400 rows,
    each starting at a GPU block start that is also a supervariable start
    (checked on rows regenerated on the host), recomputed by the oracle; the
    blocks must agree up to the last 64 rows of the window."""
    nx, ny, nz, bound, W = 174, 174, 22, 24, 400
    g = S.FemGrid(nx, ny, nz)
    A = bj.synth_fem(nx, ny, nz, 0, g.n)
    bp = bj.supervariable_blocking(A, bound).cpu().numpy()
    sizes = np.diff(bp)
    assert bp[0] == 0 and bp[-1] == g.n and sizes.min() >= 1 and sizes.max() <= bound
    rng = np.random.default_rng(11)
    checked = 0
    for j in rng.choice(len(bp) - 1, 400, replace=False):
        s = int(bp[j])
        if s == 0 or s + W > g.n:
            continue
        if np.array_equal(g.row(s - 1)[0], g.row(s)[0]):
            continue                                    # s is a piece cut inside a supervariable
        rows = [g.row(r)[0] for r in range(s, s + W)]
        rp = np.concatenate([[0], np.cumsum([len(c) for c in rows])]).astype(np.int64)
        ref = ref_blocking(rp, np.concatenate(rows), bound).astype(np.int64) + s
        got = bp[(bp >= s) & (bp < s + W - 64)]
        assert np.array_equal(got, ref[ref < s + W - 64]), s
        checked += 1
        if checked == 40:
            break
    assert checked >= 20
