"""Synthetic-input generator checks (host side) -- CPU only."""
import numpy as np

import bj_synth as S


def test_splitmix64_reference_vector():
    # splitmix64 with state 0: the first output is the published constant
    # 0xE220A8397B1DCDAF (Vigna's reference implementation, seed 0).
    z = S.mix64(np.array([0x9E3779B97F4A7C15], dtype=np.uint64))
    assert int(z[0]) == 0xE220A8397B1DCDAF


def test_counter_generator_is_shard_independent():
    full = S.block_sizes(1000, 4, 32)
    part = S.block_sizes(300, 4, 32, first=500)
    assert np.array_equal(full[500:800], part)
    vec, val = S.packed_offsets(full, 8)
    A = S.block_values(full, val)
    vs, vals = S.packed_offsets(full[500:800], 8)
    As = S.block_values(full[500:800], vals, first=500)
    for i in range(300):
        m = int(full[500 + i])
        assert np.array_equal(A[val[500 + i]: val[500 + i] + m * m], As[vals[i]: vals[i] + m * m])


def test_size_distribution_uniform():
    s = S.block_sizes(200000, 4, 32)
    assert s.min() == 4 and s.max() == 32
    h = np.bincount(s)[4:]
    assert np.abs(h / h.mean() - 1).max() < 0.05
    assert abs(s.mean() - 18) < 0.05 and abs((s.astype(float) ** 2).mean() - 394) < 2


def test_values_range_and_grid():
    v = S.uniform_pm1(2, np.arange(100000, dtype=np.uint64))
    assert v.min() >= -1 and v.max() < 1
    assert np.all(v * 2.0 ** 52 == np.round(v * 2.0 ** 52))


def test_fem_grid_counts():
    # grid 174x174x22 -> n = 1,998,216, nnz = 155,750,400
    # (closed form for the stencil part: prod over axes of (3n_a - 2) nodes-pairs x 9)
    nx, ny, nz = 174, 174, 22
    nnz = 9 * (3 * nx - 2) * (3 * ny - 2) * (3 * nz - 2)
    assert 3 * nx * ny * nz == 1998216 and nnz == 155750400
    g = S.FemGrid(7, 6, 5, skew=False)
    rp, ci, va = g.csr()
    assert rp[-1] == 9 * (3 * 7 - 2) * (3 * 6 - 2) * (3 * 5 - 2)


def test_fem_rows_sorted_unique_and_dominant():
    g = S.FemGrid(9, 8, 40)          # big enough for a few hub rows
    hubs = 0
    for r in range(g.n):
        c, v = g.row(r)
        assert len(np.unique(c)) == len(c)
        k = g.n_extra(r)
        hubs += k > 0
        st = c[: len(c) - k]
        assert np.all(np.diff(st) > 0)                       # stencil part sorted
        d = v[: len(st)][st == r][0]
        assert d == 1.0 + np.abs(v[c != r]).sum()            # exact diagonal
        if k:
            ext = c[len(c) - k:].astype(np.int64)
            dist = np.minimum((ext - r) % g.n, (r - ext) % g.n)
            assert np.all(dist > g.band)
    assert hubs >= 1


def test_hub_tail_is_pareto_like():
    g = S.FemGrid(174, 174, 22)
    ks = [g.n_extra(r) for r in range(200000)]
    ks = np.array([k for k in ks if k])
    assert 100 < len(ks) < 320                                # ~0.1% of rows
    assert ks.min() >= 100
    # Pareto(1.5, 100): median 100 * 2^(2/3) = 158.7
    assert 120 < np.median(ks) < 200


def test_fast_generator_matches_numpy():
    """bj_synth/fastgen.c reproduces the numpy generators bit for bit."""
    sizes = S.block_sizes(3000, 1, 32, first=777)
    for dt, es in ((np.float64, 8), (np.float32, 4)):
        vec, val = S.packed_offsets(sizes, es)
        for kind in ("uniform", "int"):
            a = S.block_values(sizes, val, first=777, dtype=dt, kind=kind)
            b = S.block_values_fast(sizes, val, first=777, dtype=dt, kind=kind)
            assert np.array_equal(a.view(np.uint8), b.view(np.uint8))
        ids = np.arange(5000, 8000, dtype=np.int64)[::-1].copy()
        a = S.block_values(sizes, val, dtype=dt, ids=ids)
        b = S.block_values_fast(sizes, val, dtype=dt, ids=ids)
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8))
        a = S.rhs_values(sizes, first=777, dtype=dt)
        b = S.rhs_values_fast(sizes, first=777, dtype=dt)
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8))


def test_fast_fem_matches_numpy():
    g = S.FemGrid(9, 8, 7)            # W > 0: hub rows possible
    n = g.n
    for dt in (np.float64, np.float32):
        for r0, r1 in ((0, n), (100, 700)):
            rp, col, val = g.csr(r0, r1, dtype=dt)
            rp2, col2, val2 = S.fem_csr_fast(9, 8, 7, r0, r1, dtype=dt)
            assert np.array_equal(rp, rp2) and np.array_equal(col, col2)
            assert np.array_equal(val.view(np.uint8), val2.view(np.uint8))
    # a grid big enough to contain hub rows (0.1 % of rows)
    g = S.FemGrid(30, 30, 12)
    hubs = [r for r in range(g.n) if g.n_extra(r) > 0][:3]
    assert hubs, "expected hub rows"
    for r in hubs:
        rp, col, val = g.csr(r, r + 2)
        rp2, col2, val2 = S.fem_csr_fast(30, 30, 12, r, r + 2)
        assert np.array_equal(rp, rp2) and np.array_equal(col, col2)
        assert np.array_equal(val.view(np.uint8), val2.view(np.uint8))
