"""Pins of the oracle extraction (section III.C) and of layout /
partition (hot-path rows a1, a6) -- CPU only, brute force."""
import numpy as np
import pytest
import torch

import bj_synth as S
import oracle


def _dense_blocks_bruteforce(n, row_ptr, col_idx, values, block_ptr, col_offset=0):
    """Densify with torch.sparse (library routine), slice the diagonal blocks."""
    nnz = len(col_idx)
    rows = np.repeat(np.arange(n), np.diff(row_ptr))
    cols = np.asarray(col_idx, dtype=np.int64) - col_offset
    keep = (cols >= 0) & (cols < n)
    coo = torch.sparse_coo_tensor(np.stack([rows[keep], cols[keep]]),
                                  torch.from_numpy(np.asarray(values)[keep]), (n, n),
                                  check_invariants=True)
    dense = coo.to_dense().numpy()
    out = []
    for b in range(len(block_ptr) - 1):
        bs, be = block_ptr[b], block_ptr[b + 1]
        out.append(dense[bs:be, bs:be])
    assert nnz == len(values)
    return out


def _random_csr(rng, n, density, dtype=np.float64, unsorted=True):
    rp = [0]
    cols, vals = [], []
    for r in range(n):
        k = rng.binomial(n, density)
        c = rng.choice(n, size=k, replace=False)
        if not unsorted:
            c.sort()
        cols.append(c)
        v = rng.uniform(-1, 1, size=k).astype(dtype)
        if k:
            v[rng.random(k) < 0.1] = 0.0        # explicit stored zeros
        vals.append(v)
        rp.append(rp[-1] + k)
    return (np.asarray(rp, np.int64), np.concatenate(cols).astype(np.int32),
            np.concatenate(vals).astype(dtype))


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_extract_matches_bruteforce_densify(dt):
    rng = np.random.default_rng(21)
    for trial in range(6):
        n = int(rng.integers(40, 200))
        rp, ci, va = _random_csr(rng, n, 0.15, dt)
        # random block boundaries 1..32
        edges = [0]
        while edges[-1] < n:
            edges.append(min(n, edges[-1] + int(rng.integers(1, 33))))
        bp = np.asarray(edges, np.int32)
        out, sizes, vec, val = oracle.extract(rp, ci, va, bp)
        ref = _dense_blocks_bruteforce(n, rp, ci, va, bp)
        for b, D in enumerate(ref):
            m = sizes[b]
            got = out[val[b]: val[b] + m * m].reshape(m, m, order="F")
            assert np.array_equal(got, D)


def test_extract_preserves_bits_and_ignores_outside():
    # row 0: -0.0 on the diagonal and a NaN with payload; row 1 empty; row 2 hub
    nan_payload = np.array([0x7FF8DEADBEEF0001], dtype=np.uint64).view(np.float64)[0]
    rp = np.array([0, 3, 3, 6], np.int64)
    ci = np.array([0, 1, 2, 1, 0, 2], np.int32)
    va = np.array([-0.0, nan_payload, 5.0, 1.5, -2.5, 9.0])
    # blocks {0,1} and {2}: (0,2) entry of row 0 lies outside its block
    bp = np.array([0, 2, 3], np.int32)
    out, sizes, vec, val = oracle.extract(rp, ci, va, bp)
    D0 = out[val[0]: val[0] + 4].reshape(2, 2, order="F")
    assert np.signbit(D0[0, 0]) and D0[0, 0] == 0.0
    assert D0[0, 1:].view(np.uint64)[0] == 0x7FF8DEADBEEF0001
    assert D0[1, 0] == 0.0 and not np.signbit(D0[1, 0]) and D0[1, 1] == 0.0
    assert out[val[1]] == 9.0          # row 2's diagonal (stored last, unsorted row)


def test_extract_rejects_duplicates():
    rp = np.array([0, 2], np.int64)
    ci = np.array([0, 0], np.int32)
    va = np.array([1.0, 2.0])
    with pytest.raises(ValueError):
        oracle.extract(rp, ci, va, np.array([0, 1], np.int32))


def test_extract_fem_slab_with_col_offset():
    """Row slab of a FEM grid: local rows, global columns (C5 sharding)."""
    g = S.FemGrid(6, 5, 6)
    rows_per_plane = 3 * 6 * 5
    r0, r1 = 2 * rows_per_plane, 4 * rows_per_plane
    rp, ci, va = g.csr(r0, r1)
    bp = S.uniform_block_ptr(r1 - r0, 6)
    out, sizes, vec, val = oracle.extract(rp, ci, va, bp, col_offset=r0)
    rpf, cif, vaf = g.csr()
    ref = _dense_blocks_bruteforce(g.n, rpf, cif, vaf, bp + r0)
    for b, D in enumerate(ref):
        m = sizes[b]
        assert np.array_equal(out[val[b]: val[b] + m * m].reshape(m, m, order="F"), D)


# ---------------------------------------------------------------- layout
def test_layout_closed_form():
    rng = np.random.default_rng(22)
    for es in (4, 8):
        sizes = rng.integers(0, 33, size=1000).astype(np.int32)
        vec, val = oracle.layout(sizes, es)
        q = 16 // es
        assert vec[0] == 0 and np.array_equal(np.diff(vec), sizes)
        assert val[0] == 0
        d = np.diff(val)
        assert np.all(d >= sizes.astype(np.int64) ** 2) and np.all(d - sizes.astype(np.int64) ** 2 < q)
        assert np.all(val % q == 0)                        # 16-byte aligned block starts


# ---------------------------------------------------------------- partition
def _partition_bruteforce(sizes, G):
    cost = np.asarray(sizes, np.int64) ** 2
    P = np.concatenate([[0], np.cumsum(cost)])
    tot = P[-1]
    out = [0]
    for r in range(1, G):
        cands = [i for i in range(len(sizes) + 1) if G * P[i] >= r * tot]
        out.append(min(cands))
    out.append(len(sizes))
    return out


def test_partition_bruteforce():
    rng = np.random.default_rng(23)
    for _ in range(300):
        nb = int(rng.integers(0, 40))
        G = int(rng.integers(1, 9))
        sizes = rng.integers(0, 33, size=nb).astype(np.int32)
        b = oracle.partition(sizes, G)
        assert b.tolist() == _partition_bruteforce(sizes, G)
        assert np.all(np.diff(b) >= 0)


def test_partition_balance_c3_like():
    sizes = S.block_sizes(100000, 4, 32)
    for G in (2, 4, 8):
        b = oracle.partition(sizes, G)
        cost = sizes.astype(np.int64) ** 2
        shares = [cost[b[r]:b[r + 1]].sum() for r in range(G)]
        assert max(shares) / (cost.sum() / G) < 1.001
