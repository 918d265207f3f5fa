"""GPU parity of diagonal-block extraction (row a2) and of the block-Jacobi
handle (row a5: setup = extract + getrf, apply = getrs) against the oracle."""
import numpy as np
import pytest
import torch

import bj_synth as S
import oracle
from gpu_helpers import NP, bits
from paper_conf_icpp_anztdfq17_b200 import bj

pytestmark = pytest.mark.gpu


def _extract_dev(rp, ci, va, bp, col_offset=0):
    dtype = torch.float64 if va.dtype == np.float64 else torch.float32
    A = bj.Csr(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), torch.from_numpy(va).cuda(), col_offset)
    bpt = torch.from_numpy(bp).cuda()
    sizes, vec, val = bj.layout_from_block_ptr(bpt, dtype)
    total = int(val[-1].item())
    out = bj.Batch(sizes, vec, val, torch.full((max(total, 1),), float("nan"), dtype=dtype, device="cuda"))
    bj.extract(A, bpt, out)
    torch.cuda.synchronize()
    return out


def _check(rp, ci, va, bp, col_offset=0):
    out = _extract_dev(rp, ci, va, bp, col_offset)
    ref, sizes, vec, val = oracle.extract(rp, ci, va, bp, col_offset)
    assert np.array_equal(out.sizes.cpu().numpy(), sizes)
    assert np.array_equal(out.val_off.cpu().numpy(), val)
    got = out.values.cpu().numpy()
    for b in range(len(sizes)):
        m = int(sizes[b])
        q = 16 // va.dtype.itemsize
        a, e = int(val[b]), int(val[b]) + m * m
        assert np.array_equal(bits(got[a:e]), bits(ref[a:e])), f"block {b}"
        pad = got[e: int(val[b]) + (m * m + q - 1) // q * q]
        assert np.all(bits(pad) == 0)                     # pad written as +0.0


def _random_csr(rng, n, density, dtype):
    rp = [0]
    cols, vals = [], []
    for r in range(n):
        k = rng.binomial(n, density)
        c = rng.choice(n, size=k, replace=False)
        v = rng.uniform(-1, 1, size=k).astype(dtype)
        if k:
            v[rng.random(k) < 0.1] = -0.0
        cols.append(c)
        vals.append(v)
        rp.append(rp[-1] + k)
    return np.asarray(rp, np.int64), np.concatenate(cols).astype(np.int32), np.concatenate(vals).astype(dtype)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_random_csr_unsorted(dtype):
    rng = np.random.default_rng(41)
    for _ in range(4):
        n = int(rng.integers(100, 600))
        rp, ci, va = _random_csr(rng, n, 0.08, dtype)
        edges = [0]
        while edges[-1] < n:
            edges.append(min(n, edges[-1] + int(rng.integers(1, 33))))
        _check(rp, ci, va, np.asarray(edges, np.int32))


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_empty_rows_and_long_rows(dtype):
    """Blocks with empty rows (first, last and middle rows of a block: the
    row-by-row fallback) next to blocks whose rows are longer than several
    32-entry chunks (the chunked scan, rows crossing chunk and round edges)."""
    rng = np.random.default_rng(43)
    n = 2000
    rows = []
    for r in range(n):
        u = rng.random()
        if u < 0.15:
            c = np.zeros(0, np.int64)                                 # empty row
        elif u < 0.3:
            c = rng.choice(n, size=int(rng.integers(100, 700)), replace=False)   # long row
        else:
            c = np.unique(np.clip(r + rng.integers(-40, 41, size=30), 0, n - 1))
        rng.shuffle(c)
        rows.append(c)
    rp = np.concatenate([[0], np.cumsum([len(c) for c in rows])]).astype(np.int64)
    ci = np.concatenate(rows).astype(np.int32)
    va = rng.uniform(-1, 1, size=len(ci)).astype(dtype)
    for b in (1, 5, 16, 32):
        _check(rp, ci, va, S.uniform_block_ptr(n, b))
    edges = [0]
    while edges[-1] < n:
        edges.append(min(n, edges[-1] + int(rng.integers(1, 33))))
    _check(rp, ci, va, np.asarray(edges, np.int32))


def test_heavy_rows_take_the_cta_path():
    """Rows with far more than kHeavy entries (skewed nnz)."""
    rng = np.random.default_rng(42)
    n = 50000
    rows = []
    for r in range(n):
        if r in (5, 17, 40000):
            c = rng.choice(n, size=30000, replace=False)    # hub rows
        else:
            c = np.unique(np.clip(r + rng.integers(-20, 21, size=9), 0, n - 1))
        rows.append(c)
    rp = np.concatenate([[0], np.cumsum([len(c) for c in rows])]).astype(np.int64)
    ci = np.concatenate(rows).astype(np.int32)
    va = rng.uniform(-1, 1, size=len(ci))
    _check(rp, ci, va, S.uniform_block_ptr(n, 24))


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_fem_small_grid_device_generator_and_extract(dtype):
    g = S.FemGrid(13, 11, 9)
    A = bj.synth_fem(13, 11, 9, 0, g.n, dtype=dtype)
    rp, ci, va = g.csr(dtype=NP[dtype])
    assert np.array_equal(A.row_ptr.cpu().numpy(), rp)
    assert np.array_equal(A.col_idx.cpu().numpy(), ci)
    assert np.array_equal(bits(A.values.cpu().numpy()), bits(va))
    for b in (8, 16, 24, 32, 7):
        _check(rp, ci, va, S.uniform_block_ptr(g.n, b))


@pytest.mark.parametrize("b", [8, 16, 24, 32])
def test_c4_full_size_all_blocks(b):
    """Config C4 at full size: 174x174x22 grid, 1,998,216 rows, skewed hubs,
    block sizes 8/16/24/32, in the bench's launch configuration; EVERY block
    compared bit for bit with the oracle's extraction of the host-generated
    CSR (bj_synth C generator; the device CSR is also checked against it)."""
    nx, ny, nz = 174, 174, 22
    A = bj.synth_fem(nx, ny, nz, 0, 3 * nx * ny * nz)
    rp, ci, va = S.fem_csr_fast(nx, ny, nz)
    n = len(rp) - 1
    assert np.array_equal(A.row_ptr.cpu().numpy(), rp)
    assert np.array_equal(A.col_idx.cpu().numpy(), ci)
    assert np.array_equal(bits(A.values.cpu().numpy()), bits(va))
    bp = S.uniform_block_ptr(n, b)
    bpt = torch.from_numpy(bp).cuda()
    sizes, vec, val = bj.layout_from_block_ptr(bpt, torch.float64)
    out = bj.Batch(sizes, vec, val, torch.full((int(val[-1].item()),), float("nan"), dtype=torch.float64,
                                               device="cuda"))
    bj.extract(A, bpt, out)
    torch.cuda.synchronize()
    ref, sz, vo, vl = oracle.extract(rp, ci, va, bp)
    assert np.array_equal(sizes.cpu().numpy(), sz) and np.array_equal(val.cpu().numpy(), vl)
    got = out.values.cpu().numpy()
    # compare every block's m*m elements (the alignment padding is not part of the output)
    m = sz.astype(np.int64)
    mask = np.zeros(len(ref), dtype=bool)
    starts = vl[:-1]
    for mm in np.unique(m):
        sel = starts[m == mm]
        idx = (sel[:, None] + np.arange(mm * mm)[None, :]).ravel()
        mask[idx] = True
    diff = np.flatnonzero((bits(got) != bits(ref)) & mask)
    assert diff.size == 0, f"{diff.size} elements differ, first at {diff[:5]}"


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_block_jacobi_handle_setup_apply(dtype):
    """Row a5 on a FEM slab (local rows, global columns)."""
    nx, ny, nz = 12, 10, 12
    g = S.FemGrid(nx, ny, nz)
    plane = 3 * nx * ny
    r0, r1 = 3 * plane, 8 * plane
    A = bj.synth_fem(nx, ny, nz, r0, r1, dtype=dtype)
    bp = S.uniform_block_ptr(r1 - r0, 24)
    bpt = torch.from_numpy(bp).cuda()
    sizes, vec, val = bj.layout_from_block_ptr(bpt, dtype)
    fac = bj.Batch(sizes, vec, val, torch.empty(int(val[-1].item()), dtype=dtype, device="cuda"))
    piv = torch.empty(r1 - r0, dtype=torch.int32, device="cuda")
    info = torch.empty(len(bp) - 1, dtype=torch.int32, device="cuda")
    h = bj.Handle()
    h.setup(A, bpt, fac, piv, info)
    x = torch.from_numpy(np.random.default_rng(44).uniform(-1, 1, r1 - r0).astype(NP[dtype])).cuda()
    y = torch.empty_like(x)
    h.apply(x, y)
    torch.cuda.synchronize()
    rp, ci, va = g.csr(r0, r1, dtype=NP[dtype])
    D, sz, vo, vl = oracle.extract(rp, ci, va, bp, col_offset=r0)
    LU, po, io = oracle.getrf_batch(sz, vl, vo, D)
    yo = oracle.getrs_batch(sz, vl, vo, LU, po, x.cpu().numpy())
    assert np.array_equal(info.cpu().numpy(), io) and np.array_equal(piv.cpu().numpy(), po)
    assert np.array_equal(bits(y.cpu().numpy()), bits(yo))
    # apply twice (stateless) and in place
    y2 = x.clone()
    h.apply(y2, y2)
    torch.cuda.synchronize()
    assert torch.equal(y2, y)


def test_block_jacobi_block_ptr_offset():
    """bj_setup / bj_apply with block_ptr[0] != 0 (a slice of a global block
    list): x and y are indexed relative to block_ptr[0] (include/bj.h)."""
    nx, ny, nz = 10, 9, 8
    g = S.FemGrid(nx, ny, nz)
    n = g.n
    A = bj.synth_fem(nx, ny, nz, 0, n)
    off, b = 30, 12
    bp = np.arange(off, n + 1, b, dtype=np.int32)
    bp = np.unique(np.append(bp, n)).astype(np.int32)
    bpt = torch.from_numpy(bp).cuda()
    sizes, vec, val = bj.layout_from_block_ptr(bpt, torch.float64)
    fac = bj.Batch(sizes, vec, val, torch.empty(int(val[-1].item()), dtype=torch.float64, device="cuda"))
    rows = n - off
    piv = torch.empty(rows, dtype=torch.int32, device="cuda")
    info = torch.empty(len(bp) - 1, dtype=torch.int32, device="cuda")
    h = bj.Handle()
    h.setup(A, bpt, fac, piv, info)
    x = torch.from_numpy(np.random.default_rng(45).uniform(-1, 1, rows)).cuda()
    y = torch.empty_like(x)
    h.apply(x, y)
    torch.cuda.synchronize()
    rp, ci, va = g.csr()
    D, sz, vo, vl = oracle.extract(rp, ci, va, bp)
    LU, po, io = oracle.getrf_batch(sz, vl, vo, D)
    yo = oracle.getrs_batch(sz, vl, vo, LU, po, x.cpu().numpy())
    assert np.array_equal(info.cpu().numpy(), io) and np.array_equal(piv.cpu().numpy(), po)
    assert np.array_equal(bits(y.cpu().numpy()), bits(yo))


def _setup_vs_separate(A, bp, n, dtype):
    """bj_setup (NEXT(1): extraction fused into GETRF for orders 17..32) equals
    bj_extract + bj_getrf_vbatched bit for bit (factors, pivots, info)."""
    bpt = torch.from_numpy(np.ascontiguousarray(bp, dtype=np.int32)).cuda()
    sizes, vec, val = bj.layout_from_block_ptr(bpt, dtype)
    nb = len(bp) - 1
    rows = int(bp[-1] - bp[0])
    fac = bj.Batch(sizes, vec, val, torch.full((int(val[-1].item()),), 7.0, dtype=dtype, device="cuda"))
    piv = torch.full((rows,), -5, dtype=torch.int32, device="cuda")
    info = torch.full((nb,), -9, dtype=torch.int32, device="cuda")
    h = bj.Handle()
    h.setup(A, bpt, fac, piv, info)
    sep = bj.Batch(sizes, vec, val, torch.full_like(fac.values, 7.0))
    bj.extract(A, bpt, sep)
    piv2 = torch.full_like(piv, -5)
    info2 = torch.full_like(info, -9)
    bj.getrf(sep, piv2, info2)
    torch.cuda.synchronize()
    assert torch.equal(info, info2) and torch.equal(piv, piv2)
    v = val.cpu().numpy()
    m = sizes.cpu().numpy().astype(np.int64)
    idx = np.concatenate([np.arange(v[i], v[i] + m[i] * m[i]) for i in range(nb)]) if nb else np.zeros(0, np.int64)
    it = torch.from_numpy(idx).cuda()
    a, b = fac.values[it], sep.values[it]
    iv = torch.int64 if dtype == torch.float64 else torch.int32
    assert torch.equal(a.view(iv), b.view(iv))
    return fac, piv, info


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_fused_setup_mixed_orders_and_hubs(dtype):
    """Block sizes 1..32 (fused for 17..32, separate below), hub rows (blocks
    above kHeavy entries take the extract_heavy + safe path), random values
    with pivoting; also checked against the oracle."""
    rng = np.random.default_rng(31)
    n = 20000
    rows = []
    for r in range(n):
        if r in (40, 9000):
            c = rng.choice(n, size=12000, replace=False)
        else:
            c = np.unique(np.clip(r + rng.integers(-25, 26, size=20), 0, n - 1))
        rows.append(rng.permutation(c))
    rp = np.concatenate([[0], np.cumsum([len(c) for c in rows])]).astype(np.int64)
    ci = np.concatenate(rows).astype(np.int32)
    va = rng.uniform(-1, 1, size=len(ci)).astype(NP[dtype])
    cuts = [0]
    while cuts[-1] < n:
        cuts.append(min(n, cuts[-1] + int(rng.integers(1, 33))))
    bp = np.array(cuts, np.int32)
    A = bj.Csr(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), torch.from_numpy(va).cuda())
    fac, piv, info = _setup_vs_separate(A, bp, n, dtype)
    D, sz, vo, vl = oracle.extract(rp, ci, va, bp)
    LU, po, io = oracle.getrf_batch(sz, vl, vo, D)
    assert np.array_equal(info.cpu().numpy(), io) and np.array_equal(piv.cpu().numpy(), po)
    got = fac.values.cpu().numpy()
    for i in range(len(sz)):
        mm = int(sz[i])
        assert np.array_equal(bits(got[vl[i]: vl[i] + mm * mm]), bits(LU[vl[i]: vl[i] + mm * mm]))


def test_fused_setup_c5_size():
    """C5's per-GPU slab (1,998,216 rows, b = 24) in the bench's launch
    configuration: fused setup == extract + getrf, bit for bit."""
    nx, ny, nz = 174, 174, 22
    n = 3 * nx * ny * nz
    A = bj.synth_fem(nx, ny, nz, 0, n)
    bp = S.uniform_block_ptr(n, 24)
    _setup_vs_separate(A, bp, n, torch.float64)
