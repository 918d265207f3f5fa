"""GPU parity of the inversion-based variant (NEXT(3); PAPER.md P:206-214,
P:265-278; readings R23-R26): bj_getri_vbatched / bj_gemv_vbatched /
bj_setup_inverse against the CPU oracle, bit for bit, through the C ABI."""
import numpy as np
import pytest
import torch

import bj_synth as S
import oracle
from gpu_helpers import NP, bits, device_batch, host_layout
from paper_conf_icpp_anztdfq17_b200 import bj

pytestmark = pytest.mark.gpu


def _getri(sizes, dtype, kind="uniform", values=None):
    npdt = NP[dtype]
    vec, val = host_layout(sizes, dtype)
    A = values if values is not None else S.block_values(sizes, val, dtype=npdt, kind=kind)
    batch = device_batch(sizes, dtype, values_np=A)
    nvec = int(vec[-1])
    piv = torch.full((max(nvec, 1),), -7, dtype=torch.int32, device="cuda")
    info = torch.full((max(len(sizes), 1),), -9, dtype=torch.int32, device="cuda")
    bj.getri(batch, piv, info)
    x = torch.from_numpy(S.rhs_values(np.maximum(sizes, 0), dtype=npdt)).cuda() if nvec else \
        torch.zeros(1, dtype=dtype, device="cuda")
    y = torch.full_like(x, float("nan"))
    bj.gemv(batch, x, y)
    torch.cuda.synchronize()
    D_o, p_o, i_o = oracle.getri_batch(sizes, val, vec, A)
    y_o = oracle.gemv_batch(sizes, val, vec, D_o, x.cpu().numpy()[:nvec])
    info_d = info.cpu().numpy()[: len(sizes)]
    assert np.array_equal(info_d, i_o)
    D_d = batch.values.cpu().numpy()
    piv_d = piv.cpu().numpy()[:nvec]
    y_d = y.cpu().numpy()[:nvec]
    for i, m in enumerate(sizes):
        if m < 1 or m > 32:
            continue
        a, b = int(val[i]), int(val[i]) + m * m
        assert np.array_equal(piv_d[vec[i]: vec[i] + m], p_o[vec[i]: vec[i] + m]), f"pivots block {i}"
        do, dd = D_o[a:b], D_d[a:b]
        fin = np.isfinite(do)
        assert np.array_equal(np.isnan(dd), np.isnan(do)), f"NaN pattern block {i}"
        assert np.array_equal(bits(dd[fin]), bits(do[fin])), f"inverse bits block {i} (m={m})"
        yo, yd = y_o[vec[i]: vec[i] + m], y_d[vec[i]: vec[i] + m]
        fy = np.isfinite(yo)
        assert np.array_equal(bits(yd[fy]), bits(yo[fy])), f"gemv bits block {i}"
    return info_d


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("kind", ["uniform", "int"])
def test_getri_gemv_every_order(dtype, kind):
    sizes = np.repeat(np.arange(1, 33, dtype=np.int32), 29)
    np.random.default_rng(21).shuffle(sizes)
    info = _getri(sizes, dtype, kind)
    if kind == "int":
        assert (info > 0).any()                       # singular blocks exercised (safe path)


def test_getri_edge_sizes_and_specials():
    sizes = np.array([0, 5, 33, 1, -4, 32, 0, 17, 2], dtype=np.int32)
    _getri(sizes, torch.float64)
    m = 8
    rng = np.random.default_rng(22)
    blocks = [np.eye(m), np.eye(m)[rng.permutation(m)], np.diag(rng.uniform(0.5, 2, m)), np.zeros((m, m))]
    z = rng.uniform(-1, 1, (m, m)); z[:, 3] = -0.0; blocks.append(z)
    n = rng.uniform(-1, 1, (m, m)); n[2, 4] = np.inf; blocks.append(n)
    sizes = np.full(len(blocks), m, np.int32)
    vec, val = host_layout(sizes, torch.float64)
    A = np.zeros(int(val[-1]))
    for i, B in enumerate(blocks):
        A[val[i]: val[i] + m * m] = B.reshape(-1, order="F")
    _getri(sizes, torch.float64, values=A)


def test_block_jacobi_inverse_handle_matches_oracle_and_lu_apply():
    """bj_setup_inverse on a FEM row slab; bj_apply (GEMV) equals the oracle's
    extract + getri + gemv bit for bit and agrees with the LU apply to
    rounding."""
    nx, ny, nz = 12, 10, 12
    g = S.FemGrid(nx, ny, nz)
    plane = 3 * nx * ny
    r0, r1 = 2 * plane, 9 * plane
    A = bj.synth_fem(nx, ny, nz, r0, r1)
    bp = S.uniform_block_ptr(r1 - r0, 24)
    bpt = torch.from_numpy(bp).cuda()
    sizes, vec, val = bj.layout_from_block_ptr(bpt, torch.float64)
    inv = bj.Batch(sizes, vec, val, torch.empty(int(val[-1].item()), dtype=torch.float64, device="cuda"))
    piv = torch.empty(r1 - r0, dtype=torch.int32, device="cuda")
    info = torch.empty(len(bp) - 1, dtype=torch.int32, device="cuda")
    h = bj.Handle()
    h.setup_inverse(A, bpt, inv, piv, info)
    x = torch.from_numpy(np.random.default_rng(23).uniform(-1, 1, r1 - r0)).cuda()
    y = torch.empty_like(x)
    h.apply(x, y)
    torch.cuda.synchronize()
    rp, ci, va = g.csr(r0, r1)
    D, sz, vo, vl = oracle.extract(rp, ci, va, bp, col_offset=r0)
    Dinv, po, io = oracle.getri_batch(sz, vl, vo, D)
    yo = oracle.gemv_batch(sz, vl, vo, Dinv, x.cpu().numpy())
    assert np.array_equal(info.cpu().numpy(), io) and np.array_equal(piv.cpu().numpy(), po)
    assert np.array_equal(bits(y.cpu().numpy()), bits(yo))
    LU, pl, il = oracle.getrf_batch(sz, vl, vo, D)
    ylu = oracle.getrs_batch(sz, vl, vo, LU, pl, x.cpu().numpy())
    assert np.abs(yo - ylu).max() <= 1e-12 * np.abs(ylu).max()
