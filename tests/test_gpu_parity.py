"""GPU parity of GETRF / GETRS (hot-path rows a1, a3, a4) against the CPU
oracle, through the C ABI.  Bar: pivots, info and block boundaries bit-exact;
L\\U and x bit-exact under the pinned operation order (R5: explicit FMA, IEEE
division, ascending k), which implies the north-star tolerances; backward
error <= 1e-13 (fp64) / 1e-5 (fp32) checked independently."""
import numpy as np
import pytest
import torch

import bj_synth as S
import oracle
from gpu_helpers import NP, backward_error, bits, compare_getrf, device_batch, host_layout
from paper_conf_icpp_anztdfq17_b200 import bj

pytestmark = pytest.mark.gpu

TOL = {torch.float64: 1e-13, torch.float32: 1e-5}


def _run(sizes_np, dtype, kind="uniform", values_np=None, plan=True, b_np=None):
    npdt = NP[dtype]
    vec, val = host_layout(sizes_np, dtype)
    A = values_np if values_np is not None else S.block_values(sizes_np, val, dtype=npdt, kind=kind)
    if b_np is not None:
        b = b_np
    else:
        b = S.rhs_values(np.maximum(sizes_np, 0), dtype=npdt) if len(sizes_np) else np.zeros(0, npdt)
    batch = device_batch(sizes_np, dtype, values_np=A)
    # block boundaries (a1) bit-exact
    assert np.array_equal(batch.vec_off.cpu().numpy(), vec)
    assert np.array_equal(batch.val_off.cpu().numpy(), val)
    nvec = int(vec[-1])
    piv = torch.full((max(nvec, 1),), -7, dtype=torch.int32, device="cuda")
    info = torch.full((max(len(sizes_np), 1),), -9, dtype=torch.int32, device="cuda")
    p = bj.Plan(batch.sizes) if plan else None
    bj.getrf(batch, piv, info, plan=p)
    bt = torch.from_numpy(b).to("cuda") if nvec else torch.zeros(1, dtype=dtype, device="cuda")
    x = torch.full_like(bt, float("nan"))
    bj.getrs(batch, piv, bt, x, plan=p)
    torch.cuda.synchronize()
    LU_d = batch.values.cpu().numpy()
    piv_d = piv.cpu().numpy()[:nvec]
    info_d = info.cpu().numpy()[: len(sizes_np)]
    x_d = x.cpu().numpy()[:nvec]
    LU_o, piv_o, info_o = compare_getrf(sizes_np, val, vec, A, LU_d, piv_d, info_d, dtype)
    x_o = oracle.getrs_batch(sizes_np, val, vec, LU_o, piv_o, b)
    return dict(A=A, b=b, vec=vec, val=val, x_d=x_d, x_o=x_o, info=info_d)


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_c1_parity(dtype):
    """Config C1: 1,000 random blocks, m ~ U{4..16}: full oracle comparison."""
    sizes = S.block_sizes(1000, 4, 16)
    r = _run(sizes, dtype)
    assert np.array_equal(bits(r["x_d"]), bits(r["x_o"]))
    assert backward_error(sizes, r["val"], r["vec"], r["A"], r["b"], r["x_d"]) <= TOL[dtype]


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("kind", ["uniform", "int"])
def test_every_order_1_to_32(dtype, kind):
    """Every m in 1..32, several tiles per warp and a ragged tail per order;
    'int' blocks (U{-3..3}) have many exact ties and singular steps."""
    sizes = np.repeat(np.arange(1, 33, dtype=np.int32), 37)
    rng = np.random.default_rng(5)
    rng.shuffle(sizes)
    r = _run(sizes, dtype, kind=kind)
    if kind == "uniform":
        assert np.array_equal(bits(r["x_d"]), bits(r["x_o"]))
        assert backward_error(sizes, r["val"], r["vec"], r["A"], r["b"], r["x_d"]) <= TOL[dtype]
    else:
        assert (r["info"] > 0).any()           # singular blocks were exercised
        ok = r["info"] == 0
        # nonsingular integer blocks: solutions identical where the oracle's is finite
        xd, xo = r["x_d"], r["x_o"]
        fin = np.isfinite(xo)
        assert np.array_equal(bits(xd[fin]), bits(xo[fin]))
        assert ok.sum() > 100


def test_edge_sizes_empty_invalid_and_transient_plan():
    sizes = np.array([0, 5, 33, 1, -4, 32, 0, 17, 2, 40], dtype=np.int32)
    vec, val = host_layout(sizes, torch.float64)
    A = np.random.default_rng(3).uniform(-1, 1, size=int(val[-1]))
    r = _run(sizes, torch.float64, values_np=A, plan=False)
    assert r["info"].tolist()[2] == -1 and r["info"].tolist()[4] == -1 and r["info"].tolist()[9] == -1
    assert r["info"][0] == 0 and r["info"][6] == 0


def test_empty_batch():
    _run(np.zeros(0, np.int32), torch.float64)


def test_special_matrices():
    """identity, permutation, diagonal, zero, -0 column, NaN/Inf injection."""
    rng = np.random.default_rng(9)
    blocks = []
    m = 8
    blocks.append(np.eye(m))
    blocks.append(np.eye(m)[rng.permutation(m)])
    blocks.append(np.diag(rng.uniform(0.5, 2, m)))
    blocks.append(np.zeros((m, m)))
    z = rng.uniform(-1, 1, (m, m)); z[:, 3] = -0.0
    blocks.append(z)
    n = rng.uniform(-1, 1, (m, m)); n[2, 4] = np.nan
    blocks.append(n)
    f = rng.uniform(-1, 1, (m, m)); f[5, 0] = np.inf
    blocks.append(f)
    sizes = np.full(len(blocks), m, np.int32)
    vec, val = host_layout(sizes, torch.float64)
    A = np.zeros(int(val[-1]))
    for i, B in enumerate(blocks):
        A[val[i]: val[i] + m * m] = B.flatten(order="F")
    _run(sizes, torch.float64, values_np=A)


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_extreme_ranges_slow_paths(dtype):
    """Blocks and right-hand sides scaled to the edges of the exponent range,
    mixed with ordinary blocks in the same warps (every size class): GETRF
    defers |a| >= 2^990 / tiny blocks to its exact path, GETRS flags quotients
    that need the IEEE slow path and redoes only those tiles.  Results stay
    bit-identical to the oracle (NaN positions included)."""
    npdt = NP[dtype]
    big, tiny, sub = (1e300, 1e-300, 1e-310) if dtype == torch.float64 else (1e37, 1e-37, 1e-42)
    sizes = np.repeat(np.array([3, 7, 13, 24, 32], np.int32), 37)
    vec, val = host_layout(sizes, dtype)
    A = S.block_values(sizes, val, dtype=npdt)
    b = S.rhs_values(sizes, dtype=npdt).copy()
    for i in range(len(sizes)):
        m = int(sizes[i])
        blk = slice(int(val[i]), int(val[i]) + m * m)
        seg = slice(int(vec[i]), int(vec[i]) + m)
        kind = i % 6
        if kind == 1:
            A[blk] = (A[blk].astype(np.float64) * big).astype(npdt)
        elif kind == 2:
            A[blk] = (A[blk].astype(np.float64) * tiny).astype(npdt)
        elif kind == 3:
            b[seg] = (b[seg].astype(np.float64) * sub).astype(npdt)     # subnormal right-hand sides
        elif kind == 4:
            A[blk] = (A[blk].astype(np.float64) * tiny).astype(npdt)
            b[seg] = (b[seg].astype(np.float64) * big).astype(npdt)      # quotients overflow
    r = _run(sizes, dtype, values_np=A, b_np=b)
    xd, xo = bits(r["x_d"]), bits(r["x_o"])
    nan_d, nan_o = np.isnan(r["x_d"]), np.isnan(r["x_o"])
    assert np.array_equal(nan_d, nan_o)
    assert np.array_equal(xd[~nan_d], xo[~nan_o])


def test_padding_invariance_on_device():
    """a k x k block embedded in 32 x 32 (identity padding) gives the
    same leading factors and pivots on the device as the k x k block."""
    rng = np.random.default_rng(10)
    for k in (3, 13, 17, 31):
        Ak = rng.uniform(-1, 1, (k, k))
        B = np.eye(32); B[:k, :k] = Ak
        sizes = np.array([k, 32], np.int32)
        vec, val = host_layout(sizes, torch.float64)
        A = np.zeros(int(val[-1]))
        A[val[0]: val[0] + k * k] = Ak.flatten(order="F")
        A[val[1]: val[1] + 1024] = B.flatten(order="F")
        batch = device_batch(sizes, torch.float64, values_np=A)
        piv = torch.zeros(int(vec[-1]), dtype=torch.int32, device="cuda")
        info = torch.zeros(2, dtype=torch.int32, device="cuda")
        bj.getrf(batch, piv, info)
        LU = batch.values.cpu().numpy()
        p = piv.cpu().numpy()
        assert np.array_equal(p[:k], p[k: 2 * k])
        lead = LU[val[1]: val[1] + 1024].reshape(32, 32, order="F")[:k, :k]
        assert np.array_equal(bits(lead.copy()), bits(LU[val[0]: val[0] + k * k].reshape(k, k, order="F").copy()))


def test_getrs_in_place_alias():
    sizes = S.block_sizes(500, 1, 32)
    vec, val = host_layout(sizes, torch.float64)
    batch = device_batch(sizes, torch.float64)
    piv = torch.zeros(int(vec[-1]), dtype=torch.int32, device="cuda")
    info = torch.zeros(len(sizes), dtype=torch.int32, device="cuda")
    bj.getrf(batch, piv, info)
    b = torch.from_numpy(S.rhs_values(sizes)).cuda()
    x = torch.empty_like(b)
    bj.getrs(batch, piv, b, x)
    y = b.clone()
    bj.getrs(batch, piv, y, y)
    torch.cuda.synchronize()
    assert torch.equal(x, y)


def test_device_generator_matches_host_generator():
    for dtype in (torch.float64, torch.float32):
        sizes_d = bj.synth_sizes(5000, 1, 32, first=123)
        sizes = S.block_sizes(5000, 1, 32, first=123)
        assert np.array_equal(sizes_d.cpu().numpy(), sizes)
        vec, val = host_layout(sizes, dtype)
        for kind, kname in ((0, "uniform"), (1, "int")):
            batch = device_batch(sizes, dtype, first=123, kind=kind)
            A = S.block_values(sizes, val, first=123, dtype=NP[dtype], kind=kname)
            assert np.array_equal(bits(batch.values.cpu().numpy()[: len(A)]), bits(A))
        rhs = bj.synth_rhs(batch, first=123)
        assert np.array_equal(bits(rhs.cpu().numpy()[: int(vec[-1])]), bits(S.rhs_values(sizes, first=123,
                                                                                          dtype=NP[dtype])))


@pytest.mark.parametrize("nb,pinned", [(3000, True), (300_001, True), (200_000, False)])
def test_gesv_host_end_to_end(nb, pinned):
    """bj_gesv_host (host buffers in/out) equals the oracle -- one chunk, and
    the chunked copy/compute pipeline (nb >= 131,072: 4 and 3 chunks, ragged
    chunk edges; pinned and pageable host buffers)."""
    sizes = S.block_sizes(nb, 4, 32, first=7)
    vec, val = host_layout(sizes, torch.float64)
    A = S.block_values_fast(sizes, val, first=7) if nb > 3000 else S.block_values(sizes, val, first=7)
    b = S.rhs_values(sizes, first=7)
    ws = bj.Workspace()
    pin = (lambda t: t.pin_memory()) if pinned else (lambda t: t)
    sizes_h = pin(torch.from_numpy(sizes))
    A_h = pin(torch.from_numpy(A))
    b_h = pin(torch.from_numpy(b))
    x_h = pin(torch.empty_like(b_h))
    piv_h = pin(torch.empty(int(vec[-1]), dtype=torch.int32))
    info_h = pin(torch.empty(len(sizes), dtype=torch.int32))
    ws.gesv_host(sizes_h, A_h, b_h, x_h, piv_h, info_h)
    LU_o, piv_o, info_o = oracle.getrf_batch(sizes, val, vec, A)
    x_o = oracle.getrs_batch(sizes, val, vec, LU_o, piv_o, b)
    assert np.array_equal(piv_h.numpy(), piv_o) and np.array_equal(info_h.numpy(), info_o)
    assert np.array_equal(bits(x_h.numpy()), bits(x_o))


def _c3_device(nb, dtype, first=0):
    """C3-shaped batch generated on the device (the bench's inputs), factored
    and solved in the bench's launch configuration (plan reused)."""
    sizes_d = bj.synth_sizes(nb, 4, 32, first=first)
    batch = bj.new_batch(sizes_d, dtype)
    bj.synth_blocks(batch, first=first)
    b = bj.synth_rhs(batch, first=first)
    plan = bj.Plan(batch.sizes)
    nvec = int(batch.vec_off[-1].item())
    piv = torch.empty(max(nvec, 1), dtype=torch.int32, device="cuda")
    info = torch.empty(max(nb, 1), dtype=torch.int32, device="cuda")
    x = torch.empty_like(b)
    bj.getrf(batch, piv, info, plan=plan)
    bj.getrs(batch, piv, b, x, plan=plan)
    plan.close()
    return batch, piv[:nvec], info[:nb], x[:nvec]


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_c3_full_size_all_blocks(dtype):
    """Config C3 at full size (1M blocks, m ~ U{4..32}) in the launch
    configuration bench.py times, EVERY block compared with the oracle:
    pivots, info, L\\U bits and x bits.  The oracle's input comes from the host
    generator (bj_synth, C implementation), never from the device."""
    nb = 1_000_000
    batch, piv, info, x = _c3_device(nb, dtype)
    torch.cuda.synchronize()
    sizes = S.block_sizes(nb, 4, 32)
    vec, val = host_layout(sizes, dtype)
    assert np.array_equal(batch.sizes.cpu().numpy(), sizes)
    assert np.array_equal(batch.vec_off.cpu().numpy(), vec) and np.array_equal(batch.val_off.cpu().numpy(), val)
    A = S.block_values_fast(sizes, val, dtype=NP[dtype])
    b = S.rhs_values_fast(sizes, dtype=NP[dtype])
    LU_o, piv_o, info_o = oracle.getrf_batch(sizes, val, vec, A)
    x_o = oracle.getrs_batch(sizes, val, vec, LU_o, piv_o, b)
    assert np.array_equal(info.cpu().numpy(), info_o)
    assert int((info_o != 0).sum()) == 0
    assert np.array_equal(piv.cpu().numpy(), piv_o)
    LU_d = batch.values.cpu().numpy()[: len(LU_o)]
    diff = np.flatnonzero(bits(LU_d) != bits(LU_o))
    assert diff.size == 0, f"{diff.size} L\\U elements differ, first at {diff[:5]}"
    assert np.array_equal(bits(x.cpu().numpy()), bits(x_o))
    # backward error on a sample (the bits are already the oracle's)
    ids = np.arange(0, nb, 997)
    ss = sizes[ids]
    svec, sval = host_layout(ss, dtype)
    A_s = S.block_values_fast(ss, sval, dtype=NP[dtype], ids=ids)
    b_s = S.rhs_values_fast(ss, dtype=NP[dtype], ids=ids)
    x_s = np.concatenate([x_o[vec[i]: vec[i] + sizes[i]] for i in ids])
    assert backward_error(ss, sval, svec, A_s, b_s, x_s) <= TOL[dtype]


@pytest.mark.parametrize("G", [2, 4, 8])
def test_c3_logical_sharding(G):
    """Hot-path row a6 on one device: the C3 batch (1M blocks) split into G
    contiguous cost-balanced shards (bj_partition), each regenerated from the
    counter generator with first= and factored/solved on its own; the
    concatenated pivots, info, L\\U and x are bit-equal to the unsharded run
    (which test_c3_full_size_all_blocks ties to the oracle block by block)."""
    nb = 1_000_000
    dtype = torch.float64
    full, piv, info, x = _c3_device(nb, dtype)
    sizes = S.block_sizes(nb, 4, 32)
    bounds = bj.partition(sizes, G)
    assert np.array_equal(bounds, oracle.partition(sizes, G))
    assert bounds[0] == 0 and bounds[-1] == nb and np.all(np.diff(bounds) > 0)
    cost = np.add.reduceat(sizes.astype(np.int64) ** 2, bounds[:-1])
    assert cost.max() / cost.mean() < 1.001                  # balanced by m^2
    vo = full.val_off.cpu().numpy()
    ve = full.vec_off.cpu().numpy()
    for r in range(G):
        s, e = int(bounds[r]), int(bounds[r + 1])
        sb, sp, si, sx = _c3_device(e - s, dtype, first=s)
        assert torch.equal(sb.sizes, full.sizes[s:e])
        assert torch.equal(si, info[s:e])
        assert torch.equal(sp, piv[ve[s]: ve[e]])
        n = int(vo[e] - vo[s])
        assert torch.equal(sb.values[:n].view(torch.int64), full.values[vo[s]: vo[e]].view(torch.int64))
        assert torch.equal(sx.view(torch.int64), x[ve[s]: ve[e]].view(torch.int64))
        del sb, sp, si, sx
    torch.cuda.synchronize()


def _gesv(sizes_np, dtype, kind="uniform", alias=False, values_np=None, b_np=None):
    """bj_gesv_vbatched (fused factor + solve) against the oracle's GETRF then
    GETRS, and against the library's own separate calls, bit for bit."""
    npdt = NP[dtype]
    vec, val = host_layout(sizes_np, dtype)
    A = values_np if values_np is not None else S.block_values(sizes_np, val, dtype=npdt, kind=kind)
    b = b_np if b_np is not None else S.rhs_values(np.maximum(sizes_np, 0), dtype=npdt)
    batch = device_batch(sizes_np, dtype, values_np=A)
    nvec = int(vec[-1])
    piv = torch.full((max(nvec, 1),), -7, dtype=torch.int32, device="cuda")
    info = torch.full((max(len(sizes_np), 1),), -9, dtype=torch.int32, device="cuda")
    bt = torch.from_numpy(b).to("cuda") if nvec else torch.zeros(1, dtype=dtype, device="cuda")
    x = bt if alias else torch.full_like(bt, float("nan"))
    bj.gesv(batch, piv, info, bt, x)
    torch.cuda.synchronize()
    LU_o, piv_o, info_o = compare_getrf(sizes_np, val, vec, A, batch.values.cpu().numpy(), piv.cpu().numpy()[:nvec],
                                        info.cpu().numpy()[: len(sizes_np)], dtype)
    x_o = oracle.getrs_batch(sizes_np, val, vec, LU_o, piv_o, b)
    xd = x.cpu().numpy()[:nvec]
    m = np.maximum(sizes_np.astype(np.int64), 0)
    valid = np.repeat((sizes_np >= 1) & (sizes_np <= 32), m)          # entries of factored blocks
    assert np.array_equal(np.isnan(xd[valid]), np.isnan(x_o[valid]))
    ok = valid & np.isfinite(x_o)
    assert np.array_equal(bits(xd[ok]), bits(x_o[ok]))
    return A, b, vec, val, xd


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("kind", ["uniform", "int"])
def test_gesv_every_order(dtype, kind):
    """Fused factor + solve on every order 1..32 with ragged tails (and exact
    ties / singular steps for integer blocks)."""
    sizes = np.concatenate([np.full(37, m, np.int32) for m in range(1, 33)] + [np.array([0, 5, 33, 17], np.int32)])
    _gesv(sizes, dtype, kind)


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_gesv_c1_and_alias(dtype):
    sizes = S.block_sizes(1000, 4, 16)
    A, b, vec, val, xd = _gesv(sizes, dtype, alias=True)
    assert backward_error(sizes, val, vec, A, b, xd) <= TOL[dtype]


def test_gesv_c3_full_size_all_blocks():
    """Config C3 (1M blocks) through the fused call: every block equals the
    oracle (and hence the separate getrf + getrs calls)."""
    nb = 1_000_000
    dtype = torch.float64
    sizes_d = bj.synth_sizes(nb, 4, 32)
    batch = bj.new_batch(sizes_d, dtype)
    bj.synth_blocks(batch)
    b = bj.synth_rhs(batch)
    nvec = int(batch.vec_off[-1].item())
    piv = torch.empty(nvec, dtype=torch.int32, device="cuda")
    info = torch.empty(nb, dtype=torch.int32, device="cuda")
    x = torch.empty_like(b)
    plan = bj.Plan(batch.sizes)
    bj.gesv(batch, piv, info, b, x, plan=plan)
    torch.cuda.synchronize()
    sizes = S.block_sizes(nb, 4, 32)
    vec, val = host_layout(sizes, dtype)
    A = S.block_values_fast(sizes, val)
    bh = S.rhs_values_fast(sizes)
    LU_o, piv_o, info_o = oracle.getrf_batch(sizes, val, vec, A)
    x_o = oracle.getrs_batch(sizes, val, vec, LU_o, piv_o, bh)
    assert np.array_equal(info.cpu().numpy(), info_o)
    assert np.array_equal(piv.cpu().numpy(), piv_o)
    assert np.array_equal(bits(batch.values.cpu().numpy()[: len(LU_o)]), bits(LU_o))
    assert np.array_equal(bits(x.cpu().numpy()), bits(x_o))


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_advice_division_and_sign_of_zero_cases(dtype):
    """The round-1 review's cases: a zero candidate divided by a subnormal or
    an infinite pivot (L = 0, not NaN), GETRS with y_k = 0 over a subnormal /
    infinite U(k,k), and an underflowing GER that would flip a -0 in a frozen
    row (R3-R5) -- GETRF, GETRS and the fused GESV bit-identical
    to the oracle, embedded in every tile width."""
    npdt = NP[dtype]
    sub = 1e-310 if dtype == torch.float64 else 1e-40
    tiny = 1e-170 if dtype == torch.float64 else 1e-25
    small = 1e-160 if dtype == torch.float64 else 1e-20
    cases = [np.array([[sub, 1.0], [0.0, 1.0]]), np.array([[np.inf, 1.0], [0.0, 2.0]]),
             np.array([[1.0, 0.0], [0.0, sub]]), np.array([[2.0, 1.0], [0.0, np.inf]]),
             np.array([[1, 0, 0, tiny], [small, 1, 0, 0], [0, 0, 1, -1], [0, 0, 0.5, 1]], dtype=np.float64)]
    blocks = []
    for c in cases:
        for m in (c.shape[0], 7, 16, 24, 32):           # alone and embedded (identity around it)
            B = np.eye(m)
            B[: c.shape[0], : c.shape[0]] = c
            blocks.append(B)
    sizes = np.array([B.shape[0] for B in blocks], np.int32)
    vec, val = host_layout(sizes, dtype)
    A = np.zeros(int(val[-1]), dtype=npdt)
    b = np.zeros(int(vec[-1]), dtype=npdt)
    for i, B in enumerate(blocks):
        m = B.shape[0]
        A[val[i]: val[i] + m * m] = B.astype(npdt).flatten(order="F")
        rhs = np.zeros(m)
        rhs[0] = 1.0                                     # y_1 = 0 over the special U(1,1)
        b[vec[i]: vec[i] + m] = rhs.astype(npdt)
    r = _run(sizes, dtype, values_np=A, b_np=b)
    xd, xo = bits(r["x_d"]), bits(r["x_o"])
    nan_d, nan_o = np.isnan(r["x_d"]), np.isnan(r["x_o"])
    assert np.array_equal(nan_d, nan_o)
    assert np.array_equal(xd[~nan_d], xo[~nan_o])
    _gesv(sizes, dtype, values_np=A, b_np=b)
