"""NEXT(4) parity: the block-Jacobi preconditioned BiCGSTAB of section IV.D
 and its building blocks -- SpMV (R27), dot (R28), the solve
(R29) and the communication path (R30) -- CUDA path through the C ABI vs the
CPU oracle on identical seeded inputs, bit for bit."""
import numpy as np
import pytest
import scipy.sparse as sp
import torch

import bj_synth as S
import oracle
from gpu_helpers import bits
from paper_conf_icpp_anztdfq17_b200 import bj

pytestmark = pytest.mark.gpu
DEV = "cuda"


def _t(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def _csr_dev(rp, ci, va, col_offset=0):
    return bj.Csr(_t(rp.astype(np.int64)), _t(ci.astype(np.int32)), _t(va.astype(np.float64)), col_offset)


def _random_csr(n, ncols, rng, long_rows=(), base=0):
    """Random CSR with unsorted rows, empty rows and a few long rows."""
    rows = []
    for i in range(n):
        k = int(rng.integers(0, 40)) if i % 7 else 0
        if i in long_rows:
            k = long_rows[i]
        cols = rng.choice(ncols, size=min(k, ncols), replace=False) + base
        rows.append(cols.astype(np.int32))
    rp = np.zeros(n + 1, np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    ci = np.concatenate(rows) if rp[-1] else np.zeros(0, np.int32)
    va = rng.uniform(-1, 1, int(rp[-1])) * np.exp2(rng.integers(-30, 30, int(rp[-1])))
    return rp, ci.astype(np.int32), va


@pytest.mark.parametrize("seed", [1, 2])
def test_spmv_random_unsorted_long_rows(seed):
    rng = np.random.default_rng(100 + seed)
    n, ncols = 3000, 20000
    long_rows = {5: 2049, 17: 5000, 400: 12345, 2999: 20000, 1000: 2048, 1001: 129}
    rp, ci, va = _random_csr(n, ncols, rng, long_rows)
    x = rng.uniform(-1, 1, ncols)
    y_o = oracle.spmv(rp, ci, va, x)
    y = torch.empty(n, dtype=torch.float64, device=DEV)
    bj.spmv(_csr_dev(rp, ci, va), _t(x), y)
    assert np.array_equal(bits(y.cpu().numpy()), bits(y_o))
    # the same rows with column ids shifted by col_offset
    off = 777
    y2 = torch.empty(n, dtype=torch.float64, device=DEV)
    bj.spmv(_csr_dev(rp, ci + off, va, col_offset=off), _t(x), y2)
    assert np.array_equal(bits(y2.cpu().numpy()), bits(y_o))


def test_spmv_edge_cases():
    # empty matrix, one row, rows of exactly 32 / 128 / 2048 / 2049 entries
    y = torch.empty(0, dtype=torch.float64, device=DEV)
    bj.spmv(_csr_dev(np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0)), _t(np.ones(1)), y)
    rng = np.random.default_rng(7)
    for k in (1, 31, 32, 33, 127, 128, 129, 2047, 2048, 2049, 4096, 4097, 8193):
        rp = np.array([0, k], np.int64)
        ci = rng.permutation(9000)[:k].astype(np.int32)
        va = rng.uniform(-1, 1, k)
        x = rng.uniform(-1, 1, 9000)
        y = torch.empty(1, dtype=torch.float64, device=DEV)
        bj.spmv(_csr_dev(rp, ci, va), _t(x), y)
        assert bits(y.cpu().numpy())[0] == bits(oracle.spmv(rp, ci, va, x))[0], k
    # order pin of R27 (the butterfly adds lanes 0 and 16 ... not left to right)
    rp = np.array([0, 3], np.int64)
    ci = np.array([0, 1, 2], np.int32)
    va = np.array([2.0 ** -53, 2.0 ** -53, 1.0])
    y = torch.empty(1, dtype=torch.float64, device=DEV)
    bj.spmv(_csr_dev(rp, ci, va), _t(np.ones(3)), y)
    assert y.item() == 1.0


@pytest.mark.parametrize("n", [0, 1, 255, 8192, 8193, 100003, 2_000_001])
def test_dot(n):
    rng = np.random.default_rng(n + 3)
    x = rng.uniform(-1, 1, n) * np.exp2(rng.integers(-20, 20, n))
    y = rng.uniform(-1, 1, n)
    d = bj.dot(_t(x), _t(y)).item()
    assert np.float64(d).view(np.uint64) == np.float64(oracle.dot(x, y)).view(np.uint64)


def test_dot_order_pin():
    x = np.zeros(300)
    x[0] = x[256] = 2.0 ** -53
    x[1] = 1.0
    assert bj.dot(_t(x), _t(np.ones(300))).item() == 1.0 + 2.0 ** -52


def _solve_both(rp, ci, va, bp, b, tol=1e-6, maxit=10000, inverse=False, comm=None):
    n = len(rp) - 1
    A = _csr_dev(rp, ci, va)
    bpt = _t(bp.astype(np.int32))
    sizes, vec, val = bj.layout_from_block_ptr(bpt, torch.float64)
    fac = bj.Batch(sizes, vec, val, torch.empty(max(int(val[-1].item()), 2), dtype=torch.float64, device=DEV))
    piv = torch.empty(max(n, 1), dtype=torch.int32, device=DEV)
    info = torch.empty(len(bp) - 1, dtype=torch.int32, device=DEV)
    h = bj.Handle()
    (h.setup_inverse if inverse else h.setup)(A, bpt, fac, piv, info)
    x = torch.full((max(n, 1),), float("nan"), dtype=torch.float64, device=DEV)
    it, res = bj.bicgstab(h, A, _t(b), x, tol=tol, maxit=maxit, comm=comm)
    return x[:n].cpu().numpy(), it, res


@pytest.mark.parametrize("grid,blk", [((10, 9, 8), 24), ((10, 9, 8), 8), ((7, 6, 5), 1), ((12, 11, 10), 32)])
def test_bicgstab_fem_matches_oracle(grid, blk):
    g = S.FemGrid(*grid)
    rp, ci, va = g.csr()
    bp = S.uniform_block_ptr(g.n, blk)
    b = np.ones(g.n)
    x_o, it_o, res_o, *_ = oracle.bicgstab(rp, ci, va, bp, b)
    x, it, res = _solve_both(rp, ci, va, bp, b)
    assert it == it_o and 1 < it < 200
    assert np.float64(res).view(np.uint64) == np.float64(res_o).view(np.uint64)
    assert np.array_equal(bits(x), bits(x_o))
    A = sp.csr_matrix((va, ci, rp), shape=(g.n, g.n))
    assert np.linalg.norm(b - A @ x) / np.linalg.norm(b) <= 2e-6


def test_bicgstab_not_converged_and_maxit():
    g = S.FemGrid(8, 7, 6)
    rp, ci, va = g.csr()
    bp = S.uniform_block_ptr(g.n, 24)
    b = np.ones(g.n)
    for maxit in (1, 2, 3, 5):
        x_o, it_o, res_o, *_ = oracle.bicgstab(rp, ci, va, bp, b, tol=1e-30, maxit=maxit)
        x, it, res = _solve_both(rp, ci, va, bp, b, tol=1e-30, maxit=maxit)
        assert it == it_o == maxit + 1
        assert res == res_o and np.array_equal(bits(x), bits(x_o))


def test_bicgstab_exact_preconditioner_one_step():
    rng = np.random.default_rng(53)
    Ad = rng.uniform(-1, 1, (24, 24)) + 24 * np.eye(24)
    M = sp.csr_matrix(Ad)
    rp, ci, va = M.indptr.astype(np.int64), M.indices.astype(np.int32), M.data
    bp = np.array([0, 24], np.int32)
    b = np.ones(24)
    x_o, it_o, res_o, *_ = oracle.bicgstab(rp, ci, va, bp, b)
    x, it, res = _solve_both(rp, ci, va, bp, b)
    assert it == it_o == 1 and np.array_equal(bits(x), bits(x_o)) and res == res_o


def test_bicgstab_loopback_comm_path_equal():
    """The library's communication path (pack / callbacks / rank-ordered sum)
    with one rank gives the same bits as the direct path (R30, G = 1)."""
    g = S.FemGrid(10, 9, 8)
    rp, ci, va = g.csr()
    bp = S.uniform_block_ptr(g.n, 24)
    b = np.ones(g.n)
    x0, it0, res0 = _solve_both(rp, ci, va, bp, b)
    comm = bj.LoopbackComm()
    x1, it1, res1 = _solve_both(rp, ci, va, bp, b, comm=comm)
    assert it1 == it0 and res1 == res0 and np.array_equal(bits(x1), bits(x0))
    assert comm.calls["halo"] >= 2 * it0 and comm.calls["allgather"] >= 3 * it0 + 1
    assert comm.calls["wait"] == comm.calls["halo"]


def test_bicgstab_inverse_handle_converges():
    """M^-1 by the NEXT(3) inverse handle (GEMV apply): not the oracle's
    preconditioner bit for bit, but the same solve to the tolerance."""
    g = S.FemGrid(10, 9, 8)
    rp, ci, va = g.csr()
    bp = S.uniform_block_ptr(g.n, 24)
    b = np.ones(g.n)
    x_o, it_o, *_ = oracle.bicgstab(rp, ci, va, bp, b)
    x, it, res = _solve_both(rp, ci, va, bp, b, inverse=True)
    assert res <= 1e-6 and abs(it - it_o) <= 2
    assert np.linalg.norm(x - x_o) / np.linalg.norm(x_o) <= 1e-5


def test_bicgstab_c5k_full_size():
    """The bench's C5K workload at N = 1 (174 x 174 x 22 grid, 1,998,216 rows,
    hub rows, b = 24), device-generated matrix vs the host generator's copy
    for the oracle: iterations, residual and every x bit."""
    nx, ny, nz = 174, 174, 22
    n = 3 * nx * ny * nz
    A = bj.synth_fem(nx, ny, nz, 0, n)
    A.col_offset = 0
    rp, ci, va = S.fem_csr_fast(nx, ny, nz)
    assert np.array_equal(A.row_ptr.cpu().numpy(), rp)
    bp = S.uniform_block_ptr(n, 24)
    b = np.ones(n)
    x_o, it_o, res_o, *_ = oracle.bicgstab(rp, ci, va, bp, b)
    bpt = _t(bp)
    sizes, vec, val = bj.layout_from_block_ptr(bpt, torch.float64)
    fac = bj.Batch(sizes, vec, val, torch.empty(int(val[-1].item()), dtype=torch.float64, device=DEV))
    piv = torch.empty(n, dtype=torch.int32, device=DEV)
    info = torch.empty(len(bp) - 1, dtype=torch.int32, device=DEV)
    h = bj.Handle()
    h.setup(A, bpt, fac, piv, info)
    x = torch.empty(n, dtype=torch.float64, device=DEV)
    it, res = bj.bicgstab(h, A, torch.ones(n, dtype=torch.float64, device=DEV), x)
    assert it == it_o and res == res_o
    assert np.array_equal(bits(x.cpu().numpy()), bits(x_o))


def test_bicgstab_torchcomm_nccl_one_rank():
    """The multi-rank path with the real bj.TorchComm over NCCL (world size 1,
    spawned in a fresh process): halo plan, callbacks issued from inside
    bj_bicgstab, all_gather of the rank values -- bit-equal to the direct
    single-GPU solve (R30 with one rank is R28)."""
    import subprocess
    import sys
    import textwrap
    code = textwrap.dedent("""
        import os, socket, numpy as np, torch, torch.distributed as dist
        import bj_synth as S
        from paper_conf_icpp_anztdfq17_b200 import bj
        s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        torch.cuda.set_device(0)
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
        g = S.FemGrid(10, 9, 8)
        rp, ci, va = g.csr()
        n = g.n
        cl, hc, rc = bj.halo_plan(ci, 0, n, np.array([0, n], np.int64))
        assert len(hc) == 0 and np.array_equal(cl, ci)
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
        A = bj.Csr(t(rp), t(ci), t(va), 0)
        bp = t(S.uniform_block_ptr(n, 24))
        sizes, vec, val = bj.layout_from_block_ptr(bp, torch.float64)
        fac = bj.Batch(sizes, vec, val, torch.empty(int(val[-1].item()), dtype=torch.float64, device="cuda"))
        piv = torch.empty(n, dtype=torch.int32, device="cuda")
        info = torch.empty(bp.numel() - 1, dtype=torch.int32, device="cuda")
        h = bj.Handle(); h.setup(A, bp, fac, piv, info)
        b = torch.ones(n, dtype=torch.float64, device="cuda")
        x0 = torch.empty(n, dtype=torch.float64, device="cuda")
        it0, r0 = bj.bicgstab(h, A, b, x0)
        comm = bj.TorchComm(hc, rc, 0, "cuda")
        x1 = torch.empty(n, dtype=torch.float64, device="cuda")
        it1, r1 = bj.bicgstab(h, A, b, x1, comm=comm)
        assert it1 == it0 and r1 == r0, (it0, it1, r0, r1)
        assert torch.equal(x0.view(torch.int64), x1.view(torch.int64))
        dist.destroy_process_group()
        print("torchcomm ok", it0)
    """)
    root = __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__)))
    env = dict(__import__("os").environ, PYTHONPATH=root)
    p = subprocess.run([sys.executable, "-c", code], cwd=root, env=env, capture_output=True, text=True, timeout=300)
    assert p.returncode == 0 and "torchcomm ok" in p.stdout, p.stdout[-2000:] + p.stderr[-4000:]
