"""Pins of the oracle's NEXT(4) building blocks and solver (section IV.D,
P:830-858; readings R27-R29): the fixed-order SpMV and dot product and the
block-Jacobi preconditioned BiCGSTAB.  CPU only."""
import numpy as np
import scipy.sparse as sp
import scipy.sparse.linalg as spla

import bj_synth as S
import oracle


def _csr(M):
    M = sp.csr_matrix(M)
    return M.indptr.astype(np.int64), M.indices.astype(np.int32), M.data.astype(np.float64)


def test_spmv_exact_on_integers_and_tree_order():
    rng = np.random.default_rng(51)
    D = rng.integers(-9, 10, size=(300, 300)) * (rng.random((300, 300)) < 0.3)
    D[:, 17] = rng.integers(-9, 10, 300)             # a dense column, rows longer than 32 entries too
    rp, ci, va = _csr(D)
    x = rng.integers(-20, 21, 300).astype(np.float64)
    assert np.array_equal(oracle.spmv(rp, ci, va, x), D @ x)
    # order pin: entries (2^-53, 2^-53, 1) sit in lanes 0, 1, 2; the butterfly adds
    # 1 + 2^-53 first (-> 1), a left-to-right sum would give 1 + 2^-52
    rp = np.array([0, 3], np.int64)
    ci = np.array([0, 1, 2], np.int32)
    va = np.array([2.0 ** -53, 2.0 ** -53, 1.0])
    assert oracle.spmv(rp, ci, va, np.ones(3))[0] == 1.0
    # a row slab with global columns (col_offset)
    rp2, ci2, va2 = _csr(D[100:200])
    y = oracle.spmv(rp2, ci2, va2, x[:], col_offset=0)
    assert np.array_equal(y, D[100:200] @ x)


def test_dot_exact_on_integers_and_chunk_order():
    rng = np.random.default_rng(52)
    for n in (1, 255, 8192, 8193, 50000):
        x = rng.integers(-100, 101, n).astype(np.float64)
        y = rng.integers(-100, 101, n).astype(np.float64)
        assert oracle.dot(x, y) == float(np.dot(x.astype(np.int64), y.astype(np.int64)))
    # order pin: thread 0 holds 2^-53 and 2^-53 (elements 0 and 256), thread 1 holds 1:
    # thread sums 2^-52 and 1, tree 1 + 2^-52 (exact); a left-to-right sum gives 1 + 2^-53 -> 1... + 2^-53 -> 1
    x = np.zeros(300)
    x[0] = x[256] = 2.0 ** -53
    x[1] = 1.0
    assert oracle.dot(x, np.ones(300)) == 1.0 + 2.0 ** -52
    z = rng.uniform(-1, 1, 100000)
    exact = np.sum(z.astype(np.longdouble) * z.astype(np.longdouble))
    assert abs(oracle.dot(z, z) - float(exact)) <= 1e-12 * float(exact)


def test_bicgstab_exact_preconditioner_converges_in_one_step():
    """One block covering the whole (n <= 32) system: M^-1 = A^-1, so the
    first iterate is the solution (to rounding)."""
    rng = np.random.default_rng(53)
    A = rng.uniform(-1, 1, (24, 24)) + 24 * np.eye(24)
    rp, ci, va = _csr(A)
    b = np.ones(24)
    x, it, res, *_ = oracle.bicgstab(rp, ci, va, np.array([0, 24], np.int32), b)
    assert it == 1 and res <= 1e-13
    assert np.abs(x - np.linalg.solve(A, b)).max() <= 1e-13


def test_bicgstab_fem_block_jacobi():
    """The section IV.D set-up on a small synthetic FEM matrix: b = ones,
    x0 = 0, stop at a 10^6 residual reduction; the true residual agrees with
    the recurrence and the solution with a direct solver."""
    g = S.FemGrid(10, 9, 8)
    rp, ci, va = g.csr()
    n = g.n
    bp = S.uniform_block_ptr(n, 24)
    b = np.ones(n)
    x, it, res, *_ = oracle.bicgstab(rp, ci, va, bp, b)
    assert 1 < it < 200 and res <= 1e-6
    A = sp.csr_matrix((va, ci, rp), shape=(n, n))
    true_res = np.linalg.norm(b - A @ x) / np.linalg.norm(b)
    assert true_res <= 2e-6
    xd = spla.spsolve(A.tocsc(), b)
    assert np.linalg.norm(x - xd) / np.linalg.norm(xd) <= 1e-4
    # point Jacobi (1x1 blocks) converges as well on this diagonally dominant matrix
    x1, it1, res1, *_ = oracle.bicgstab(rp, ci, va, S.uniform_block_ptr(n, 1), b)
    assert res1 <= 1e-6 and it1 < 200
    # not converged within maxit -> maxit + 1
    _, it2, res2, *_ = oracle.bicgstab(rp, ci, va, bp, b, tol=1e-30, maxit=3)
    assert it2 == 4 and res2 > 1e-30


def test_dot_sharded_r30():
    """R30: per-shard R28 values summed in shard order from +0; one shard is R28."""
    rng = np.random.default_rng(54)
    z = rng.uniform(-1, 1, 30000)
    w = rng.uniform(-1, 1, 30000)
    assert oracle.dot_sharded(z, w, [0, 30000]) == oracle.dot(z, w)
    bnd = [0, 7001, 7001, 19999, 30000]                      # an empty shard too
    manual = 0.0
    for a, b in zip(bnd[:-1], bnd[1:]):
        manual = manual + oracle.dot(z[a:b], w[a:b])
    assert oracle.dot_sharded(z, w, bnd) == manual
    zi = rng.integers(-50, 51, 30000).astype(np.float64)
    assert oracle.dot_sharded(zi, zi, bnd) == float(np.dot(zi.astype(np.int64), zi.astype(np.int64)))
    # order pin: elements (1, 2^-53, 0, 2^-53).  One chunk: the tree adds positions
    # 1 and 3 first (2^-52), then 1 + 2^-52.  Shards [0,1) [1,2) [2,4): 1 + 2^-53 + 2^-53 -> 1.
    x = np.array([1.0, 2.0 ** -53, 0.0, 2.0 ** -53])
    assert oracle.dot(x, np.ones(4)) == 1.0 + 2.0 ** -52
    assert oracle.dot_sharded(x, np.ones(4), [0, 1, 2, 4]) == 1.0


def test_bicgstab_sharded_r30():
    g = S.FemGrid(10, 9, 8)
    rp, ci, va = g.csr()
    n = g.n
    bp = S.uniform_block_ptr(n, 24)
    b = np.ones(n)
    x1, it1, res1, *_ = oracle.bicgstab(rp, ci, va, bp, b)
    xs, its, ress, *_ = oracle.bicgstab(rp, ci, va, bp, b, bounds=[0, n])
    assert its == it1 and ress == res1 and np.array_equal(xs.view(np.uint64), x1.view(np.uint64))
    bnd = [0, 3 * 10 * 9 * 3, 3 * 10 * 9 * 5, n]            # z-slab shards
    x3, it3, res3, *_ = oracle.bicgstab(rp, ci, va, bp, b, bounds=bnd)
    A = sp.csr_matrix((va, ci, rp), shape=(n, n))
    assert res3 <= 1e-6 and np.linalg.norm(b - A @ x3) / np.linalg.norm(b) <= 2e-6
    assert abs(it3 - it1) <= 2
