"""Pins of the oracle's inversion-based variant (NEXT(3) of SURVEY 8(f);
PAPER.md P:206-214; readings R23-R26 in DESIGN.md): GETRI by
Gauss-Jordan elimination with implicit pivoting, and the GEMV apply.
CPU only."""
from fractions import Fraction

import numpy as np
import pytest

import bj_synth as S
import oracle
from exact_gje import gje_implicit, inverse_exact


def _exact_double(v: Fraction) -> bool:
    return float(v) == v and abs(float(v)) < 2.0 ** 1000


def test_exact_rational_gje_is_the_inverse():
    """The exact R23-R26 algorithm computes A^-1 (A * X == I exactly) and agrees
    with the textbook explicit-swap Gauss-Jordan inverse."""
    rng = np.random.default_rng(11)
    for _ in range(150):
        m = int(rng.integers(1, 7))
        A = rng.integers(-4, 5, size=(m, m))
        X, perm, info, _ = gje_implicit(A.tolist())
        ref = inverse_exact(A.tolist())
        if ref is None:
            assert info > 0
            continue
        assert info == 0
        assert X == ref
        for i in range(m):
            for j in range(m):
                assert sum(Fraction(int(A[i][t])) * X[t][j] for t in range(m)) == (1 if i == j else 0)


def test_oracle_matches_exact_rational_bitwise():
    """Dyadic blocks whose every GJE intermediate is a binary64 number: the
    fp64 oracle reproduces the exact algorithm bit for bit (pivots, info,
    inverse)."""
    rng = np.random.default_rng(12)
    hits = 0
    for _ in range(3000):
        m = int(rng.integers(1, 6))
        # entries +-2^e and small integers: many exact-binary eliminations
        A = rng.choice([-4.0, -2.0, -1.0, -0.5, 0.5, 1.0, 2.0, 4.0, 0.0, 3.0, -3.0], size=(m, m))
        X, perm, info, inter = gje_implicit(A.tolist())
        if info or not all(_exact_double(v) for v in inter):
            continue
        hits += 1
        Xo, po, io = oracle.getri(A)
        assert io == 0 and po.tolist() == perm
        assert np.array_equal(Xo, np.array([[float(v) for v in row] for row in X]))
    assert hits > 300


def test_closed_form_2x2_and_3x3():
    rng = np.random.default_rng(13)
    for _ in range(200):
        a, b, c, d = rng.uniform(-1, 1, 4)
        A = np.array([[a, b], [c, d]])
        det = a * d - b * c
        if abs(det) < 1e-3:
            continue
        ref = np.array([[d, -b], [-c, a]]) / det
        X, _, info = oracle.getri(A)
        kappa = np.linalg.cond(A, np.inf)
        assert info == 0 and np.abs(X - ref).max() <= 8 * kappa * 2.0 ** -52 * np.abs(ref).max()
    for _ in range(200):
        A = rng.uniform(-1, 1, (3, 3))
        adj = np.array([[np.linalg.det(np.delete(np.delete(A, i, 0), j, 1)) * (-1) ** (i + j) for i in range(3)]
                        for j in range(3)])
        ref = adj.T.T / np.linalg.det(A)
        X, _, info = oracle.getri(A)
        kappa = np.linalg.cond(A, np.inf)
        if kappa > 1e6:
            continue
        assert np.abs(X - ref).max() <= 50 * kappa * 2.0 ** -52 * np.abs(ref).max()


def test_special_matrices_exact():
    m = 7
    rng = np.random.default_rng(14)
    X, perm, info = oracle.getri(np.eye(m))
    assert info == 0 and np.array_equal(X, np.eye(m)) and perm.tolist() == list(range(m))
    P = np.eye(m)[rng.permutation(m)]
    X, _, info = oracle.getri(P)
    assert info == 0 and np.array_equal(X, P.T)
    dg = rng.uniform(0.5, 4, m)
    X, _, info = oracle.getri(np.diag(dg))
    assert info == 0 and np.array_equal(np.diag(X), 1.0 / dg) and np.count_nonzero(X - np.diag(np.diag(X))) == 0
    Z = np.zeros((m, m))
    _, _, info = oracle.getri(Z)
    assert info == 1
    # fp32 mode: the same special cases in binary32
    X, _, info = oracle.getri(np.diag(dg).astype(np.float32))
    assert info == 0 and np.array_equal(np.diag(X), (np.float32(1) / dg.astype(np.float32)))


def test_random_blocks_residual_and_lapack():
    """A * Dinv ~ I and agreement with LAPACK (numpy.linalg.inv) to kappa*u;
    pivots equal GETRF's on tie-free random blocks in the vast majority."""
    sizes = S.block_sizes(400, 1, 32, first=99)
    vec, val = oracle.layout(sizes, 8)
    A = S.block_values(sizes, val, first=99)
    Dinv, perm, info = oracle.getri_batch(sizes, val, vec, A)
    LU, perm_lu, _ = oracle.getrf_batch(sizes, val, vec, A)
    assert (info == 0).all()
    same = 0
    for i, m in enumerate(sizes):
        Ai = A[val[i]: val[i] + m * m].reshape(m, m, order="F")
        Xi = Dinv[val[i]: val[i] + m * m].reshape(m, m, order="F")
        kappa = np.linalg.cond(Ai, np.inf)
        res = np.abs(Ai @ Xi - np.eye(m)).max()
        assert res <= 40 * m * kappa * 2.0 ** -52
        ref = np.linalg.inv(Ai)
        assert np.abs(Xi - ref).max() <= 40 * m * kappa * 2.0 ** -52 * np.abs(ref).max()
        same += np.array_equal(perm[vec[i]: vec[i] + m], perm_lu[vec[i]: vec[i] + m])
    assert same >= 0.97 * len(sizes)


def test_gemv_apply_pins():
    """y = Dinv x: integer data (exact sums) equal numpy's product; unit
    vectors select columns (a -0 entry gives +0: the chain starts at +0);
    the fp32 mode is the binary32 chain."""
    rng = np.random.default_rng(15)
    for m in (1, 5, 17, 32):
        D = rng.integers(-50, 51, size=(m, m)).astype(np.float64)
        x = rng.integers(-50, 51, size=m).astype(np.float64)
        assert np.array_equal(oracle.gemv(D, x), D @ x)
        for j in range(m):
            e = np.zeros(m)
            e[j] = 1.0
            assert np.array_equal(oracle.gemv(D, e), D[:, j] + 0.0)
    D = np.array([[-0.0, 1.0], [2.0, -0.0]])
    y = oracle.gemv(D, np.array([1.0, 0.0]))
    assert np.signbit(y[0]) == False and y[1] == 2.0
    # accumulation order: a case where the order of the fma chain decides the bits
    D = np.array([[1.0, 2.0 ** -53, 2.0 ** -53]])
    D = np.vstack([D, D, D])
    y = oracle.gemv(D, np.array([1.0, 1.0, 1.0]))
    assert y[0] == 1.0                       # ((0 + 1) + 2^-53) + 2^-53, ties to even each time
    # binary32 mode: the same order pin with 2^-24, and exact small-grid sums
    D32 = np.array([[1.0, 2.0 ** -24, 2.0 ** -24]] * 3, np.float32)
    assert oracle.gemv(D32, np.ones(3, np.float32))[0] == np.float32(1.0)
    D32 = (rng.integers(-64, 65, (9, 9)) / 64.0).astype(np.float32)
    x32 = (rng.integers(-64, 65, 9) / 64.0).astype(np.float32)
    assert np.array_equal(oracle.gemv(D32, x32), (D32.astype(np.float64) @ x32.astype(np.float64)).astype(np.float32))


def test_batch_drivers_and_invalid_sizes():
    sizes = np.array([0, 3, 33, 1, -2, 5], np.int32)
    vec, val = oracle.layout(sizes, 8)
    A = np.random.default_rng(16).uniform(-1, 1, int(val[-1]))
    Dinv, perm, info = oracle.getri_batch(sizes, val, vec, A)
    assert info[2] == -1 and info[4] == -1 and info[0] == 0
    for i in (1, 3, 5):
        m = sizes[i]
        X, p, inf = oracle.getri(A[val[i]: val[i] + m * m].reshape(m, m, order="F"))
        assert np.array_equal(Dinv[val[i]: val[i] + m * m], X.reshape(-1, order="F"))
    x = np.random.default_rng(17).uniform(-1, 1, int(vec[-1]))
    y = oracle.gemv_batch(sizes, val, vec, Dinv, x)
    for i in (1, 3, 5):
        m = sizes[i]
        Xi = Dinv[val[i]: val[i] + m * m].reshape(m, m, order="F")
        assert np.array_equal(y[vec[i]: vec[i] + m], oracle.gemv(Xi, x[vec[i]: vec[i] + m]))
