"""Pins of the oracle GETRS (Fig. 2) -- CPU only."""
import os
from fractions import Fraction

import numpy as np
import pytest
import torch

import oracle
from exact_lu import lu_implicit, representable, solve
from test_oracle_getrf import _bits, _exact_cases, _parse_golden


def test_golden_tie_example_solve():
    g = _parse_golden("tie3x3.txt")
    A = np.array([[float(x) for x in r] for r in g["A"]])
    b = np.array([float(x) for x in g["b"]])
    xs = np.array([float(x) for x in g["x"]])
    LU, perm, _ = oracle.getrf(A)
    x = oracle.getrs(LU, perm, b)
    # kappa_inf(A) * u bound: |x - x*| <= few ulps here (kappa ~ 60)
    np.testing.assert_allclose(x, xs, rtol=0, atol=64 * np.finfo(float).eps)


def test_closed_form_2x2_and_3x3_inverses():
    rng = np.random.default_rng(11)
    for _ in range(500):
        a, b_, c, d = rng.uniform(-1, 1, 4)
        A = np.array([[a, b_], [c, d]])
        det = a * d - b_ * c
        if abs(det) < 1e-3:
            continue
        Ainv = np.array([[d, -b_], [-c, a]]) / det
        LU, perm, _ = oracle.getrf(A)
        kappa = np.abs(A).sum(1).max() * np.abs(Ainv).sum(1).max()
        for j in range(2):
            e = np.eye(2)[j]
            x = oracle.getrs(LU, perm, e)
            assert np.abs(x - Ainv[:, j]).max() <= 8 * kappa * np.finfo(float).eps * np.abs(Ainv).max()
    for _ in range(300):
        A = rng.uniform(-1, 1, size=(3, 3))
        det = (A[0, 0] * (A[1, 1] * A[2, 2] - A[1, 2] * A[2, 1])
               - A[0, 1] * (A[1, 0] * A[2, 2] - A[1, 2] * A[2, 0])
               + A[0, 2] * (A[1, 0] * A[2, 1] - A[1, 1] * A[2, 0]))
        if abs(det) < 1e-2:
            continue
        adj = np.empty((3, 3))
        for i in range(3):
            for j in range(3):
                minor = np.delete(np.delete(A, j, 0), i, 1)
                adj[i, j] = (-1) ** (i + j) * (minor[0, 0] * minor[1, 1] - minor[0, 1] * minor[1, 0])
        Ainv = adj / det
        LU, perm, _ = oracle.getrf(A)
        kappa = np.abs(A).sum(1).max() * np.abs(Ainv).sum(1).max()
        X = np.stack([oracle.getrs(LU, perm, np.eye(3)[j]) for j in range(3)], 1)
        assert np.abs(X - Ainv).max() <= 16 * kappa * np.finfo(float).eps * np.abs(Ainv).max()


def test_exact_rational_solves():
    """Where the exact solve stays in binary64 the oracle reproduces it."""
    rng = np.random.default_rng(12)
    hits = 0
    for A, LUx, permx, infox in _exact_cases(13, 300):
        if infox:
            continue
        m = A.shape[0]
        b = rng.choice(np.array([0, 1, -1, 2, -4, 8]), size=m)
        y = solve(LUx, permx, [Fraction(int(v)) for v in b])
        # every intermediate of the exact solve must be representable
        ok = all(representable(q) for q in y)
        if not ok:
            continue
        LU, perm, _ = oracle.getrf(A.astype(np.float64))
        x = oracle.getrs(LU, perm, b.astype(np.float64))
        if np.array_equal(x, np.array([float(q) for q in y])):
            hits += 1
        else:
            # an intermediate was not representable: rounding only
            np.testing.assert_allclose(x, [float(q) for q in y], rtol=1e-12, atol=1e-12)
    assert hits > 50


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_eager_equals_lazy_accumulating(dt):
    """Fig. 2: lazy (DOT) accumulated term by term == eager (AXPY) bitwise."""
    rng = np.random.default_rng(14)
    for m in range(1, 33):
        for _ in range(5):
            A = rng.uniform(-1, 1, size=(m, m)).astype(dt)
            b = rng.uniform(-1, 1, size=m).astype(dt)
            LU, perm, _ = oracle.getrf(A)
            x1 = oracle.getrs(LU, perm, b, "eager")
            x2 = oracle.getrs(LU, perm, b, "lazy")
            assert np.array_equal(_bits(x1), _bits(x2))


def test_matches_lapack_lu_solve():
    rng = np.random.default_rng(15)
    for m in (1, 3, 8, 17, 32):
        for _ in range(40):
            A = rng.uniform(-1, 1, size=(m, m))
            b = rng.uniform(-1, 1, size=m)
            LU, perm, _ = oracle.getrf(A)
            x = oracle.getrs(LU, perm, b)
            xr = torch.linalg.solve(torch.from_numpy(A), torch.from_numpy(b)).numpy()
            kappa = np.linalg.cond(A, np.inf)
            assert np.abs(x - xr).max() / np.abs(xr).max() <= 50 * m * kappa * np.finfo(float).eps


@pytest.mark.parametrize("dt,tol", [(np.float64, 1e-13), (np.float32, 1e-5)])
def test_backward_error(dt, tol):
    """beta = ||A x - b||_inf / (||A||_inf ||x||_inf) computed in fp64 (R13)."""
    rng = np.random.default_rng(16)
    worst = 0.0
    for m in range(1, 33):
        for _ in range(20):
            A = rng.uniform(-1, 1, size=(m, m)).astype(dt)
            b = rng.uniform(-1, 1, size=m).astype(dt)
            LU, perm, _ = oracle.getrf(A)
            x = oracle.getrs(LU, perm, b).astype(np.float64)
            A64 = A.astype(np.float64)
            beta = np.abs(A64 @ x - b).max() / (np.abs(A64).sum(1).max() * np.abs(x).max())
            worst = max(worst, beta)
    assert worst <= tol


def test_special_solves():
    # m = 1: x = b / a
    LU, perm, _ = oracle.getrf(np.array([[3.0]]))
    assert oracle.getrs(LU, perm, np.array([1.0]))[0] == 1.0 / 3.0
    # permutation matrix: x = P^T b exactly
    rng = np.random.default_rng(17)
    pi = rng.permutation(9)
    Pm = np.eye(9)[pi]
    b = rng.uniform(-1, 1, 9)
    LU, perm, _ = oracle.getrf(Pm)
    x = oracle.getrs(LU, perm, b)
    assert np.array_equal(Pm @ x, b)
    # diagonal: x = b / d (one correctly rounded division per entry)
    d = rng.uniform(0.5, 2, 9)
    LU, perm, _ = oracle.getrf(np.diag(d))
    assert np.array_equal(oracle.getrs(LU, perm, b), b / d)


def test_batch_getrs_matches_single():
    import bj_synth as S
    sizes = S.block_sizes(200, 1, 32)
    vec, val = oracle.layout(sizes, 8)
    A = S.block_values(sizes, val)
    b = S.rhs_values(sizes)
    LU, perm, info = oracle.getrf_batch(sizes, val, vec, A)
    x = oracle.getrs_batch(sizes, val, vec, LU, perm, b)
    for i, m in enumerate(sizes):
        lu = LU[val[i]: val[i] + m * m].reshape(m, m, order="F")
        xi = oracle.getrs(lu, perm[vec[i]: vec[i] + m], b[vec[i]: vec[i] + m])
        assert np.array_equal(_bits(xi), _bits(x[vec[i]: vec[i] + m].copy()))
