"""Pins of the oracle GETRF (Fig. 1) -- CPU only.

Each test checks the oracle against something other than itself: exact
rationals, the textbook explicit-swap variant, LAPACK, closed forms, special
matrices and invariants.
"""
import os
from fractions import Fraction

import numpy as np
import pytest
import torch

import oracle
from exact_lu import lu_implicit, matmul, representable, split_lu

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _parse_golden(name):
    out = {}
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        key, rest = line.split(None, 1)
        rows = [[Fraction(t) for t in r.split()] for r in rest.split(";")]
        out[key] = rows if len(rows) > 1 else rows[0]
    return out


def _bits(a):
    a = np.ascontiguousarray(a)
    return a.view(np.uint64 if a.dtype == np.float64 else np.uint32)


def _rng(seed):
    return np.random.default_rng(seed)


# ---------------------------------------------------------------- golden
def test_golden_tie_example():
    """Hand-worked Fig. 1 example with an exact tie at step 1 (R1)."""
    g = _parse_golden("tie3x3.txt")
    A = np.array([[float(x) for x in r] for r in g["A"]])
    for dt in (np.float64, np.float32):
        LU, perm, info = oracle.getrf(A.astype(dt))
        assert info == 0
        assert perm.tolist() == [int(x) for x in g["perm_implicit"]]
        assert np.array_equal(LU, np.array([[float(x) for x in r] for r in g["LU_implicit"]], dt))
        LUe, perme, _ = oracle.getrf(A.astype(dt), "explicit")
        assert perme.tolist() == [int(x) for x in g["perm_explicit"]]
        assert np.array_equal(LUe, np.array([[float(x) for x in r] for r in g["LU_explicit"]], dt))


# ---------------------------------------------------------------- exact rationals
def _exact_cases(seed, count, mmax=6):
    """Random small matrices with entries in {0,+-1,+-2,+-4,+-8}; keep those
    whose exact elimination stays in binary64 (then fp64 must be exact)."""
    rng = _rng(seed)
    vals = np.array([0, 1, -1, 2, -2, 4, -4, 8, -8], dtype=np.int64)
    got = 0
    tries = 0
    while got < count and tries < 50 * count:
        tries += 1
        m = int(rng.integers(1, mmax + 1))
        A = rng.choice(vals, size=(m, m))
        LU, perm, info, inter = lu_implicit(A.tolist())
        if all(representable(q) for q in inter):
            got += 1
            yield A, LU, perm, info


def test_exact_rational_pins_pivots_and_bits():
    n_ties = 0
    n_sing = 0
    for A, LUx, permx, infox in _exact_cases(1, 400):
        m = A.shape[0]
        # the exact reference is itself pinned by the exact invariant P A = L U
        L, U = split_lu(LUx)
        PA = [[Fraction(int(v)) for v in A[permx[k]]] for k in range(m)]
        if infox == 0:
            assert matmul(L, U) == PA
        LU, perm, info = oracle.getrf(A.astype(np.float64))
        assert perm.tolist() == permx
        assert info == infox
        assert np.array_equal(LU, np.array([[float(q) for q in r] for r in LUx]))
        n_sing += infox != 0
        # count exact ties that occurred in the pivot search
        col = np.abs(A[:, 0])
        n_ties += int((col == col.max()).sum() > 1)
    assert n_ties > 50 and n_sing > 5          # the sample exercises ties and zero pivots


def test_exact_rational_singular_invariant():
    """Singular blocks: P A = L U still holds exactly (R4 skips no-op steps)."""
    rng = _rng(2)
    done = 0
    for _ in range(2000):
        m = int(rng.integers(2, 6))
        A = rng.choice(np.array([0, 1, -1, 2, -2]), size=(m, m))
        A[:, int(rng.integers(0, m))] = 0                    # force a zero column
        LUx, permx, infox, inter = lu_implicit(A.tolist())
        if not all(representable(q) for q in inter):
            continue
        assert infox > 0
        L, U = split_lu(LUx)
        PA = [[Fraction(int(v)) for v in A[permx[k]]] for k in range(m)]
        assert matmul(L, U) == PA
        LU, perm, info = oracle.getrf(A.astype(np.float64))
        assert info == infox and perm.tolist() == permx
        assert np.array_equal(LU, np.array([[float(q) for q in r] for r in LUx]))
        assert not np.isnan(LU).any()
        done += 1
    assert done > 100


# ---------------------------------------------------------------- explicit variant
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_implicit_equals_textbook_explicit_on_tie_free_inputs(dt):
    """with no exact ties both variants do identical per-row work."""
    rng = _rng(3)
    for m in list(range(1, 33)) + [32] * 20:
        for _ in range(6):
            A = rng.uniform(-1, 1, size=(m, m)).astype(dt)
            LU, perm, info = oracle.getrf(A)
            LUe, perme, infoe = oracle.getrf(A, "explicit")
            assert info == infoe == 0
            assert np.array_equal(perm, perme)
            assert np.array_equal(_bits(LU), _bits(LUe))


# ---------------------------------------------------------------- LAPACK
def _ipiv_to_perm(ipiv):
    m = len(ipiv)
    p = list(range(m))
    for k in range(m):
        j = int(ipiv[k]) - 1
        p[k], p[j] = p[j], p[k]
    return np.array(p)


def test_pivots_match_lapack():
    """LAPACK getrf (torch CPU) picks the same pivots on random blocks and
    agrees on the factors to rounding (it is blocked and scales by 1/d)."""
    rng = _rng(4)
    mism = 0
    total = 0
    for m in (1, 2, 4, 7, 13, 16, 23, 31, 32):
        A = rng.uniform(-1, 1, size=(300, m, m))
        LUt, piv = torch.linalg.lu_factor(torch.from_numpy(A))
        for t in range(A.shape[0]):
            LU, perm, info = oracle.getrf(A[t])
            pl = _ipiv_to_perm(piv[t].numpy())
            total += 1
            if not np.array_equal(perm, pl):
                mism += 1
                continue
            np.testing.assert_allclose(LU, LUt[t].numpy(), rtol=0, atol=1e-11)
    assert mism == 0, f"{mism}/{total} pivot mismatches vs LAPACK"


# ---------------------------------------------------------------- invariants
@pytest.mark.parametrize("dt,tol", [(np.float64, 1e-13), (np.float32, 1e-5)])
def test_invariants_random(dt, tol):
    rng = _rng(5)
    for m in range(1, 33):
        for _ in range(10):
            A = rng.uniform(-1, 1, size=(m, m)).astype(dt)
            LU, perm, info = oracle.getrf(A)
            assert info == 0
            assert sorted(perm.tolist()) == list(range(m))
            L = np.tril(LU.astype(np.float64), -1) + np.eye(m)
            U = np.triu(LU.astype(np.float64))
            assert np.abs(L).max() <= 1.0                       # |a| <= |d| => |a/d| <= 1
            # U(k,k) has the maximal |.| among the candidates of step k
            PA = A.astype(np.float64)[perm]
            res = np.abs(PA - L @ U).max()
            assert res <= 4 * m * np.finfo(dt).eps * np.abs(L).sum(1).max() * np.abs(U).sum(1).max()
            # relative residual within the north-star tolerance
            assert np.abs(PA - L @ U).sum(1).max() / np.abs(A).sum(1).max() <= tol


def test_pivot_is_max_of_candidates():
    rng = _rng(6)
    for m in (5, 17, 32):
        A = rng.uniform(-1, 1, size=(m, m))
        LU, perm, _ = oracle.getrf(A)
        # replay with exact rationals on the fp64 values: the chosen pivot at
        # step 0 is the largest |a_i0|
        assert perm[0] == int(np.argmax(np.abs(A[:, 0])))
        assert abs(LU[0, 0]) == np.abs(A[:, 0]).max()


# ---------------------------------------------------------------- special cases
def test_special_matrices():
    rng = _rng(7)
    # m = 1
    LU, perm, info = oracle.getrf(np.array([[-3.5]]))
    assert LU[0, 0] == -3.5 and perm.tolist() == [0] and info == 0
    # identity / diagonal -> perm identity, L = I
    for m in (1, 5, 32):
        D = np.diag(rng.uniform(0.5, 2, m) * rng.choice([-1, 1], m))
        LU, perm, info = oracle.getrf(D)
        assert perm.tolist() == list(range(m)) and np.array_equal(LU, D)
    # permutation matrix: rows of ones -> perm = order of the ones, L = U = I
    for m in (3, 8, 32):
        pi = rng.permutation(m)
        Pm = np.eye(m)[pi]                       # row i has its one in column pi[i]
        LU, perm, info = oracle.getrf(Pm)
        assert np.array_equal(LU, np.eye(m))
        assert np.array_equal(Pm[perm], np.eye(m))
    # strictly column diagonally dominant -> GEPP never swaps (Golub & Van Loan)
    for m in (4, 16, 32):
        A = rng.uniform(-1, 1, size=(m, m))
        A[np.arange(m), np.arange(m)] = np.abs(A).sum(0) + 1.0
        LU, perm, info = oracle.getrf(A)
        assert perm.tolist() == list(range(m))
    # zero matrix: info = 1, perm identity, LU all zero, no NaN
    LU, perm, info = oracle.getrf(np.zeros((6, 6)))
    assert info == 1 and perm.tolist() == list(range(6)) and not LU.any()


def test_zero_pivot_keeps_signed_zeros_and_continues():
    """R4: a candidate column of +-0 skips SCAL and GER (no NaN, -0 kept)."""
    A = np.array([[0.0, 2.0, 1.0], [-0.0, 1.0, 3.0], [0.0, 4.0, -1.0]])
    LU, perm, info = oracle.getrf(A)
    assert info == 1
    assert perm.tolist() == [0, 2, 1]
    assert not np.isnan(LU).any()
    assert np.signbit(LU[2, 0])               # row 1 (-0.0) untouched by step 0


def test_padding_invariance():
    """a k x k block embedded in 32 x 32 (identity padding) factors
    to the same bits in its leading part."""
    rng = _rng(8)
    for k in (1, 3, 9, 16, 31):
        A = rng.uniform(-1, 1, size=(k, k))
        B = np.eye(32)
        B[:k, :k] = A
        LU, perm, _ = oracle.getrf(A)
        LUb, permb, _ = oracle.getrf(B)
        assert permb[:k].tolist() == perm.tolist()
        assert permb[k:].tolist() == list(range(k, 32))
        assert np.array_equal(_bits(LUb[:k, :k].copy()), _bits(LU))


def test_batch_matches_single_and_flags_bad_sizes():
    sizes = np.array([4, 0, 33, 1, 16, 32, -1, 7], dtype=np.int32)
    vec, val = oracle.layout(sizes, 8)
    vals = _rng(9).uniform(-1, 1, size=int(val[-1]))
    LU, perm, info = oracle.getrf_batch(sizes, val, vec, vals)
    for i, m in enumerate(sizes):
        if m < 0 or m > 32:
            assert info[i] == -1
            n = max(int(m), 0) ** 2
            assert np.array_equal(LU[val[i]: val[i] + n], vals[val[i]: val[i] + n])
            continue
        A = vals[val[i]: val[i] + m * m].reshape(m, m, order="F")
        L1, p1, i1 = oracle.getrf(A)
        assert np.array_equal(LU[val[i]: val[i] + m * m], L1.flatten(order="F"))
        assert np.array_equal(perm[vec[i]: vec[i] + m], p1)
        assert info[i] == i1
