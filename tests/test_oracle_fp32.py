"""Pins of the oracle's binary32 mode (R12: fp32 pivots and bits are fixed by
bjo_*_s with fmaf, no FTZ): exact-rational cases whose every intermediate is a
binary32 number, and cases that separate a single-rounding fmaf from a
double-rounded fp64 fma (the mistake an fp64 oracle in fp32 clothing makes).
CPU only."""
from fractions import Fraction

import numpy as np

import oracle
from exact_lu import lu_implicit, representable32, solve_with_inter


def _cases32(seed, count, mmax=6):
    rng = np.random.default_rng(seed)
    vals = np.array([0, 1, -1, 2, -2, 4, -4, 8, -8, 3, -3], dtype=np.int64)
    got = tries = 0
    while got < count and tries < 80 * count:
        tries += 1
        m = int(rng.integers(1, mmax + 1))
        A = rng.choice(vals, size=(m, m))
        LU, perm, info, inter = lu_implicit(A.tolist())
        if all(representable32(q) for q in inter):
            got += 1
            yield A, LU, perm, info


def test_exact_rational_getrf_fp32_bitwise():
    n = sing = 0
    for A, LUx, permx, infox in _cases32(41, 400):
        LU, perm, info = oracle.getrf(A.astype(np.float32))
        assert LU.dtype == np.float32
        assert perm.tolist() == permx and info == infox
        assert np.array_equal(LU, np.array([[np.float32(float(q)) for q in r] for r in LUx], np.float32))
        n += 1
        sing += infox != 0
    assert n == 400 and sing > 5


def test_exact_rational_getrs_fp32_bitwise():
    rng = np.random.default_rng(42)
    hits = 0
    for A, LUx, permx, infox in _cases32(43, 400):
        if infox:
            continue
        m = A.shape[0]
        b = rng.choice(np.array([0, 1, -1, 2, -4, 8, 3]), size=m)
        y, inter = solve_with_inter(LUx, permx, [Fraction(int(v)) for v in b])
        if not all(representable32(q) for q in inter):
            continue
        LU, perm, _ = oracle.getrf(A.astype(np.float32))
        x = oracle.getrs(LU, perm, b.astype(np.float32))
        assert np.array_equal(x, np.array([np.float32(float(q)) for q in y], np.float32))
        hits += 1
    assert hits > 100


# 641 * 6700417 = 2^32 + 1: with a = 641*2^-10 and u = 6700417*2^-46 the product
# a*u = 2^-24 + 2^-56.  1 + a*u lies just above the binary32 midpoint 1 + 2^-24:
# fmaf rounds it up to 1 + 2^-23; rounding through binary64 first lands on the
# midpoint exactly and ties-to-even then gives 1.0 (double rounding).
C = np.float32(-641.0 * 2.0 ** -10)
U = np.float32(6700417.0 * 2.0 ** -46)


def test_getrf_fp32_single_rounding_fma():
    A = np.array([[1.0, U], [C, 1.0]], dtype=np.float32)      # row 0 pivots (|1| > |C|), l = C
    LU, perm, info = oracle.getrf(A)
    assert perm.tolist() == [0, 1] and info == 0
    assert LU[1, 0] == C
    assert LU[1, 1] == np.float32(1.0 + 2.0 ** -23)          # fmaf; a double-rounded fma gives 1.0
    assert float(LU[1, 1]) != float(np.float32(np.float64(1.0) + np.float64(-C) * np.float64(U)))


def test_getrs_fp32_single_rounding_fma():
    LU = np.array([[1.0, 0.0], [C, 1.0]], dtype=np.float32)   # L10 = C, U = I
    x = oracle.getrs(LU, np.array([0, 1], np.int32), np.array([U, 1.0], np.float32))
    assert x[0] == U and x[1] == np.float32(1.0 + 2.0 ** -23)


def test_getri_and_gemv_fp32_single_rounding():
    """GJE (R23) and the GEMV apply (R26) in binary32 use fmaf as well."""
    A = np.array([[1.0, U], [C, 1.0]], dtype=np.float32)
    # step 0 (pivot row 0, d = 1): W(1,1) = fma(-C, U, 1) = 1 + 2^-23 (not 1.0);
    # step 1 pivots row 1 with d = 1 + 2^-23, so Dinv(1,1) = 1 / (1 + 2^-23)
    X, perm, info = oracle.getri(A)
    assert info == 0 and perm.tolist() == [0, 1]
    d1 = np.float32(1.0 + 2.0 ** -23)
    assert X[1, 1] == np.float32(1.0) / d1
    # apply: acc = fma(1, 1, +0) = 1, then fma(U, 641*2^-10, 1) = 1 + 2^-23
    D = np.array([[1.0, U], [0.0, 1.0]], np.float32)
    y = oracle.gemv(D, np.array([1.0, np.float32(641.0 * 2.0 ** -10)], np.float32))
    assert y[0] == d1
