"""CPU oracle for the block-Jacobi hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_icpp_anztdfq17_b200``) never imports it and shares
no code with it.

The arithmetic lives in ``bj_oracle.c`` (plain C99, explicit ``fma``/``fmaf``,
IEEE division, compiled with ``-ffp-contract=off``); this module only
marshals numpy arrays through ctypes.  Every function cites the passage of
``/root/reference/PAPER.md`` it follows in the C source.

Pinned by ``tests/test_oracle_*.py`` (``-m "not gpu"``): exact-rational LU,
textbook explicit-swap LU, LAPACK pivots, closed-form inverses, brute-force
densification, brute-force partition search and the invariants listed in
DESIGN.md section 4.  No function here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bj_oracle.c")
_LIB = os.path.join(_HERE, "libbj_oracle.so")

CFLAGS = ["-std=gnu99", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
          "-fPIC", "-shared", "-Wall"]


def build(force: bool = False) -> str:
    """Compile bj_oracle.c -> libbj_oracle.so (gcc).  Returns the path."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_LIB)
        _declare(_lib)
    return _lib


_p = ctypes.c_void_p
_i64 = ctypes.c_int64
_i32 = ctypes.c_int


def _declare(L):
    for s in ("d", "s"):
        for n in (f"bjo_getrf_{s}", f"bjo_getrf_explicit_{s}"):
            getattr(L, n).argtypes = [_i32, _p, _p]
            getattr(L, n).restype = _i32
        for n in (f"bjo_getrs_{s}", f"bjo_getrs_lazy_{s}"):
            getattr(L, n).argtypes = [_i32, _p, _p, _p, _p]
            getattr(L, n).restype = None
        getattr(L, f"bjo_getrf_batch_{s}").argtypes = [_i64, _p, _p, _p, _p, _p, _p, _i32]
        getattr(L, f"bjo_getrf_batch_{s}").restype = None
        getattr(L, f"bjo_getrs_batch_{s}").argtypes = [_i64, _p, _p, _p, _p, _p, _p, _p, _i32]
        getattr(L, f"bjo_getrs_batch_{s}").restype = None
    for s in ("d", "s"):
        getattr(L, f"bjo_getri_{s}").argtypes = [_i32, _p, _p]
        getattr(L, f"bjo_getri_{s}").restype = _i32
        getattr(L, f"bjo_gemv_{s}").argtypes = [_i32, _p, _p, _p]
        getattr(L, f"bjo_gemv_{s}").restype = None
        getattr(L, f"bjo_getri_batch_{s}").argtypes = [_i64, _p, _p, _p, _p, _p, _p, _i32]
        getattr(L, f"bjo_getri_batch_{s}").restype = None
        getattr(L, f"bjo_gemv_batch_{s}").argtypes = [_i64, _p, _p, _p, _p, _p, _p, _i32]
        getattr(L, f"bjo_gemv_batch_{s}").restype = None
    L.bjo_spmv_d.argtypes = [_i64, _p, _p, _p, _i64, _p, _p]
    L.bjo_spmv_d.restype = None
    L.bjo_dot_d.argtypes = [_i64, _p, _p]
    L.bjo_dot_d.restype = ctypes.c_double
    L.bjo_bicgstab_d.argtypes = [_i64, _p, _p, _p, _i64, _i64, _p, _p, _p, _p, _p, _p, ctypes.c_double, _i32, _p, _p]
    L.bjo_bicgstab_d.restype = _i32
    L.bjo_fma_vec.argtypes = [_i64, _p, _p, _p, _p]
    L.bjo_fma_vec.restype = None
    L.bjo_dot_sharded_d.argtypes = [_i64, _p, _p, _i32, _p]
    L.bjo_dot_sharded_d.restype = ctypes.c_double
    L.bjo_bicgstab_sharded_d.argtypes = [_i64, _p, _p, _p, _i64, _i64, _p, _p, _p, _p, _p, _p, ctypes.c_double,
                                         _i32, _i32, _p, _p, _p]
    L.bjo_bicgstab_sharded_d.restype = _i32
    L.bjo_layout.argtypes = [_i64, _p, _i32, _p, _p]
    L.bjo_layout.restype = None
    L.bjo_extract.argtypes = [_i64, _p, _p, _p, _i32, _i64, _i64, _p, _p, _p]
    L.bjo_extract.restype = _i32
    L.bjo_partition.argtypes = [_i64, _p, _i32, _p]
    L.bjo_partition.restype = None
    L.bjo_max_threads.argtypes = []
    L.bjo_max_threads.restype = _i32


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _sfx(dtype) -> str:
    dt = np.dtype(dtype)
    if dt == np.float64:
        return "d"
    if dt == np.float32:
        return "s"
    raise TypeError(f"oracle supports float64/float32, got {dt}")


def max_threads() -> int:
    return int(lib().bjo_max_threads())


# --------------------------------------------------------------------------
# single block
# --------------------------------------------------------------------------
def getrf(A: np.ndarray, variant: str = "implicit"):
    """LU of one m x m block (Fig. 1).  Returns (LU, perm, info).

    ``variant="implicit"`` is the method (Fig. 1 bottom, swap-free, combined
    row swap at the end); ``"explicit"`` the textbook cross-check (Fig. 1
    top).  LU is column-major in a 2-D array indexed LU[i, j].
    """
    A = np.asarray(A)
    m = A.shape[0]
    assert A.shape == (m, m)
    s = _sfx(A.dtype)
    buf = np.array(A, dtype=A.dtype, order="F", copy=True)
    perm = np.zeros(max(m, 1), dtype=np.int32)
    fn = getattr(lib(), f"bjo_getrf_{s}" if variant == "implicit" else f"bjo_getrf_explicit_{s}")
    info = fn(m, _ptr(buf), _ptr(perm))
    return buf, perm[:m].copy(), int(info)


def getrs(LU: np.ndarray, perm: np.ndarray, b: np.ndarray, variant: str = "eager"):
    """x = A^{-1} b from the factors (Fig. 2)."""
    LU = np.asarray(LU)
    m = LU.shape[0]
    s = _sfx(LU.dtype)
    lu = np.array(LU, order="F", copy=True)
    p = np.ascontiguousarray(perm, dtype=np.int32)
    bb = np.ascontiguousarray(b, dtype=LU.dtype)
    x = np.zeros(max(m, 1), dtype=LU.dtype)
    fn = getattr(lib(), f"bjo_getrs_{s}" if variant == "eager" else f"bjo_getrs_lazy_{s}")
    fn(m, _ptr(lu), _ptr(p), _ptr(bb), _ptr(x))
    return x[:m].copy()


# --------------------------------------------------------------------------
# batches (packed layout, see layout())
# --------------------------------------------------------------------------
def layout(sizes: np.ndarray, elem_size: int):
    """(vec_off, val_off), both int64[nb+1] (hot-path row a1)."""
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    nb = sizes.shape[0]
    vec = np.zeros(nb + 1, dtype=np.int64)
    val = np.zeros(nb + 1, dtype=np.int64)
    lib().bjo_layout(nb, _ptr(sizes), int(elem_size), _ptr(vec), _ptr(val))
    return vec, val


def getrf_batch(sizes, val_off, vec_off, values, nthreads: int = 0):
    """In-place batched GETRF on a packed copy; returns (LU, perm, info)."""
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    val_off = np.ascontiguousarray(val_off, dtype=np.int64)
    vec_off = np.ascontiguousarray(vec_off, dtype=np.int64)
    A = np.array(values, copy=True)
    s = _sfx(A.dtype)
    nb = sizes.shape[0]
    perm = np.zeros(max(int(vec_off[nb]), 1), dtype=np.int32)
    info = np.zeros(max(nb, 1), dtype=np.int32)
    getattr(lib(), f"bjo_getrf_batch_{s}")(nb, _ptr(sizes), _ptr(val_off), _ptr(vec_off),
                                           _ptr(A), _ptr(perm), _ptr(info), int(nthreads))
    return A, perm[: int(vec_off[nb])], info[:nb]


def getrs_batch(sizes, val_off, vec_off, LU, perm, b, nthreads: int = 0):
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    val_off = np.ascontiguousarray(val_off, dtype=np.int64)
    vec_off = np.ascontiguousarray(vec_off, dtype=np.int64)
    LU = np.ascontiguousarray(LU)
    s = _sfx(LU.dtype)
    perm = np.ascontiguousarray(perm, dtype=np.int32)
    b = np.ascontiguousarray(b, dtype=LU.dtype)
    nb = sizes.shape[0]
    x = np.zeros(max(int(vec_off[nb]), 1), dtype=LU.dtype)
    getattr(lib(), f"bjo_getrs_batch_{s}")(nb, _ptr(sizes), _ptr(val_off), _ptr(vec_off),
                                           _ptr(LU), _ptr(perm), _ptr(b), _ptr(x), int(nthreads))
    return x[: int(vec_off[nb])]


def getri(A: np.ndarray):
    """Inverse of one block by Gauss-Jordan elimination with implicit partial
    pivoting (inversion-based variant; readings R23-R26).
    Returns (Dinv as a 2-D array Dinv[a, b], perm, info)."""
    A = np.asarray(A)
    m = A.shape[0]
    s = _sfx(A.dtype)
    buf = np.array(A, dtype=A.dtype, order="F", copy=True)
    perm = np.zeros(max(m, 1), dtype=np.int32)
    info = getattr(lib(), f"bjo_getri_{s}")(m, _ptr(buf), _ptr(perm))
    return buf, perm[:m].copy(), int(info)


def gemv(Dinv: np.ndarray, x: np.ndarray):
    """y = Dinv x, fma chain over columns in order from +0 (R26)."""
    Dinv = np.asarray(Dinv)
    m = Dinv.shape[0]
    s = _sfx(Dinv.dtype)
    d = np.array(Dinv, order="F", copy=True)
    xx = np.ascontiguousarray(x, dtype=Dinv.dtype)
    y = np.zeros(max(m, 1), dtype=Dinv.dtype)
    getattr(lib(), f"bjo_gemv_{s}")(m, _ptr(d), _ptr(xx), _ptr(y))
    return y[:m].copy()


def getri_batch(sizes, val_off, vec_off, values, nthreads: int = 0):
    """Batched GJE inverse on a packed copy; returns (Dinv, perm, info)."""
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    val_off = np.ascontiguousarray(val_off, dtype=np.int64)
    vec_off = np.ascontiguousarray(vec_off, dtype=np.int64)
    A = np.array(values, copy=True)
    s = _sfx(A.dtype)
    nb = sizes.shape[0]
    perm = np.zeros(max(int(vec_off[nb]), 1), dtype=np.int32)
    info = np.zeros(max(nb, 1), dtype=np.int32)
    getattr(lib(), f"bjo_getri_batch_{s}")(nb, _ptr(sizes), _ptr(val_off), _ptr(vec_off),
                                           _ptr(A), _ptr(perm), _ptr(info), int(nthreads))
    return A, perm[: int(vec_off[nb])], info[:nb]


def gemv_batch(sizes, val_off, vec_off, Dinv, x, nthreads: int = 0):
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    val_off = np.ascontiguousarray(val_off, dtype=np.int64)
    vec_off = np.ascontiguousarray(vec_off, dtype=np.int64)
    Dinv = np.ascontiguousarray(Dinv)
    s = _sfx(Dinv.dtype)
    x = np.ascontiguousarray(x, dtype=Dinv.dtype)
    nb = sizes.shape[0]
    y = np.zeros(max(int(vec_off[nb]), 1), dtype=Dinv.dtype)
    getattr(lib(), f"bjo_gemv_batch_{s}")(nb, _ptr(sizes), _ptr(val_off), _ptr(vec_off),
                                          _ptr(Dinv), _ptr(x), _ptr(y), int(nthreads))
    return y[: int(vec_off[nb])]


def spmv(row_ptr, col_idx, values, x, col_offset: int = 0):
    """y = A x with the fixed summation order R27 (fp64)."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    values = np.ascontiguousarray(values, dtype=np.float64)
    x = np.ascontiguousarray(x, dtype=np.float64)
    n = row_ptr.shape[0] - 1
    y = np.zeros(max(n, 1))
    lib().bjo_spmv_d(n, _ptr(row_ptr), _ptr(col_idx), _ptr(values), int(col_offset), _ptr(x), _ptr(y))
    return y[:n]


def dot(x, y) -> float:
    """dot product with the fixed chunked order R28 (fp64)."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.ascontiguousarray(y, dtype=np.float64)
    return float(lib().bjo_dot_d(x.shape[0], _ptr(x), _ptr(y)))


def fma_vec(a, x, y):
    """out = fma(a, x, y) elementwise (C99 fma, single rounding)."""
    a = np.ascontiguousarray(a, dtype=np.float64)
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.ascontiguousarray(y, dtype=np.float64)
    out = np.empty(max(x.shape[0], 1))
    lib().bjo_fma_vec(x.shape[0], _ptr(a), _ptr(x), _ptr(y), _ptr(out))
    return out[: x.shape[0]]


def dot_sharded(x, y, bounds) -> float:
    """R30: per-shard R28 dots summed in shard order from +0."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.ascontiguousarray(y, dtype=np.float64)
    b = np.ascontiguousarray(bounds, dtype=np.int64)
    return float(lib().bjo_dot_sharded_d(x.shape[0], _ptr(x), _ptr(y), b.shape[0] - 1, _ptr(b)))


def bicgstab(row_ptr, col_idx, values, block_ptr, b, tol: float = 1e-6, maxit: int = 10000,
             col_offset: int = 0, bounds=None):
    """Block-Jacobi (LU) preconditioned BiCGSTAB, R27-R29 (section IV.D,
    P:852-856); with `bounds` (row shards, int64[G+1]) the dots follow R30.
    Returns (x, iterations, relative residual, LU, perm, info)."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    values = np.ascontiguousarray(values, dtype=np.float64)
    D, sizes, vec, val = extract(row_ptr, col_idx, values, block_ptr, col_offset)
    LU, perm, info = getrf_batch(sizes, val, vec, D)
    n = row_ptr.shape[0] - 1
    b = np.ascontiguousarray(b, dtype=np.float64)
    x = np.zeros(max(n, 1))
    res = ctypes.c_double(0.0)
    if bounds is None:
        it = lib().bjo_bicgstab_d(n, _ptr(row_ptr), _ptr(col_idx), _ptr(values), int(col_offset), len(sizes),
                                  _ptr(sizes), _ptr(val), _ptr(vec), _ptr(LU), _ptr(perm), _ptr(b), float(tol),
                                  int(maxit), _ptr(x), ctypes.byref(res))
    else:
        bd = np.ascontiguousarray(bounds, dtype=np.int64)
        it = lib().bjo_bicgstab_sharded_d(n, _ptr(row_ptr), _ptr(col_idx), _ptr(values), int(col_offset),
                                          len(sizes), _ptr(sizes), _ptr(val), _ptr(vec), _ptr(LU), _ptr(perm),
                                          _ptr(b), float(tol), int(maxit), bd.shape[0] - 1, _ptr(bd), _ptr(x),
                                          ctypes.byref(res))
    return x[:n], int(it), float(res.value), LU, perm, info


def extract(row_ptr, col_idx, values, block_ptr, col_offset: int = 0):
    """Dense diagonal blocks of a CSR matrix (section III.C).

    Returns (blocks packed at val_off, sizes, vec_off, val_off).
    """
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    values = np.ascontiguousarray(values)
    block_ptr = np.ascontiguousarray(block_ptr, dtype=np.int32)
    es = values.dtype.itemsize
    nb = block_ptr.shape[0] - 1
    sizes = np.diff(block_ptr).astype(np.int32)
    vec_off, val_off = layout(sizes, es)
    out = np.full(max(int(val_off[nb]), 1), np.nan, dtype=values.dtype)  # holes stay NaN
    rc = lib().bjo_extract(row_ptr.shape[0] - 1, _ptr(row_ptr), _ptr(col_idx), _ptr(values),
                           es, int(col_offset), nb, _ptr(block_ptr), _ptr(val_off), _ptr(out))
    if rc != 0:
        raise ValueError("duplicate (row, col) entry inside a diagonal block")
    return out[: int(val_off[nb])], sizes, vec_off, val_off


def partition(sizes, G: int):
    """Contiguous cost-balanced shard boundaries, int64[G+1] (row a6)."""
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    bounds = np.zeros(G + 1, dtype=np.int64)
    lib().bjo_partition(sizes.shape[0], _ptr(sizes), int(G), _ptr(bounds))
    return bounds
