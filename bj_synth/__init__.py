"""Seeded synthetic inputs for the block-Jacobi hot path (host side, numpy).

This module holds NO arithmetic of the method.  It only draws random numbers
and builds input structures; both the oracle (tests, cpu baseline) and the
CUDA path consume what it produces.  The device-side generator in
``paper_conf_icpp_anztdfq17_b200/csrc/synth.cu`` implements the *same*
counter-based generator (splitmix64 keyed by (seed, global index)); the two
are checked bit for bit against each other in ``tests/test_gpu_parity.py``
(test_device_generator_matches_host_generator) and ``tests/test_gpu_extract.py``.
Because every value depends only on (seed, global index), any shard or
subset of a workload regenerates identically.

Recipe:
  * block sizes  m_i ~ U{lo..hi}                          seed 1
  * block values A_i(r,c) ~ U[-1, 1) (53-bit grid)         seed 2, key gid*1024 + c*32 + r
  * right-hand sides b_i(r) ~ U[-1, 1)                     seed 3, key gid*32 + r
  * integer stress blocks A_i(r,c) ~ U{-3..3}              seed 7 (many exact ties)
  * FEM-like CSR: 27-point stencil x 3 dofs/node on an nx*ny*nz grid
    (x fastest, dofs interleaved); off-diagonals -(1..2^20)*2^-20 (U(-1,0)),
    diagonal 1 + sum|off| (exact in binary64 by construction);
    0.1% of rows (seed 4) get Pareto(alpha=1.5, x_min=100, cap 100000)
    extra entries at columns outside the stencil band (seed 5), values
    (k-K)*2^-30 ~ U(-1e-3, 1e-3) (seed 6), appended after the sorted stencil
    entries (so those rows are unsorted).
"""
from __future__ import annotations

import numpy as np

M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
GOLDEN = np.uint64(0x9E3779B97F4A7C15)
SEED_SALT = np.uint64(0x632BE59BD9B4E019)
C1 = np.uint64(0xBF58476D1CE4E5B9)
C2 = np.uint64(0x94D049BB133111EB)

SEED_SIZES, SEED_VALUES, SEED_RHS, SEED_SKEW, SEED_HUBCOL, SEED_HUBVAL, SEED_INT = 1, 2, 3, 4, 5, 6, 7
BLOCK_KEY_STRIDE = 1024   # max m*m
VEC_KEY_STRIDE = 32       # max m
HUB_THRESHOLD = 9007199254740      # floor(2^53 / 1000): P(hub) = 1e-3
HUB_CAP = 100000
HUB_VAL_K = 1073741                # floor(1e-3 * 2^30)
HUB_PRIMES = (1000003, 1000033, 1000037, 1000039, 1000081)


def _u64(x) -> np.ndarray:
    return np.asarray(x, dtype=np.uint64)


def mix64(z) -> np.ndarray:
    """splitmix64 finaliser (bijective on uint64)."""
    z = _u64(z)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * C1
        z = (z ^ (z >> np.uint64(27))) * C2
    return z ^ (z >> np.uint64(31))


def seed_key(seed: int) -> np.uint64:
    with np.errstate(over="ignore"):
        return mix64(_u64([seed]) * GOLDEN + SEED_SALT)[0]


def hash64(seed: int, idx) -> np.ndarray:
    """i-th splitmix64 output of the stream keyed by ``seed``."""
    idx = _u64(idx)
    with np.errstate(over="ignore"):
        return mix64(seed_key(seed) + (idx + np.uint64(1)) * GOLDEN)


def uniform_pm1(seed: int, idx) -> np.ndarray:
    """U[-1, 1) on the 2^-52 grid: 2*((h >> 11) * 2^-53) - 1 (exact)."""
    h = hash64(seed, idx)
    u = (h >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
    return 2.0 * u - 1.0


def uniform_int(seed: int, idx, lo: int, hi: int) -> np.ndarray:
    """U{lo..hi} via the multiply-shift map of the high 32 bits."""
    h = hash64(seed, idx) >> np.uint64(32)
    span = np.uint64(hi - lo + 1)
    return (lo + ((h * span) >> np.uint64(32)).astype(np.int64)).astype(np.int64)


# --------------------------------------------------------------------------
# dense block batches (configs C1-C3)
# --------------------------------------------------------------------------
def block_sizes(nb: int, lo: int, hi: int, first: int = 0, seed: int = SEED_SIZES) -> np.ndarray:
    """Sizes of global blocks first..first+nb-1, uniform in lo..hi."""
    return uniform_int(seed, np.arange(first, first + nb, dtype=np.uint64), lo, hi).astype(np.int32)


def packed_offsets(sizes: np.ndarray, elem_size: int):
    """Input-layout helper (pure bookkeeping): vec_off, val_off as the
    library's layout contract defines them (16-B aligned block starts)."""
    sizes = np.asarray(sizes, dtype=np.int64)
    q = 16 // elem_size
    sq = ((sizes * sizes + q - 1) // q) * q
    vec = np.zeros(len(sizes) + 1, dtype=np.int64)
    val = np.zeros(len(sizes) + 1, dtype=np.int64)
    np.cumsum(sizes, out=vec[1:])
    np.cumsum(sq, out=val[1:])
    return vec, val


def block_values(sizes: np.ndarray, val_off: np.ndarray, first: int = 0, dtype=np.float64,
                 kind: str = "uniform", ids=None) -> np.ndarray:
    """Packed column-major blocks.  Element (r, c) of global block g has key
    g*1024 + c*32 + r.  ``kind``: "uniform" U[-1,1) (seed 2) or "int" U{-3..3}
    (seed 7).  fp32 values are the fp64 draws rounded to nearest.  Block i has
    global id first+i, or ids[i] when ``ids`` is given."""
    sizes = np.asarray(sizes, dtype=np.int64)
    nb = len(sizes)
    out = np.zeros(int(val_off[nb]), dtype=dtype)
    if nb == 0:
        return out
    cnt = sizes * sizes
    tot = int(cnt.sum())
    blk = np.repeat(np.arange(nb, dtype=np.int64), cnt)
    start = np.repeat(np.cumsum(cnt) - cnt, cnt)
    e = np.arange(tot, dtype=np.int64) - start          # element index inside block
    m = sizes[blk]
    r = e % np.maximum(m, 1)
    c = e // np.maximum(m, 1)
    gid = (blk + first) if ids is None else np.asarray(ids, dtype=np.int64)[blk]
    key = gid.astype(np.uint64) * np.uint64(BLOCK_KEY_STRIDE) + \
        (c * VEC_KEY_STRIDE + r).astype(np.uint64)
    if kind == "uniform":
        v = uniform_pm1(SEED_VALUES, key)
    elif kind == "int":
        v = uniform_int(SEED_INT, key, -3, 3).astype(np.float64)
    else:
        raise ValueError(kind)
    out[(np.asarray(val_off[:nb], dtype=np.int64)[blk] + e)] = v.astype(dtype)
    return out


def rhs_values(sizes: np.ndarray, first: int = 0, dtype=np.float64, ids=None) -> np.ndarray:
    """Packed right-hand sides; element r of global block g has key g*32 + r."""
    sizes = np.asarray(sizes, dtype=np.int64)
    nb = len(sizes)
    blk = np.repeat(np.arange(nb, dtype=np.int64), sizes)
    start = np.repeat(np.cumsum(sizes) - sizes, sizes)
    r = np.arange(int(sizes.sum()), dtype=np.int64) - start
    gid = (blk + first) if ids is None else np.asarray(ids, dtype=np.int64)[blk]
    key = gid.astype(np.uint64) * np.uint64(VEC_KEY_STRIDE) + r.astype(np.uint64)
    return uniform_pm1(SEED_RHS, key).astype(dtype)


# --------------------------------------------------------------------------
# FEM-like CSR (configs C4, C5)
# --------------------------------------------------------------------------
def icbrt(v: int) -> int:
    """floor(cbrt(v)) for a non-negative Python int (exact)."""
    if v <= 0:
        return 0
    x = int(round(v ** (1.0 / 3.0)))
    while x * x * x > v:
        x -= 1
    while (x + 1) ** 3 <= v:
        x += 1
    return x


class FemGrid:
    """27-point x 3-dof FEM-like sparsity on an nx*ny*nz node grid."""

    def __init__(self, nx: int, ny: int, nz: int, skew: bool = True):
        self.nx, self.ny, self.nz = nx, ny, nz
        self.n = 3 * nx * ny * nz
        self.band = 3 * (1 + nx + nx * ny) + 2
        self.W = self.n - (2 * self.band + 1)
        self.skew = skew and self.W > 0
        self.P = 1
        if self.W > 0:
            for p in HUB_PRIMES:
                if self.W % p != 0:
                    self.P = p
                    break

    # ---- per-row pieces (independent of any other row) ----
    def stencil_cols(self, r: int) -> np.ndarray:
        node, _ = divmod(r, 3)
        nx, ny, nz = self.nx, self.ny, self.nz
        x = node % nx
        y = (node // nx) % ny
        z = node // (nx * ny)
        cols = []
        for dz in (-1, 0, 1):
            zz = z + dz
            if zz < 0 or zz >= nz:
                continue
            for dy in (-1, 0, 1):
                yy = y + dy
                if yy < 0 or yy >= ny:
                    continue
                for dx in (-1, 0, 1):
                    xx = x + dx
                    if xx < 0 or xx >= nx:
                        continue
                    nd = xx + nx * (yy + ny * zz)
                    cols.extend((3 * nd, 3 * nd + 1, 3 * nd + 2))
        return np.asarray(cols, dtype=np.int64)

    def n_extra(self, r: int) -> int:
        if not self.skew:
            return 0
        h = int(hash64(SEED_SKEW, [2 * r])[0])
        if (h >> 11) >= HUB_THRESHOLD:
            return 0
        uu = 1 + (int(hash64(SEED_SKEW, [2 * r + 1])[0]) >> 44)
        v = (10 ** 6 * (1 << 40)) // (uu * uu)
        return min(icbrt(v), HUB_CAP, self.W)

    def extra_cols(self, r: int, k: int) -> np.ndarray:
        if k == 0:
            return np.zeros(0, dtype=np.int64)
        h0 = int(hash64(SEED_HUBCOL, [r])[0]) % self.W
        j = np.arange(k, dtype=np.int64)
        t = (h0 + j * self.P) % self.W
        return (r + self.band + 1 + t) % self.n

    def row(self, r: int, dtype=np.float64):
        """(cols int32, values) of global row r, in storage order."""
        sc = self.stencil_cols(r)
        off = sc != r
        key = np.uint64(r) * np.uint64(1 << 32) + sc.astype(np.uint64)
        h = hash64(SEED_VALUES, key)
        v = -((h >> np.uint64(44)).astype(np.float64) + 1.0) * (2.0 ** -20)
        k = self.n_extra(r)
        ec = self.extra_cols(r, k)
        if k:
            ekey = np.uint64(r) * np.uint64(1 << 32) + ec.astype(np.uint64)
            eh = hash64(SEED_HUBVAL, ekey) >> np.uint64(40)
            ev = ((eh % np.uint64(2 * HUB_VAL_K + 1)).astype(np.int64) - HUB_VAL_K).astype(np.float64) \
                * (2.0 ** -30)
        else:
            ev = np.zeros(0)
        diag = 1.0 + np.abs(v[off]).sum() + np.abs(ev).sum()      # exact (all on the 2^-30 grid)
        v = np.where(off, v, diag)
        cols = np.concatenate([sc, ec]).astype(np.int32)
        vals = np.concatenate([v, ev]).astype(dtype)
        return cols, vals

    def row_nnz(self, r: int) -> int:
        return len(self.stencil_cols(r)) + self.n_extra(r)

    def csr(self, r0: int = 0, r1: int | None = None, dtype=np.float64):
        """CSR of rows [r0, r1) (local rows, global columns)."""
        r1 = self.n if r1 is None else r1
        cols, vals, rp = [], [], [0]
        for r in range(r0, r1):
            c, v = self.row(r, dtype)
            cols.append(c)
            vals.append(v)
            rp.append(rp[-1] + len(c))
        row_ptr = np.asarray(rp, dtype=np.int64)
        col = np.concatenate(cols) if cols else np.zeros(0, np.int32)
        val = np.concatenate(vals) if vals else np.zeros(0, dtype)
        return row_ptr, col.astype(np.int32), val.astype(dtype)


def uniform_block_ptr(n: int, b: int, r0: int = 0) -> np.ndarray:
    """Blocks of b consecutive rows over rows [0, n) (last block n mod b)."""
    edges = list(range(0, n, b)) + [n]
    return np.asarray(edges, dtype=np.int32)


# --------------------------------------------------------------------------
# C implementation of the same generators (bj_synth/fastgen.c) for full-size
# inputs; checked bit for bit against the numpy functions above
# (tests/test_synth.py).
# --------------------------------------------------------------------------
import ctypes as _ct
import os as _os
import subprocess as _sp

_HERE = _os.path.dirname(_os.path.abspath(__file__))
_FAST_SRC = _os.path.join(_HERE, "fastgen.c")
_FAST_LIB = _os.path.join(_HERE, "libbjs_fast.so")
_fast = None


def build_fast(force: bool = False) -> str:
    if force or not _os.path.exists(_FAST_LIB) or _os.path.getmtime(_FAST_LIB) < _os.path.getmtime(_FAST_SRC):
        tmp = _FAST_LIB + ".tmp%d" % _os.getpid()
        _sp.check_call(["gcc", "-std=gnu99", "-O2", "-fopenmp", "-fPIC", "-shared", "-Wall", _FAST_SRC,
                        "-o", tmp, "-lm"])
        _os.replace(tmp, _FAST_LIB)
    return _FAST_LIB


def _fastlib():
    global _fast
    if _fast is None:
        build_fast()
        L = _ct.CDLL(_FAST_LIB)
        P, I64, I32 = _ct.c_void_p, _ct.c_int64, _ct.c_int
        for s in ("d", "s"):
            getattr(L, f"bjs_block_values_{s}").argtypes = [I64, I64, I32, P, P, P, P]
            getattr(L, f"bjs_rhs_values_{s}").argtypes = [I64, I64, P, P, P, P]
            getattr(L, f"bjs_fem_fill_{s}").argtypes = [I32, I32, I32, I32, I64, I64, P, P, P]
            getattr(L, f"bjs_fem_fill_{s}").restype = I32
        L.bjs_fem_row_ptr.argtypes = [I32, I32, I32, I32, I64, I64, P]
        L.bjs_fem_row_ptr.restype = I32
        _fast = L
    return _fast


def _pp(a):
    return None if a is None else a.ctypes.data_as(_ct.c_void_p)


def _sfx(dtype):
    return "d" if np.dtype(dtype) == np.float64 else "s"


def block_values_fast(sizes, val_off, first: int = 0, dtype=np.float64, kind: str = "uniform", ids=None):
    """Same output as block_values() (C, OpenMP)."""
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    val_off = np.ascontiguousarray(val_off, dtype=np.int64)
    nb = len(sizes)
    out = np.empty(int(val_off[nb]), dtype=dtype)
    idv = None if ids is None else np.ascontiguousarray(ids, dtype=np.int64)
    getattr(_fastlib(), f"bjs_block_values_{_sfx(dtype)}")(nb, first, 0 if kind == "uniform" else 1, _pp(sizes),
                                                          _pp(val_off), _pp(idv), _pp(out))
    return out


def rhs_values_fast(sizes, first: int = 0, dtype=np.float64, ids=None):
    """Same output as rhs_values() (C, OpenMP)."""
    sizes = np.ascontiguousarray(sizes, dtype=np.int32)
    nb = len(sizes)
    vec = np.zeros(nb + 1, dtype=np.int64)
    np.cumsum(sizes, out=vec[1:])
    out = np.empty(int(vec[nb]), dtype=dtype)
    idv = None if ids is None else np.ascontiguousarray(ids, dtype=np.int64)
    getattr(_fastlib(), f"bjs_rhs_values_{_sfx(dtype)}")(nb, first, _pp(sizes), _pp(vec), _pp(idv), _pp(out))
    return out


def fem_csr_fast(nx: int, ny: int, nz: int, r0: int = 0, r1: int | None = None, dtype=np.float64,
                 skew: bool = True):
    """Same output as FemGrid(nx, ny, nz, skew).csr(r0, r1, dtype) (C, OpenMP)."""
    n = 3 * nx * ny * nz
    r1 = n if r1 is None else r1
    L = _fastlib()
    rp = np.empty(r1 - r0 + 1, dtype=np.int64)
    if L.bjs_fem_row_ptr(nx, ny, nz, int(skew), r0, r1, _pp(rp)) != 0:
        raise ValueError("bad FEM row range")
    nnz = int(rp[-1])
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=dtype)
    if getattr(L, f"bjs_fem_fill_{_sfx(dtype)}")(nx, ny, nz, int(skew), r0, r1, _pp(rp), _pp(col), _pp(val)) != 0:
        raise ValueError("bad FEM row range")
    return rp, col, val
