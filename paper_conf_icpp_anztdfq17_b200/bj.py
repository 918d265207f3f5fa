"""Thin Python binding of the C ABI in include/bj.h (ctypes).

Argument marshalling only: every step of the hot path runs in libbj.so's
CUDA kernels.  PyTorch supplies device memory (``tensor.data_ptr()``) and the
stream (``torch.cuda.current_stream().cuda_stream``).  There is no CPU
fallback: if libbj.so is missing or a call fails, an exception is raised.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libbj.so")

BJ_F32, BJ_F64 = 0, 1
_STATUS = {0: "BJ_OK", -1: "BJ_ERR_ARG", -2: "BJ_ERR_BLOCK_SIZE", -3: "BJ_ERR_ALIGN", -4: "BJ_ERR_CUDA",
           -5: "BJ_ERR_NOMEM", -6: "BJ_ERR_STATE", -7: "BJ_ERR_COMM"}

# every symbol include/bj.h and include/bj_synth.h declare
EXPORTS = (
    "bj_status_string", "bj_version", "bj_layout", "bj_layout_from_block_ptr", "bj_plan_create",
    "bj_plan_destroy", "bj_extract", "bj_getrf_vbatched", "bj_getrs_vbatched", "bj_gesv_vbatched",
    "bj_getri_vbatched", "bj_gemv_vbatched", "bj_setup_inverse", "bj_selftest_div",
    "bj_create", "bj_setup",
    "bj_apply", "bj_destroy", "bj_partition", "bj_workspace_create", "bj_workspace_destroy", "bj_gesv_host",
    "bj_launch_count", "bj_launch_count_reset", "bj_supervariable_blocking",
    "bj_spmv", "bj_dot", "bj_bicgstab", "bj_halo_plan",
    "bj_synth_sizes", "bj_synth_blocks", "bj_synth_rhs", "bj_synth_fem_row_ptr", "bj_synth_fem_fill",
)


class BJError(RuntimeError):
    pass


class CSR(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("nnz", ctypes.c_int64), ("col_offset", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("values", ctypes.c_void_p),
                ("dtype", ctypes.c_int)]


HALO_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p)
GATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p)


class CommC(ctypes.Structure):
    _fields_ = [("ctx", ctypes.c_void_p), ("nranks", ctypes.c_int), ("rank", ctypes.c_int),
                ("nhalo", ctypes.c_int64), ("nsend", ctypes.c_int64), ("send_idx", ctypes.c_void_p),
                ("send_buf", ctypes.c_void_p), ("recv_buf", ctypes.c_void_p), ("gather_buf", ctypes.c_void_p),
                ("halo_exchange", HALO_FN), ("allgather", GATHER_FN), ("halo_wait", HALO_FN)]


class BatchC(ctypes.Structure):
    _fields_ = [("nblocks", ctypes.c_int64), ("sizes", ctypes.c_void_p), ("vec_off", ctypes.c_void_p),
                ("val_off", ctypes.c_void_p), ("values", ctypes.c_void_p), ("dtype", ctypes.c_int)]


_lib = None


def lib() -> ctypes.CDLL:
    """Load libbj.so (fails loudly if it has not been built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise BJError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                          "(python -m paper_conf_icpp_anztdfq17_b200.build); there is no fallback path")
        L = ctypes.CDLL(LIB_PATH)
        P, I64, I32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        sig = {
            "bj_status_string": ([I32], ctypes.c_char_p),
            "bj_version": ([], ctypes.c_char_p),
            "bj_layout": ([I64, P, I32, P, P, P], I32),
            "bj_layout_from_block_ptr": ([I64, P, I32, P, P, P, P], I32),
            "bj_plan_create": ([P, I64, P, P], I32),
            "bj_plan_destroy": ([P], I32),
            "bj_extract": ([P, P, P, P], I32),
            "bj_getrf_vbatched": ([P, P, P, P, P], I32),
            "bj_getrs_vbatched": ([P, P, P, P, P, P], I32),
            "bj_gesv_vbatched": ([P, P, P, P, P, P, P], I32),
            "bj_getri_vbatched": ([P, P, P, P, P], I32),
            "bj_gemv_vbatched": ([P, P, P, P, P], I32),
            "bj_setup_inverse": ([P, P, P, P, P, P, P], I32),
            "bj_selftest_div": ([I32, I64, ctypes.c_uint64, P, P, I64], I32),
            "bj_create": ([P], I32),
            "bj_setup": ([P, P, P, P, P, P, P], I32),
            "bj_apply": ([P, P, P, P], I32),
            "bj_destroy": ([P], I32),
            "bj_partition": ([I64, P, I32, P], I32),
            "bj_supervariable_blocking": ([P, I32, P, P, P], I32),
            "bj_workspace_create": ([P], I32),
            "bj_workspace_destroy": ([P], I32),
            "bj_gesv_host": ([P, I64, P, I64, P, I64, P, P, P, P, I32, P], I32),
            "bj_spmv": ([P, P, P, P], I32),
            "bj_dot": ([I64, P, P, P, P], I32),
            "bj_bicgstab": ([P, P, P, P, P, ctypes.c_double, I32, P, P, P], I32),
            "bj_halo_plan": ([I64, P, I64, I64, I32, P, P, P, P, P], I32),
            "bj_launch_count": ([], I64),
            "bj_launch_count_reset": ([], None),
            "bj_synth_sizes": ([I64, I64, I32, I32, ctypes.c_uint64, P, P], I32),
            "bj_synth_blocks": ([P, I64, I32, P], I32),
            "bj_synth_rhs": ([P, I64, P, P], I32),
            "bj_synth_fem_row_ptr": ([I32, I32, I32, I32, I64, I64, P, P], I32),
            "bj_synth_fem_fill": ([I32, I32, I32, I32, I64, I64, P, P, P, I32, P], I32),
        }
        for name, (args, res) in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _lib = L
    return _lib


def _check(st: int, what: str):
    if st != 0:
        raise BJError(f"{what}: {_STATUS.get(st, st)}")


def _stream(stream=None) -> ctypes.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _p(t: torch.Tensor | None):
    return ctypes.c_void_p(t.data_ptr()) if t is not None else None


def dtype_code(dt: torch.dtype) -> int:
    if dt == torch.float64:
        return BJ_F64
    if dt == torch.float32:
        return BJ_F32
    raise TypeError(f"unsupported dtype {dt}")


def version() -> str:
    return lib().bj_version().decode()


def launch_count() -> int:
    return int(lib().bj_launch_count())


def launch_count_reset():
    lib().bj_launch_count_reset()


# --------------------------------------------------------------------------
# batches
# --------------------------------------------------------------------------
@dataclass
class Batch:
    """Packed dense blocks (layout of include/bj.h).  All tensors on one CUDA
    device: sizes int32[nb], vec_off/val_off int64[nb+1], values fp32/fp64."""
    sizes: torch.Tensor
    vec_off: torch.Tensor
    val_off: torch.Tensor
    values: torch.Tensor

    @property
    def nblocks(self) -> int:
        return int(self.sizes.numel())

    def c(self) -> BatchC:
        return BatchC(self.nblocks, self.sizes.data_ptr(), self.vec_off.data_ptr(), self.val_off.data_ptr(),
                      self.values.data_ptr(), dtype_code(self.values.dtype))


def layout(sizes: torch.Tensor, dtype: torch.dtype, stream=None):
    """Hot-path row a1: (vec_off, val_off) int64[nb+1] on sizes' device."""
    nb = sizes.numel()
    vec = torch.empty(nb + 1, dtype=torch.int64, device=sizes.device)
    val = torch.empty(nb + 1, dtype=torch.int64, device=sizes.device)
    _check(lib().bj_layout(nb, _p(sizes), dtype_code(dtype), _p(vec), _p(val), _stream(stream)), "bj_layout")
    return vec, val


def layout_from_block_ptr(block_ptr: torch.Tensor, dtype: torch.dtype, stream=None):
    nb = block_ptr.numel() - 1
    sizes = torch.empty(max(nb, 0), dtype=torch.int32, device=block_ptr.device)
    vec = torch.empty(nb + 1, dtype=torch.int64, device=block_ptr.device)
    val = torch.empty(nb + 1, dtype=torch.int64, device=block_ptr.device)
    _check(lib().bj_layout_from_block_ptr(nb, _p(block_ptr), dtype_code(dtype), _p(sizes), _p(vec), _p(val),
                                          _stream(stream)), "bj_layout_from_block_ptr")
    return sizes, vec, val


def new_batch(sizes: torch.Tensor, dtype: torch.dtype, stream=None) -> Batch:
    """Allocate a batch for `sizes` (values uninitialised).  Syncs once to size
    the value buffer."""
    vec, val = layout(sizes, dtype, stream)
    total = int(val[-1].item()) if sizes.numel() else 0
    values = torch.empty(max(total, 1), dtype=dtype, device=sizes.device)
    return Batch(sizes, vec, val, values)


class Plan:
    """Size-bucket plan (bj_plan_create); reuse across calls on the same sizes."""

    def __init__(self, sizes: torch.Tensor, stream=None):
        self._h = ctypes.c_void_p()
        self.nblocks = sizes.numel()
        _check(lib().bj_plan_create(ctypes.byref(self._h), self.nblocks, _p(sizes), _stream(stream)),
               "bj_plan_create")

    @property
    def handle(self):
        return self._h

    def close(self):
        if self._h:
            lib().bj_plan_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def getrf(batch: Batch, pivots: torch.Tensor, info: torch.Tensor, plan: Plan | None = None, stream=None):
    """Hot-path row a3: in-place LU with implicit pivoting."""
    b = batch.c()
    _check(lib().bj_getrf_vbatched(ctypes.byref(b), _p(pivots), _p(info), plan.handle if plan else None,
                                   _stream(stream)), "bj_getrf_vbatched")


def getrs(batch: Batch, pivots: torch.Tensor, rhs: torch.Tensor, x: torch.Tensor, plan: Plan | None = None,
          stream=None):
    """Hot-path row a4: x = D^{-1} rhs per block (x may be rhs)."""
    b = batch.c()
    _check(lib().bj_getrs_vbatched(ctypes.byref(b), _p(pivots), _p(rhs), _p(x), plan.handle if plan else None,
                                   _stream(stream)), "bj_getrs_vbatched")


def gesv(batch: Batch, pivots: torch.Tensor, info: torch.Tensor, rhs: torch.Tensor, x: torch.Tensor,
         plan: Plan | None = None, stream=None):
    """Rows a3 + a4 fused: in-place LU with implicit pivoting and x = A^{-1} rhs
    per block, bit-identical to getrf() then getrs() (x may be rhs)."""
    b = batch.c()
    _check(lib().bj_gesv_vbatched(ctypes.byref(b), _p(pivots), _p(info), _p(rhs), _p(x),
                                  plan.handle if plan else None, _stream(stream)), "bj_gesv_vbatched")


def getri(batch: Batch, pivots: torch.Tensor, info: torch.Tensor, plan: Plan | None = None, stream=None):
    """NEXT(3): in-place block inverses by Gauss-Jordan elimination (R23-R25)."""
    b = batch.c()
    _check(lib().bj_getri_vbatched(ctypes.byref(b), _p(pivots), _p(info), plan.handle if plan else None,
                                   _stream(stream)), "bj_getri_vbatched")


def gemv(inv: Batch, x: torch.Tensor, y: torch.Tensor, plan: Plan | None = None, stream=None):
    """NEXT(3): y = Dinv x per block (R26); y may be x."""
    b = inv.c()
    _check(lib().bj_gemv_vbatched(ctypes.byref(b), _p(x), _p(y), plan.handle if plan else None, _stream(stream)),
           "bj_gemv_vbatched")


@dataclass
class Csr:
    row_ptr: torch.Tensor     # int64[nrows+1]
    col_idx: torch.Tensor     # int32[nnz]
    values: torch.Tensor      # fp32/fp64[nnz]
    col_offset: int = 0

    def c(self) -> CSR:
        return CSR(self.row_ptr.numel() - 1, self.col_idx.numel(), int(self.col_offset), self.row_ptr.data_ptr(),
                   self.col_idx.data_ptr(), self.values.data_ptr(), dtype_code(self.values.dtype))


def extract(A: Csr, block_ptr: torch.Tensor, out: Batch, stream=None):
    """Hot-path row a2: dense diagonal blocks of A into `out` (layout of
    layout_from_block_ptr(block_ptr))."""
    a = A.c()
    o = out.c()
    _check(lib().bj_extract(ctypes.byref(a), _p(block_ptr), ctypes.byref(o), _stream(stream)), "bj_extract")


class Handle:
    """Hot-path row a5: block-Jacobi preconditioner (setup = extract + getrf,
    apply = getrs)."""

    def __init__(self):
        self._h = ctypes.c_void_p()
        _check(lib().bj_create(ctypes.byref(self._h)), "bj_create")
        self._keep = None

    def setup(self, A: Csr, block_ptr: torch.Tensor, factors: Batch, pivots: torch.Tensor, info: torch.Tensor,
              stream=None):
        a = A.c()
        f = factors.c()
        _check(lib().bj_setup(self._h, ctypes.byref(a), _p(block_ptr), ctypes.byref(f), _p(pivots), _p(info),
                              _stream(stream)), "bj_setup")
        self._keep = (A, block_ptr, factors, pivots, info)

    def setup_inverse(self, A: Csr, block_ptr: torch.Tensor, inverses: Batch, pivots: torch.Tensor,
                      info: torch.Tensor, stream=None):
        """NEXT(3): setup = extract + explicit inverses (apply then = GEMV)."""
        a = A.c()
        f = inverses.c()
        _check(lib().bj_setup_inverse(self._h, ctypes.byref(a), _p(block_ptr), ctypes.byref(f), _p(pivots),
                                      _p(info), _stream(stream)), "bj_setup_inverse")
        self._keep = (A, block_ptr, inverses, pivots, info)

    def apply(self, x: torch.Tensor, y: torch.Tensor, stream=None):
        _check(lib().bj_apply(self._h, _p(x), _p(y), _stream(stream)), "bj_apply")

    def close(self):
        if self._h:
            lib().bj_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def supervariable_blocking(A: Csr, max_block: int, stream=None) -> torch.Tensor:
    """NEXT(2): block_ptr (int32 device tensor [nb+1]) of supervariable
    blocking with upper bound `max_block` (R20-R22).  Synchronous."""
    n = A.row_ptr.numel() - 1
    bp = torch.empty(n + 1, dtype=torch.int32, device=A.row_ptr.device)
    nb = ctypes.c_int64(0)
    a = A.c()
    _check(lib().bj_supervariable_blocking(ctypes.byref(a), int(max_block), _p(bp), ctypes.byref(nb),
                                           _stream(stream)), "bj_supervariable_blocking")
    return bp[: nb.value + 1]


def partition(sizes: np.ndarray, G: int) -> np.ndarray:
    """Hot-path row a6 (host): contiguous cost-balanced shard boundaries."""
    s = np.ascontiguousarray(sizes, dtype=np.int32)
    out = np.zeros(G + 1, dtype=np.int64)
    _check(lib().bj_partition(s.shape[0], s.ctypes.data_as(ctypes.c_void_p), int(G),
                              out.ctypes.data_as(ctypes.c_void_p)), "bj_partition")
    return out


class Workspace:
    """Device workspace of bj_gesv_host (end-to-end call with host buffers)."""

    def __init__(self):
        self._h = ctypes.c_void_p()
        _check(lib().bj_workspace_create(ctypes.byref(self._h)), "bj_workspace_create")

    def gesv_host(self, sizes_h: torch.Tensor, blocks_h: torch.Tensor, b_h: torch.Tensor, x_h: torch.Tensor,
                  pivots_h: torch.Tensor | None = None, info_h: torch.Tensor | None = None, stream=None):
        _check(lib().bj_gesv_host(self._h, sizes_h.numel(), _p(sizes_h), blocks_h.numel(), _p(blocks_h),
                                  b_h.numel(), _p(b_h), _p(x_h), _p(pivots_h), _p(info_h),
                                  dtype_code(blocks_h.dtype), _stream(stream)), "bj_gesv_host")

    def close(self):
        if self._h:
            lib().bj_workspace_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# --------------------------------------------------------------------------
# device-side synthetic inputs (bj_synth.h)
# --------------------------------------------------------------------------
def synth_sizes(nb: int, lo: int, hi: int, first: int = 0, seed: int = 1, device="cuda", stream=None):
    s = torch.empty(max(nb, 1), dtype=torch.int32, device=device)[:nb]
    _check(lib().bj_synth_sizes(nb, first, lo, hi, seed, _p(s), _stream(stream)), "bj_synth_sizes")
    return s


def synth_blocks(batch: Batch, first: int = 0, kind: int = 0, stream=None):
    b = batch.c()
    _check(lib().bj_synth_blocks(ctypes.byref(b), first, kind, _stream(stream)), "bj_synth_blocks")


def synth_rhs(batch: Batch, first: int = 0, stream=None) -> torch.Tensor:
    n = int(batch.vec_off[-1].item()) if batch.nblocks else 0
    out = torch.empty(max(n, 1), dtype=batch.values.dtype, device=batch.values.device)
    b = batch.c()
    _check(lib().bj_synth_rhs(ctypes.byref(b), first, _p(out), _stream(stream)), "bj_synth_rhs")
    return out


def synth_fem(nx: int, ny: int, nz: int, r0: int, r1: int, dtype=torch.float64, skew: bool = True,
              device="cuda", stream=None) -> Csr:
    """FEM-like CSR rows [r0, r1) (local rows, global columns; col_offset=r0)."""
    n = r1 - r0
    rp = torch.empty(n + 1, dtype=torch.int64, device=device)
    _check(lib().bj_synth_fem_row_ptr(nx, ny, nz, int(skew), r0, r1, _p(rp), _stream(stream)),
           "bj_synth_fem_row_ptr")
    nnz = int(rp[-1].item())
    ci = torch.empty(max(nnz, 1), dtype=torch.int32, device=device)
    va = torch.empty(max(nnz, 1), dtype=dtype, device=device)
    _check(lib().bj_synth_fem_fill(nx, ny, nz, int(skew), r0, r1, _p(rp), _p(ci), _p(va), dtype_code(dtype),
                                   _stream(stream)), "bj_synth_fem_fill")
    return Csr(rp, ci[:nnz], va[:nnz], r0)


def selftest_div(dtype: torch.dtype, n: int, seed: int = 1, nsample: int = 0):
    """Test hook: device check of the split IEEE divisions (bj_selftest_div).
    Returns (counts[6], sample (nsample, 3) array of a, b, a/b)."""
    counts = np.zeros(6, dtype=np.uint64)
    npdt = np.float64 if dtype == torch.float64 else np.float32
    sample = np.zeros((max(nsample, 1), 3), dtype=npdt)
    _check(lib().bj_selftest_div(dtype_code(dtype), int(n), int(seed), counts.ctypes.data_as(ctypes.c_void_p),
                                 sample.ctypes.data_as(ctypes.c_void_p), int(nsample)), "bj_selftest_div")
    return counts, sample[:nsample]


# ---------------------------------------------------------------------------
# NEXT(4): block-Jacobi preconditioned BiCGSTAB (section IV.D, R27-R30)

def spmv(A: Csr, x: torch.Tensor, y: torch.Tensor, stream=None):
    """y = A x in the fixed order R27 (fp64)."""
    a = A.c()
    _check(lib().bj_spmv(ctypes.byref(a), _p(x), _p(y), _stream(stream)), "bj_spmv")


def dot(x: torch.Tensor, y: torch.Tensor, stream=None) -> torch.Tensor:
    """dot(x, y) in the fixed order R28 (fp64); returns a 0-d device tensor."""
    out = torch.empty((), dtype=torch.float64, device=x.device)
    _check(lib().bj_dot(x.numel(), _p(x), _p(y), _p(out), _stream(stream)), "bj_dot")
    return out


def halo_plan(col_idx_h: np.ndarray, lo: int, hi: int, row_bounds: np.ndarray):
    """Host halo plan (bj_halo_plan): (col_local int32[nnz], halo_cols
    int32[nhalo] ascending, recv_counts int64[G])."""
    ci = np.ascontiguousarray(col_idx_h, dtype=np.int32)
    rb = np.ascontiguousarray(row_bounds, dtype=np.int64)
    G = rb.shape[0] - 1
    cl = np.empty(max(ci.shape[0], 1), dtype=np.int32)
    hc = np.empty(max(ci.shape[0], 1), dtype=np.int32)
    nh = ctypes.c_int64(0)
    rc = np.zeros(G, dtype=np.int64)
    vp = ctypes.c_void_p
    _check(lib().bj_halo_plan(ci.shape[0], ci.ctypes.data_as(vp), int(lo), int(hi), G, rb.ctypes.data_as(vp),
                              cl.ctypes.data_as(vp), hc.ctypes.data_as(vp), ctypes.byref(nh),
                              rc.ctypes.data_as(vp)), "bj_halo_plan")
    return cl[: ci.shape[0]], hc[: nh.value].copy(), rc


class TorchComm:
    """bj_comm over torch.distributed (NCCL on GPUs, gloo on CPU): the halo
    exchange is one all_to_all_single, the dot combination one
    all_gather_into_tensor.  Built once from this rank's halo plan: the
    requested column ids are exchanged so every rank knows what to send."""

    def __init__(self, halo_cols: np.ndarray, recv_counts: np.ndarray, lo: int, device, group=None):
        import torch.distributed as dist
        self.dist, self.group = dist, group
        self.rank, self.nranks = dist.get_rank(group), dist.get_world_size(group)
        self.device = torch.device(device)
        rc = torch.as_tensor(np.asarray(recv_counts, dtype=np.int64), device=self.device)
        sc = torch.empty_like(rc)
        dist.all_to_all_single(sc, rc, group=group)                   # how many each peer wants from me
        self.recv_counts = [int(v) for v in rc.tolist()]
        self.send_counts = [int(v) for v in sc.tolist()]
        req = torch.as_tensor(np.asarray(halo_cols, dtype=np.int32), device=self.device)
        want = torch.empty(sum(self.send_counts), dtype=torch.int32, device=self.device)
        dist.all_to_all_single(want, req, output_split_sizes=self.send_counts,
                               input_split_sizes=self.recv_counts, group=group)
        self.send_idx = (want.long() - int(lo)).to(torch.int32)       # own rows to send, by peer
        self.send_buf = torch.zeros(max(want.numel(), 1), dtype=torch.float64, device=self.device)
        self.recv_buf = torch.zeros(max(req.numel(), 1), dtype=torch.float64, device=self.device)
        self.gather_buf = torch.zeros(self.nranks * 4, dtype=torch.float64, device=self.device)
        self.nsend, self.nhalo = want.numel(), req.numel()
        self._halo_cb = HALO_FN(self._halo)
        self._gather_cb = GATHER_FN(self._gather)
        self._wait_cb = HALO_FN(self._wait)

    def halo_exchange(self, async_op: bool = False):
        """send_buf -> recv_buf (grouped by owner rank, halo order).  With
        async_op the exchange is left in flight until halo_wait()."""
        self._work = self.dist.all_to_all_single(self.recv_buf[: self.nhalo], self.send_buf[: self.nsend],
                                                 output_split_sizes=self.recv_counts,
                                                 input_split_sizes=self.send_counts, group=self.group,
                                                 async_op=async_op)

    def halo_wait(self):
        """make the current stream wait for the exchange started by halo_exchange(async_op=True)."""
        w, self._work = getattr(self, "_work", None), None
        if w is not None:
            w.wait()

    def allgather(self, k: int):
        """every rank's row gather_buf[r*4 : r*4+4] to every rank."""
        mine = self.gather_buf[self.rank * 4: self.rank * 4 + 4].clone()
        self.dist.all_gather_into_tensor(self.gather_buf, mine, group=self.group)

    def _halo(self, ctx, stream):
        try:
            self.halo_exchange(async_op=True)     # the library computes the interior rows meanwhile
            return 0
        except Exception:
            return 1

    def _wait(self, ctx, stream):
        try:
            self.halo_wait()
            return 0
        except Exception:
            return 1

    def _gather(self, ctx, k, stream):
        try:
            self.allgather(int(k))
            return 0
        except Exception:
            return 1

    def c(self) -> CommC:
        return CommC(None, self.nranks, self.rank, self.nhalo, self.nsend, _p(self.send_idx), _p(self.send_buf),
                     _p(self.recv_buf), _p(self.gather_buf), self._halo_cb, self._gather_cb, self._wait_cb)


class LoopbackComm(TorchComm):
    """One-rank bj_comm without torch.distributed (exercises the library's
    communication path on a single GPU: empty halo, identity allgather)."""

    def __init__(self, device="cuda"):
        self.rank, self.nranks, self.device = 0, 1, torch.device(device)
        self.send_idx = torch.zeros(1, dtype=torch.int32, device=self.device)
        self.send_buf = torch.zeros(1, dtype=torch.float64, device=self.device)
        self.recv_buf = torch.zeros(1, dtype=torch.float64, device=self.device)
        self.gather_buf = torch.zeros(4, dtype=torch.float64, device=self.device)
        self.nsend = self.nhalo = 0
        self.calls = {"halo": 0, "allgather": 0, "wait": 0}
        self._halo_cb = HALO_FN(self._halo)
        self._gather_cb = GATHER_FN(self._gather)
        self._wait_cb = HALO_FN(self._wait)

    def halo_exchange(self, async_op: bool = False):
        self.calls["halo"] += 1

    def halo_wait(self):
        self.calls["wait"] += 1

    def allgather(self, k: int):
        self.calls["allgather"] += 1


def bicgstab(M: Handle, A: Csr, b: torch.Tensor, x: torch.Tensor, tol: float = 1e-6, maxit: int = 10000,
             comm: TorchComm | None = None, stream=None):
    """NEXT(4): block-Jacobi (M = a set-up Handle) preconditioned BiCGSTAB,
    R29 / R30.  x is overwritten.  Returns (iterations, relative residual);
    iterations = maxit + 1 when not converged.  Synchronous."""
    a = A.c()
    it = ctypes.c_int(0)
    res = ctypes.c_double(0.0)
    cc = comm.c() if comm is not None else None
    _check(lib().bj_bicgstab(M._h, ctypes.byref(a), ctypes.byref(cc) if cc is not None else None, _p(b), _p(x),
                             float(tol), int(maxit), ctypes.byref(it), ctypes.byref(res), _stream(stream)),
           "bj_bicgstab")
    return it.value, res.value
