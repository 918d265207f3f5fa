"""Shared helpers of the -m gpu parity tests (CUDA path through the C ABI vs
the CPU oracle on identical seeded inputs)."""
from __future__ import annotations

import numpy as np
import torch

import bj_synth as S
import oracle
from paper_conf_icpp_anztdfq17_b200 import bj

DEV = "cuda"
NP = {torch.float64: np.float64, torch.float32: np.float32}


def bits(a: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(a)
    return a.view(np.uint64 if a.dtype == np.float64 else np.uint32)


def device_batch(sizes_np: np.ndarray, dtype: torch.dtype, values_np: np.ndarray | None = None,
                 first: int = 0, kind: int = 0):
    """Batch on the device: values copied from numpy, or generated on the
    device with the same counter generator."""
    sizes = torch.from_numpy(np.ascontiguousarray(sizes_np, dtype=np.int32)).to(DEV)
    batch = bj.new_batch(sizes, dtype)
    if values_np is not None:
        batch.values[: values_np.size].copy_(torch.from_numpy(values_np))
    else:
        bj.synth_blocks(batch, first=first, kind=kind)
    return batch


def host_layout(sizes_np, dtype):
    return oracle.layout(np.asarray(sizes_np, np.int32), np.dtype(NP[dtype]).itemsize)


def compare_getrf(sizes_np, val_np, vec_np, A_host, LU_dev, piv_dev, info_dev, dtype, exact_bits=True):
    """Oracle GETRF on A_host vs the device results; returns oracle outputs."""
    LU_o, piv_o, info_o = oracle.getrf_batch(sizes_np, val_np, vec_np, A_host)
    assert np.array_equal(info_dev, info_o), "info mismatch"
    nb = len(sizes_np)
    for i in range(nb):
        m = int(sizes_np[i])
        if m < 1 or m > 32:
            continue                                        # invalid blocks are not touched
        assert np.array_equal(piv_dev[vec_np[i]: vec_np[i] + m], piv_o[vec_np[i]: vec_np[i] + m]), \
            f"pivot mismatch in block {i} (m={m})"
        a, b = int(val_np[i]), int(val_np[i]) + m * m
        if exact_bits:
            ok = np.array_equal(bits(LU_dev[a:b]), bits(LU_o[a:b]))
            if not ok and np.isnan(LU_o[a:b]).any():        # NaN payloads are not specified
                ok = np.array_equal(np.isnan(LU_dev[a:b]), np.isnan(LU_o[a:b])) and np.array_equal(
                    np.nan_to_num(LU_dev[a:b], nan=0.0), np.nan_to_num(LU_o[a:b], nan=0.0))
            assert ok, f"L\\U bits differ in block {i} (m={m})"
    return LU_o, piv_o, info_o


def backward_error(sizes_np, val_np, vec_np, A_host, b_host, x):
    """max over blocks of ||A x - b||_inf / (||A||_inf ||x||_inf), in fp64 (R13)."""
    worst = 0.0
    for i in range(len(sizes_np)):
        m = int(sizes_np[i])
        if m < 1 or m > 32:
            continue
        A = A_host[val_np[i]: val_np[i] + m * m].astype(np.float64).reshape(m, m, order="F")
        xi = x[vec_np[i]: vec_np[i] + m].astype(np.float64)
        bi = b_host[vec_np[i]: vec_np[i] + m].astype(np.float64)
        den = np.abs(A).sum(1).max() * np.abs(xi).max()
        if den == 0:
            continue
        worst = max(worst, np.abs(A @ xi - bi).max() / den)
    return worst
