"""Multi-GPU plumbing for the batched hot path (hot-path row a6).

The blocks are independent ("embarrassingly parallel", PAPER.md P:19-20,
P:83-85), so ranks own contiguous, cost-balanced block ranges (bj_partition,
reading R19) and never exchange data on the hot path; torch.distributed is used
only for a barrier, the max-over-ranks timing reduction and optional gathers.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import bj


def shard(sizes: np.ndarray, world: int, rank: int) -> tuple[int, int]:
    """[first, last) block range of `rank` (same answer on every rank)."""
    b = bj.partition(np.asarray(sizes, dtype=np.int32), world)
    return int(b[rank]), int(b[rank + 1])


def max_over_ranks(value: float, device=None) -> float:
    """Max of a scalar over all ranks (identity without a process group)."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_shards(local: torch.Tensor, device=None) -> torch.Tensor:
    """Concatenate variable-length 1-D shards from all ranks in rank order."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return local
    world = dist.get_world_size()
    n = torch.tensor([local.numel()], dtype=torch.int64, device=device)
    ns = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(ns, n)
    mx = int(max(int(x.item()) for x in ns))
    buf = torch.zeros(mx, dtype=local.dtype, device=device)
    buf[: local.numel()] = local
    outs = [torch.zeros_like(buf) for _ in range(world)]
    dist.all_gather(outs, buf)
    return torch.cat([o[: int(k.item())] for o, k in zip(outs, ns)])
