"""Small invocation of every library kernel (C1-sized) for compute-sanitizer
(scripts/sanitize.sh): layout, plan, GETRF (all order classes incl. the safe
path), GETRS, fused GESV, GETRI + GEMV, extraction (incl. a hub block),
block-Jacobi setup (fused) / apply, supervariable blocking."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bj_synth as S  # noqa: E402
from paper_conf_icpp_anztdfq17_b200 import bj  # noqa: E402

torch.cuda.set_device(0)
for dtype in (torch.float64, torch.float32):
    sizes_np = np.concatenate([S.block_sizes(300, 1, 32), np.array([32, 24, 0, 33], np.int32)])
    sizes = torch.from_numpy(sizes_np).cuda()
    batch = bj.new_batch(sizes, dtype)
    bj.synth_blocks(batch)
    # a block that takes the safe path (an Inf entry) and an integer block with ties
    batch.values[int(batch.val_off[300].item())] = float("inf")
    rhs = bj.synth_rhs(batch)
    nvec = int(batch.vec_off[-1].item())
    piv = torch.empty(nvec, dtype=torch.int32, device="cuda")
    info = torch.empty(len(sizes_np), dtype=torch.int32, device="cuda")
    x = torch.empty_like(rhs)
    pristine = batch.values.clone()
    plan = bj.Plan(sizes)
    bj.getrf(batch, piv, info, plan=plan)
    bj.getrs(batch, piv, rhs, x, plan=plan)
    batch.values.copy_(pristine)
    bj.gesv(batch, piv, info, rhs, x, plan=plan)
    batch.values.copy_(pristine)
    bj.getri(batch, piv, info, plan=plan)
    bj.gemv(batch, rhs, x, plan=plan)
    plan.close()
    g = S.FemGrid(9, 8, 7)
    A = bj.synth_fem(9, 8, 7, 0, g.n, dtype=dtype)
    for b in (5, 24):
        bp = torch.from_numpy(S.uniform_block_ptr(g.n, b)).cuda()
        sz, vec, val = bj.layout_from_block_ptr(bp, dtype)
        out = bj.Batch(sz, vec, val, torch.empty(int(val[-1].item()), dtype=dtype, device="cuda"))
        bj.extract(A, bp, out)
        p2 = torch.empty(g.n, dtype=torch.int32, device="cuda")
        i2 = torch.empty(len(bp) - 1, dtype=torch.int32, device="cuda")
        h = bj.Handle()
        h.setup(A, bp, out, p2, i2)
        xv = torch.rand(g.n, dtype=dtype, device="cuda")
        yv = torch.empty_like(xv)
        h.apply(xv, yv)
        h.setup_inverse(A, bp, out, p2, i2)
        h.apply(xv, yv)
        h.close()
    bj.supervariable_blocking(A, 24)
torch.cuda.synchronize()
print("sanitize driver ok")
