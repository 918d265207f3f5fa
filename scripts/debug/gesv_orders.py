"""Debug: bj_gesv_vbatched per order with a sync after each call."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import bj_synth as S
from paper_conf_icpp_anztdfq17_b200 import bj
dt = torch.float64 if len(sys.argv) < 2 else getattr(torch, sys.argv[1])
for m in list(range(17, 33)) + list(range(1, 17)):
    sizes = torch.full((37,), m, dtype=torch.int32, device="cuda")
    batch = bj.new_batch(sizes, dt)
    bj.synth_blocks(batch)
    rhs = bj.synth_rhs(batch)
    nvec = int(batch.vec_off[-1].item())
    piv = torch.empty(nvec, dtype=torch.int32, device="cuda")
    info = torch.empty(37, dtype=torch.int32, device="cuda")
    x = torch.empty_like(rhs)
    try:
        bj.gesv(batch, piv, info, rhs, x)
        torch.cuda.synchronize()
        print("m", m, "ok", flush=True)
    except Exception as e:
        print("m", m, "FAIL", e, flush=True)
        break
