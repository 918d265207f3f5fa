import torch, time, sys
sys.path.insert(0, '.')
from paper_conf_icpp_anztdfq17_b200 import bj
dt = torch.float64
nx, ny, nz = 174, 174, 22
n = 3 * nx * ny * nz
A = bj.synth_fem(nx, ny, nz, 0, n, dtype=dt)
for b in (32, 24, 32, 8):
    bp = torch.arange(0, n + b, b, dtype=torch.int32, device="cuda").clamp_(max=n)
    bp = torch.unique_consecutive(bp)
    sizes, vec, val = bj.layout_from_block_ptr(bp, dt)
    out = bj.Batch(sizes, vec, val, torch.empty(int(val[-1].item()), dtype=dt, device="cuda"))
    for _ in range(3): bj.extract(A, bp, out)
    torch.cuda.synchronize()
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(11)]
    for i in range(10):
        evs[i].record(); bj.extract(A, bp, out)
    evs[10].record(); torch.cuda.synchronize()
    print(b, [round(evs[i].elapsed_time(evs[i+1]), 3) for i in range(10)], flush=True)
