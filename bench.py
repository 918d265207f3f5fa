#!/usr/bin/env python3
"""Benchmark of the hot path: batched variable-size LU (implicit pivoting) +
triangular solves on B200, one process per GPU.

Default workload (BASELINE.json metric, north-star target): config C3 -- 1M
blocks with orders m ~ U{4..32}, fp64.  A *step* is one pass of the whole hot
path over one batch: layout (a1) + size plan + GETRF (a3) + GETRS (a4).  Each
step factors its own pristine copy of the batch (generated before the timed
region; 3.2 GB >> 126 MB L2, so no L2 flush is needed).

Multi-GPU (one process per GPU, NCCL): ``--gpus N`` started as a plain process
re-launches itself under torch.distributed.run.  The batch (C3: 1M blocks) is
split by the contiguous cost-balanced partitioner (row a6) -- strong scaling
(``--scaling weak`` replicates the per-GPU batch instead); ranks regenerate
their shard from the counter generator; no collective on the data path;
barrier + max over ranks of the CUDA-event time.

``--impl reference`` times the CPU oracle (the reference arm of this tier).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

FEM = {"C4": (174, 174, 22), "C5": (174, 174, 22), "SV": (174, 174, 22), "C5K": (174, 174, 22)}   # per-GPU z-slab of 22 planes

CONFIGS = {
    # name: (nblocks per GPU, lo, hi, dtype, description)
    "C3": (1_000_000, 4, 32, torch.float64, "C3: 1M blocks (sharded over the GPUs), m ~ U{4..32}, fp64, LU + solve"),
    "C3f32": (1_000_000, 4, 32, torch.float32, "C3: 1M blocks (sharded over the GPUs), m ~ U{4..32}, fp32, LU + solve"),
    "C2": (40_000, 32, 32, torch.float64, "C2: 40,000 blocks 32x32, fp64, LU + solve"),
    "C1": (1_000, 4, 16, torch.float64, "C1: 1,000 blocks m ~ U{4..16}, fp64 (latency case, L2-resident)"),
    "C4": (0, 24, 24, torch.float64, "C4: diagonal-block extraction, 27-pt x 3-dof FEM CSR, 1,998,216 rows/GPU, skewed hubs"),
    "C5": (0, 24, 24, torch.float64, "C5: block-Jacobi setup (extract + getrf) + 100 applies, 1,998,216 rows/GPU, b = 24"),
    "C5K": (0, 24, 24, torch.float64, "C5K (NEXT 4): block-Jacobi setup + BiCGSTAB solve (b = ones, x0 = 0, 1e-6 reduction) "
                                      "on the 27-pt x 3-dof FEM matrix, 1,998,216 rows/GPU (z-slabs, halo exchange), b = 24"),
    "SV": (0, 24, 24, torch.float64, "SV (NEXT 2): supervariable blocking of the C4 CSR pattern, 1,998,216 rows/GPU, bound 24"),
}


def esize(dt):
    return 8 if dt == torch.float64 else 4


def algorithmic_bytes(sizes: np.ndarray, dt) -> tuple[int, int]:
    """GETRF 2 s m^2 + 4m + 4 + 16; GETRS s m^2 + 4m + 2 s m + 16."""
    s = esize(dt)
    m = sizes.astype(np.int64)
    getrf = int((2 * s * m * m + 4 * m + 4 + 16).sum())
    getrs = int((s * m * m + 4 * m + 2 * s * m + 16).sum())
    return getrf, getrs


def fused_bytes(sizes: np.ndarray, dt) -> int:
    """bj_gesv_vbatched per block: A read + L\\U written (2 s m^2), b read + x
    written (2 s m), perm (4 m), info (4), val_off + vec_off (16)."""
    s = esize(dt)
    m = sizes.astype(np.int64)
    return int((2 * s * m * m + 2 * s * m + 4 * m + 20).sum())


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """SM clock / throttle-reason sampling (NVML, every ~2 ms) during the timed
    region, so even a short region gets samples."""

    REASONS = {  # nvmlClocksEventReason* bit -> name
        0x0000000000000004: "sw_power_cap",
        0x0000000000000008: "hw_slowdown",
        0x0000000000000020: "sw_thermal_slowdown",
        0x0000000000000040: "hw_thermal_slowdown",
        0x0000000000000080: "hw_power_brake_slowdown",
    }

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._ok = False

    def __enter__(self):
        try:
            import pynvml as N
            N.nvmlInit()
            self.N = N
            self.h = N.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = N.nvmlDeviceGetMaxClockInfo(self.h, N.NVML_CLOCK_SM)
            self._ok = True
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        except Exception:
            self._ok = False
        return self

    def _run(self):
        N = self.N
        while not self._stop.is_set():
            try:
                self.samples.append(N.nvmlDeviceGetClockInfo(self.h, N.NVML_CLOCK_SM))
                try:
                    mask = N.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                except AttributeError:
                    mask = N.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                for bit, name in self.REASONS.items():
                    if mask & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.002)

    def __exit__(self, *a):
        self._stop.set()
        if self._ok:
            self.t.join(timeout=2)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unsampled"]}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples), "source": "nvml"}


def dist_setup(args):
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if ws > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    return ws, rank, local


def barrier(ws):
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()


def max_over_ranks(v: float, ws: int) -> float:
    if ws == 1:
        return v
    t = torch.tensor([v], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


METRIC = "blocks/s (batched LU + solve)"


def workload(args, ws):
    """(nblocks_total, lo, hi, dtype, description, scaling) of the batched
    configs.  Multi-GPU default: STRONG scaling -- the config's batch (C3: 1M
    blocks) is sharded over the ranks by the partitioner (row a6); with
    --scaling weak every rank gets the full per-GPU batch instead."""
    nb, lo, hi, dt, desc = CONFIGS[args.config]
    if args.nblocks:
        nb = args.nblocks
    scaling = "weak" if (args.scaling == "weak" and ws > 1) else "strong"
    nb_total = nb * ws if scaling == "weak" else nb
    return nb_total, lo, hi, dt, desc, scaling


# --------------------------------------------------------------------------
# CPU oracle timing (cpu_baseline leg and --impl reference)
# --------------------------------------------------------------------------
def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_data(nb: int, lo: int, hi: int, dt, first: int = 0):
    """The first nb blocks of the workload (same counter generator as the GPU
    arm), generated with the C generator (bj_synth/fastgen.c)."""
    import bj_synth as S
    import oracle
    npdt = np.float64 if dt == torch.float64 else np.float32
    sizes = S.block_sizes(nb, lo, hi, first=first)
    vec, val = oracle.layout(sizes, esize(dt))
    A = S.block_values_fast(sizes, val, first=first, dtype=npdt)
    b = S.rhs_values_fast(sizes, first=first, dtype=npdt)
    return sizes, vec, val, A, b


def oracle_run(data, nthreads: int = 0):
    """One oracle GETRF + GETRS pass over `data`; returns (t_getrf, t_getrs) in s."""
    import oracle
    sizes, vec, val, A, b = data
    t0 = time.perf_counter()
    LU, piv, info = oracle.getrf_batch(sizes, val, vec, A, nthreads=nthreads)
    t1 = time.perf_counter()
    oracle.getrs_batch(sizes, val, vec, LU, piv, b, nthreads=nthreads)
    t2 = time.perf_counter()
    return t1 - t0, t2 - t1


def oracle_sample_size(nb_max: int, lo: int, hi: int, dt, seconds: float, nthreads: int = 0) -> int:
    """Blocks of the workload the oracle handles in about `seconds`."""
    probe = min(nb_max, 20000)
    tf, ts = oracle_run(oracle_data(probe, lo, hi, dt), nthreads)
    rate = probe / max(tf + ts, 1e-6)
    return int(max(min(nb_max, rate * seconds), min(nb_max, 1000)))


def oracle_baseline(nb: int, lo: int, hi: int, dt, budget_s: float):
    """cpu_baseline: the oracle as it stands on the host cores, on a bounded
    sample (the workload's first blocks), all cores (OpenMP over blocks) and
    one thread; GETRF and GETRS timed separately; median of 3."""
    import oracle
    cores = oracle.max_threads()
    n_all = oracle_sample_size(nb, lo, hi, dt, budget_s / 5.0)
    data = oracle_data(n_all, lo, hi, dt)
    reps = [oracle_run(data) for _ in range(3)]
    tf = float(np.median([r[0] for r in reps]))
    ts = float(np.median([r[1] for r in reps]))
    n_one = min(n_all, max(1000, int(n_all / max(cores, 1) / 2)))
    one = oracle_run((data[0][:n_one], data[1][:n_one + 1], data[2][:n_one + 1], data[3], data[4]), 1)
    getrf_b, getrs_b = algorithmic_bytes(data[0], dt)
    return {"value": n_all / (tf + ts), "unit": "blocks/s", "cores": cores, "kind": "oracle",
            "sample": f"first {n_all} blocks of the workload (GETRF+GETRS, OpenMP over blocks, median of 3)",
            "cpu_model": cpu_model(), "getrf_s": tf, "getrs_s": ts,
            "gbs": (getrf_b + getrs_b) / (tf + ts) / 1e9,
            "single_thread": {"value": n_one / (one[0] + one[1]), "unit": "blocks/s",
                              "sample": f"first {n_one} blocks", "getrf_s": one[0], "getrs_s": one[1]}}


def run_reference(args, ws, rank):
    """Reference arm of this tier: the CPU oracle as it stands, timed on the
    host cores, on the same workload / metric as our arm.  Each step is one
    GETRF + GETRS pass over a bounded sample (the workload's first blocks,
    sized so the whole run ends within a few minutes)."""
    nb_total, lo, hi, dt, desc, scaling = workload(args, ws)
    if rank != 0:
        return
    per_step = max(0.3, min(2.0, 90.0 / max(args.steps + args.warmup, 1)))
    n = oracle_sample_size(nb_total, lo, hi, dt, per_step)
    data = oracle_data(n, lo, hi, dt)
    import oracle
    cores = oracle.max_threads()
    times = []
    for i in range(args.warmup + args.steps):
        tf, ts = oracle_run(data)
        if i >= args.warmup:
            times.append(tf + ts)
    tot = sum(times)
    value = n * len(times) / tot
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "blocks/s",
        "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * tot / max(args.steps, 1), "higher_is_better": True, "scaling": scaling,
        "vs_baseline": None, "dtype": "f64" if dt == torch.float64 else "f32", "data": "synthetic",
        "config": {"workload": desc, "nblocks_total": nb_total,
                   "sample": f"each step: GETRF+GETRS over the first {n} blocks of the workload"},
        "cpu_baseline": {"value": value, "unit": "blocks/s", "cores": cores, "kind": "oracle",
                         "sample": f"{n} blocks per step (GETRF+GETRS, OpenMP over blocks)",
                         "cpu_model": cpu_model()},
        "e2e": {"value": value, "unit": "blocks/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------------
# GPU arm
# --------------------------------------------------------------------------
def run_ours(args, ws, rank, local):
    from paper_conf_icpp_anztdfq17_b200 import bj
    nb_total, lo, hi, dt, desc, scaling = workload(args, ws)
    # --- partition (row a6): global sizes from the counter generator
    from paper_conf_icpp_anztdfq17_b200 import dist as D
    sizes_all = bj.synth_sizes(nb_total, lo, hi)
    sizes_h = sizes_all.cpu().numpy()
    first, last = D.shard(sizes_h, ws, rank)
    nb = last - first
    sizes = sizes_all[first:last].clone()
    del sizes_all
    my_sizes = sizes_h[first:last]
    getrf_bytes, getrs_bytes = algorithmic_bytes(my_sizes, dt)

    base = bj.new_batch(sizes, dt)
    bj.synth_blocks(base, first=first, kind=1 if args.kind == "int" else 0)
    rhs = bj.synth_rhs(base, first=first)
    nvec = int(base.vec_off[-1].item())
    piv = torch.empty(max(nvec, 1), dtype=torch.int32, device="cuda")
    info = torch.empty(max(nb, 1), dtype=torch.int32, device="cuda")
    x = torch.empty_like(rhs)

    # pool of pristine copies (one per step, inputs > L2)
    copy_bytes = base.values.numel() * esize(dt)
    free = torch.cuda.mem_get_info()[0]
    cap = max(1, int((free - 8e9) // max(copy_bytes, 1)))
    pool_n = max(1, min(args.steps + args.warmup, cap, 64))
    pool = [base.values.clone() for _ in range(pool_n)]

    stream = torch.cuda.current_stream()

    def one_step(values, fused, evs=None):
        if evs is not None:
            evs[0].record(stream)
        v2, l2 = bj.layout(sizes, dt)                       # a1 (recomputed per step)
        plan = bj.Plan(sizes)                               # size buckets
        batch = bj.Batch(sizes, v2, l2, values)
        if evs is not None:
            evs[1].record(stream)
        if fused:
            bj.gesv(batch, piv, info, rhs, x, plan=plan)    # a3 + a4 fused (bj_gesv_vbatched)
            if evs is not None:
                evs[2].record(stream)
                evs[3].record(stream)
        else:
            bj.getrf(batch, piv, info, plan=plan)           # a3
            if evs is not None:
                evs[2].record(stream)
            bj.getrs(batch, piv, rhs, x, plan=plan)         # a4
            if evs is not None:
                evs[3].record(stream)
        return plan

    def timed(fused):
        """W warm-up steps, then K timed steps (each on its own pristine copy);
        returns (total ms over K steps, per-step [plan, getrf(+solve), getrs]
        ms, launches, clock summary)."""
        for i in range(args.warmup):
            one_step(pool[i % pool_n], fused).close()       # stream-ordered free, no sync
        barrier(ws)
        for i in range(min(args.warmup, pool_n)):           # restore used copies
            pool[i].copy_(base.values)
        barrier(ws)
        done, t_total_ms, per, launches = 0, 0.0, [], 0
        sampler = ClockSampler(local)
        with sampler:
            while done < args.steps:
                n = min(pool_n, args.steps - done)
                evs = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in range(n)]
                barrier(ws)
                start = torch.cuda.Event(enable_timing=True)
                end = torch.cuda.Event(enable_timing=True)
                bj.launch_count_reset()
                start.record(stream)
                for i in range(n):
                    one_step(pool[i], fused, evs[i]).close()
                end.record(stream)
                launches += bj.launch_count()
                barrier(ws)
                t_total_ms += start.elapsed_time(end)
                for e in evs:
                    per.append((e[0].elapsed_time(e[1]), e[1].elapsed_time(e[2]), e[2].elapsed_time(e[3])))
                done += n
                for i in range(min(n, pool_n)):              # pristine copies for what follows
                    pool[i].copy_(base.values)
        barrier(ws)
        return t_total_ms, np.array(per), launches, sampler.summary()

    # the separate calls (getrf + getrs: the headline step), then the fused call
    t_sep, per_sep, launches, clocks = timed(False)
    t_fus, per_fus, launches_fus, clocks_fus = timed(True) if not args.no_fused else (None, None, 0, None)
    t_ms = max_over_ranks(t_sep, ws)
    plan_ms = float(per_sep[:, 0].mean())
    getrf_ms = max_over_ranks(float(per_sep[:, 1].mean()), ws)
    getrs_ms = max_over_ranks(float(per_sep[:, 2].mean()), ws)
    step_each = per_sep.sum(axis=1)
    step_med, step_min = float(np.median(step_each)), float(step_each.min())

    # correctness sentinel on the timed data (cheap): no zero pivots expected
    bad = int((info[:nb] != 0).sum().item())

    hbm, peak_src = load_peaks()
    dom = "getrf" if getrf_ms >= getrs_ms else "getrs"
    dom_bytes, dom_ms = (getrf_bytes, getrf_ms) if dom == "getrf" else (getrs_bytes, getrs_ms)
    achieved = dom_bytes / (dom_ms * 1e-3) / 1e9
    traffic = None
    tf = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tf):
        traffic = json.load(open(tf)).get(f"{args.config}:{dom}")
    step_bytes = getrf_bytes + getrs_bytes
    ms_per_step = t_ms / args.steps
    value = nb_total / (ms_per_step * 1e-3)
    fused = None
    if t_fus is not None:
        t_fus = max_over_ranks(t_fus, ws)
        gesv_ms = max_over_ranks(float(per_fus[:, 1].mean()), ws)
        gesv_bytes = fused_bytes(my_sizes, dt)
        fms = t_fus / args.steps
        fused = {"ms_per_step": fms, "value": nb_total / (fms * 1e-3), "unit": "blocks/s",
                 "step": "layout + plan + bj_gesv_vbatched (GETRF + GETRS fused; bit-identical outputs)",
                 "gesv_ms": gesv_ms, "gesv_bytes": gesv_bytes,
                 "gesv_frac": gesv_bytes / (gesv_ms * 1e-3) / 1e9 / hbm, "gpu_launches": launches_fus}

    # ---- e2e: the C-ABI call with HOST buffers (bj_gesv_host), copies inside
    e2e = None
    if not args.no_e2e:
        ws_obj = bj.Workspace()
        sizes_pin = sizes.cpu().pin_memory()
        A_pin = base.values.cpu().pin_memory()
        b_pin = rhs.cpu().pin_memory()
        x_pin = torch.empty_like(b_pin).pin_memory()
        p_pin = torch.empty(max(nvec, 1), dtype=torch.int32).pin_memory()
        i_pin = torch.empty(max(nb, 1), dtype=torch.int32).pin_memory()
        e2e_steps = max(1, min(args.steps, 3))
        ws_obj.gesv_host(sizes_pin, A_pin, b_pin, x_pin, p_pin, i_pin)        # warm-up
        barrier(ws)
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for _ in range(e2e_steps):
            ws_obj.gesv_host(sizes_pin, A_pin, b_pin, x_pin, p_pin, i_pin)
        t1.record(stream)
        barrier(ws)
        e_ms = max_over_ranks(t0.elapsed_time(t1) / e2e_steps, ws)
        h2d = sizes_pin.numel() * 4 + A_pin.numel() * esize(dt) + b_pin.numel() * esize(dt)
        d2h = x_pin.numel() * esize(dt) + p_pin.numel() * 4 + i_pin.numel() * 4
        e2e = {"value": nb_total / (e_ms * 1e-3), "unit": "blocks/s", "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h), "ms_per_step": e_ms, "steps": e2e_steps,
               "api": "bj_gesv_host (pinned host buffers, synchronous)"}
        ws_obj.close()

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu:
        cpu = oracle_baseline(nb_total, lo, hi, dt, args.cpu_budget)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "blocks/s", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": scaling, "vs_baseline": None, "dtype": "f64" if dt == torch.float64 else "f32",
            "data": "synthetic (counter-based splitmix64, generated on device)",
            "config": {"workload": desc, "nblocks_total": nb_total, "nblocks_rank0": nb, "sizes": f"U{{{lo}..{hi}}}",
                       "values": "U[-1,1)" if args.kind == "uniform" else "U{-3..3} integers (ties, singular blocks)",
                       "step": "layout + plan + bj_getrf_vbatched + bj_getrs_vbatched",
                       "parallelism": f"dp{ws} (contiguous cost-balanced shards, {scaling} scaling)",
                       "l2": f"inputs larger than L2: each step factors its own pristine {copy_bytes / 1e9:.2f} GB copy"},
            "roofline": {"bound": "hbm", "kernel": f"bj_{dom}_vbatched (all its launches)", "achieved": achieved,
                         "peak": hbm, "unit": "GB/s", "frac": achieved / hbm, "traffic": traffic,
                         "peak_source": peak_src, "bytes_per_launch": dom_bytes,
                         "bytes_formula": ("per block 2 s m^2 + 4 m + 20" if dom == "getrf"
                                           else "per block s m^2 + 2 s m + 4 m + 16")},
            "other_call_roofline": ({"kernel": "bj_getrs_vbatched", "frac": getrs_bytes / (getrs_ms * 1e-3) / 1e9 / hbm}
                                    if dom == "getrf" else
                                    {"kernel": "bj_getrf_vbatched", "frac": getrf_bytes / (getrf_ms * 1e-3) / 1e9 / hbm}),
            "step_hbm": {"algorithmic_bytes": step_bytes, "achieved_gbs": step_bytes / (ms_per_step * 1e-3) / 1e9,
                         "frac": step_bytes / (ms_per_step * 1e-3) / 1e9 / hbm},
            "breakdown_ms": {"layout_plan": plan_ms, "getrf": getrf_ms, "getrs": getrs_ms},
            "fused_gesv": fused,
            "step_ms_rank0": {"median": step_med, "min": step_min},
            "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches, "clocks": clocks,
            "nonzero_info_blocks": bad,
        }
        print(json.dumps(line), flush=True)


def run_fem(args, ws, rank, local):
    """C4 (extraction) and C5 (setup + 100 applies) on a per-rank z-slab of a
    174 x 174 x (22 * ws) node grid (rows sharded; global column ids)."""
    from paper_conf_icpp_anztdfq17_b200 import bj
    nx, ny, nzr = FEM[args.config]
    b = args.block or 24
    dt = torch.float64
    nz = nzr * ws
    plane = 3 * nx * ny
    r0, r1 = rank * nzr * plane, (rank + 1) * nzr * plane
    n = r1 - r0
    A = bj.synth_fem(nx, ny, nz, r0, r1, dtype=dt)
    bp = torch.arange(0, n + b, b, dtype=torch.int32, device="cuda").clamp_(max=n)
    bp = torch.unique_consecutive(bp)
    nb = bp.numel() - 1
    sizes, vec, val = bj.layout_from_block_ptr(bp, dt)
    out = bj.Batch(sizes, vec, val, torch.empty(int(val[-1].item()), dtype=dt, device="cuda"))
    # algorithmic bytes
    rows = torch.repeat_interleave(torch.arange(n, device="cuda"), A.row_ptr.diff())
    blk_of_row = torch.div(rows, b, rounding_mode="floor")
    c = A.col_idx.long() - r0
    hits = int(((c >= blk_of_row * b) & (c < torch.clamp((blk_of_row + 1) * b, max=n))).sum().item())
    del rows, blk_of_row, c
    m = sizes.long()
    ext_bytes = 8 * (n + 1) + 4 * A.col_idx.numel() + 8 * hits + 8 * int((m * m).sum().item()) + 4 * (nb + 1)
    getrf_bytes = int((2 * 8 * m * m + 4 * m + 20).sum().item())
    getrs_bytes = int((8 * m * m + 4 * m + 16 * m + 16).sum().item())
    stream = torch.cuda.current_stream()
    hbm, peak_src = load_peaks()
    piv = torch.empty(n, dtype=torch.int32, device="cuda")
    info = torch.empty(nb, dtype=torch.int32, device="cuda")
    x = torch.rand(n, dtype=dt, device="cuda") * 2 - 1
    y = torch.empty_like(x)
    h = bj.Handle() if args.config == "C5" else None
    hinv = bj.Handle() if args.config == "C5" else None
    napply = 100

    sv_bytes = 8 * (n + 1) + 4 * A.col_idx.numel() + 4 * (n // b + 2)   # row_ptr + col_idx read, block_ptr written
    sv_nb = [0]

    def step(evs=None, inverse=False):
        if args.config == "SV":
            sv_nb[0] = bj.supervariable_blocking(A, b).numel() - 1
        elif args.config == "C4":
            bj.extract(A, bp, out)
        else:
            hh = hinv if inverse else h
            if evs is not None:
                evs[0].record(stream)
            if inverse:
                hh.setup_inverse(A, bp, out, piv, info)      # NEXT(3): extract + GJE inverses
            else:
                hh.setup(A, bp, out, piv, info)              # extract + GETRF
            if evs is not None:
                evs[1].record(stream)
            for _ in range(napply):
                hh.apply(x, y)                               # GETRS / GEMV

    def timed(inverse=False):
        for _ in range(args.warmup):
            step(inverse=inverse)
        barrier(ws)
        sampler = ClockSampler(local)
        bj.launch_count_reset()
        with sampler:
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            evs = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(args.steps)]
            barrier(ws)
            e0.record(stream)
            for i in range(args.steps):
                step(evs[i] if args.config == "C5" else None, inverse)
            e1.record(stream)
            barrier(ws)
        return e0, e1, evs, bj.launch_count(), sampler

    e0, e1, evs, launches, sampler = timed()
    t_ms = max_over_ranks(e0.elapsed_time(e1), ws)
    ms = t_ms / args.steps
    inverse_variant = None
    if args.config == "C5":
        i0, i1, ievs, ilaunch, _ = timed(inverse=True)
        ims = max_over_ranks(i0.elapsed_time(i1), ws) / args.steps
        isetup = float(np.mean([e[0].elapsed_time(e[1]) for e in ievs]))
        iapply = (ims - isetup) / napply
        inv_bytes = int((8 * m * m + 16 * m + 16).sum().item())     # GEMV: Dinv + x in + y out + offsets
        inverse_variant = {"ms_per_step": ims, "value": ws / (ims * 1e-3), "unit": "setups/s",
                           "step": "bj_setup_inverse (extract + Gauss-Jordan inverses) + 100 bj_apply (GEMV)",
                           "breakdown_ms": {"setup": isetup, "apply": iapply},
                           "apply_roofline": {"achieved": inv_bytes / (iapply * 1e-3) / 1e9,
                                              "frac": inv_bytes / (iapply * 1e-3) / 1e9 / load_peaks()[0],
                                              "bytes": inv_bytes}, "gpu_launches": ilaunch}
    line = {"n_gpus": ws, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic (counter-based FEM CSR generated on device)",
            "gpu_launches": launches, "clocks": sampler.summary()}
    if args.config == "SV":
        achieved = sv_bytes / (ms * 1e-3) / 1e9
        line.update({"metric": "matrix rows blocked per second", "value": n * ws / (ms * 1e-3),
                     "unit": "rows/s", "higher_is_better": True,
                     "config": {"workload": CONFIGS["SV"][4], "bound": b, "rows_per_gpu": n,
                                "nnz_per_gpu": A.col_idx.numel(), "blocks": sv_nb[0],
                                "l2": "col_idx (0.62 GB) larger than L2"},
                     "roofline": {"bound": "hbm", "kernel": "bj_supervariable_blocking (all launches)",
                                  "achieved": achieved, "peak": hbm, "unit": "GB/s", "frac": achieved / hbm,
                                  "traffic": None, "peak_source": peak_src, "bytes_per_launch": sv_bytes}})
    elif args.config == "C4":
        achieved = ext_bytes / (ms * 1e-3) / 1e9
        line.update({"metric": "diagonal blocks extracted per second", "value": nb * ws / (ms * 1e-3),
                     "unit": "blocks/s", "higher_is_better": True,
                     "config": {"workload": CONFIGS["C4"][4], "block": b, "rows_per_gpu": n, "nnz_per_gpu": A.col_idx.numel(),
                                "in_block_hits": hits, "l2": "inputs (1.2 GB) larger than L2"},
                     "roofline": {"bound": "hbm", "kernel": "bj_extract", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                                  "frac": achieved / hbm, "traffic": None, "peak_source": peak_src,
                                  "bytes_per_launch": ext_bytes}})
    else:
        setup_ms = float(np.mean([e[0].elapsed_time(e[1]) for e in evs]))
        apply_ms = (ms - setup_ms) / napply
        line.update({"metric": "block-Jacobi setup + 100 applies per second", "value": ws / (ms * 1e-3),
                     "unit": "setups/s", "higher_is_better": True,
                     "config": {"workload": CONFIGS["C5"][4], "block": b, "rows_per_gpu": n, "applies": napply},
                     "breakdown_ms": {"setup": setup_ms, "apply": apply_ms},
                     "inverse_variant": inverse_variant,
                     "step_hbm": {"algorithmic_bytes": ext_bytes + getrf_bytes + napply * getrs_bytes,
                                  "achieved_gbs": (ext_bytes + getrf_bytes + napply * getrs_bytes) / (ms * 1e-3) / 1e9},
                     "roofline": {"bound": "hbm", "kernel": "bj_apply", "achieved": getrs_bytes / (apply_ms * 1e-3) / 1e9,
                                  "peak": hbm, "unit": "GB/s", "frac": getrs_bytes / (apply_ms * 1e-3) / 1e9 / hbm,
                                  "traffic": None, "peak_source": peak_src, "bytes_per_launch": getrs_bytes}})
    if rank == 0:
        print(json.dumps(line), flush=True)


def run_krylov(args, ws, rank, local):
    """C5K (NEXT 4): block-Jacobi setup + preconditioned BiCGSTAB solve of
    the section IV.D set-up on a 174 x 174 x (22 * ws) FEM grid,
    rank r owning the r-th 22-plane z-slab (weak scaling; halo exchange and
    rank-ordered dot sums through bj.TorchComm over NCCL when ws > 1)."""
    from paper_conf_icpp_anztdfq17_b200 import bj
    nx, ny, nzr = FEM["C5K"]
    b = args.block or 24
    dt = torch.float64
    nz = nzr * ws
    plane = 3 * nx * ny
    r0, r1 = rank * nzr * plane, (rank + 1) * nzr * plane
    n = r1 - r0
    A = bj.synth_fem(nx, ny, nz, r0, r1, dtype=dt)            # local rows, global columns
    nnz = A.col_idx.numel()
    bp = torch.arange(0, n + b, b, dtype=torch.int32, device="cuda").clamp_(max=n)
    bp = torch.unique_consecutive(bp)
    nb = bp.numel() - 1
    sizes, vec, val = bj.layout_from_block_ptr(bp, dt)
    fac = bj.Batch(sizes, vec, val, torch.empty(int(val[-1].item()), dtype=dt, device="cuda"))
    piv = torch.empty(n, dtype=torch.int32, device="cuda")
    info = torch.empty(nb, dtype=torch.int32, device="cuda")
    comm = None
    Aloc = bj.Csr(A.row_ptr, A.col_idx, A.values, 0)           # SpMV view: column ids as stored
    if ws > 1:
        bounds = np.arange(ws + 1, dtype=np.int64) * n
        cl, hc, rc = bj.halo_plan(A.col_idx.cpu().numpy(), r0, r1, bounds)
        comm = bj.TorchComm(hc, rc, r0, "cuda")
        Aloc = bj.Csr(A.row_ptr, torch.from_numpy(cl).cuda(), A.values, 0)
    rhs = torch.ones(n, dtype=dt, device="cuda")
    x = torch.empty(n + (comm.nhalo if comm else 0), dtype=dt, device="cuda")
    xs = torch.rand(n + (comm.nhalo if comm else 0), dtype=dt, device="cuda") * 2 - 1
    ys = torch.empty(n, dtype=dt, device="cuda")
    h = bj.Handle()
    stream = torch.cuda.current_stream()
    hbm, peak_src = load_peaks()
    iters = [0]

    def step(evs=None):
        if evs is not None:
            evs[0].record(stream)
        h.setup(A, bp, fac, piv, info)                         # extract + GETRF (fused for m = 17..32)
        if evs is not None:
            evs[1].record(stream)
        it, res = bj.bicgstab(h, Aloc, rhs, x, tol=1e-6, maxit=10000, comm=comm)
        iters[0] = it
        return res

    for _ in range(args.warmup):
        step()
    barrier(ws)
    sampler = ClockSampler(local)
    bj.launch_count_reset()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(args.steps)]
    with sampler:
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        barrier(ws)
        e0.record(stream)
        for i in range(args.steps):
            res = step(evs[i])
        e1.record(stream)
        barrier(ws)
    torch.cuda.synchronize()
    launches = bj.launch_count()
    ms = max_over_ranks(e0.elapsed_time(e1), ws) / args.steps
    setup_ms = float(np.mean([e[0].elapsed_time(e[1]) for e in evs]))
    it = iters[0]
    # SpMV alone (the dominant kernel): R27 over the local rows, CUDA events on its stream
    nrep = 20
    s0 = torch.cuda.Event(enable_timing=True)
    s1 = torch.cuda.Event(enable_timing=True)
    bj.spmv(Aloc, xs, ys)
    s0.record(stream)
    for _ in range(nrep):
        bj.spmv(Aloc, xs, ys)
    s1.record(stream)
    torch.cuda.synchronize()
    spmv_ms = s0.elapsed_time(s1) / nrep
    spmv_bytes = 8 * (n + 1) + 12 * nnz + 16 * n          # row_ptr + (col, val) per entry + x read once + y write
    achieved = spmv_bytes / (spmv_ms * 1e-3) / 1e9
    solve_ms = ms - setup_ms
    # per-iteration algorithmic bytes: 2 SpMV + 2 GETRS applies + vector updates / dots (16 vector passes)
    m = sizes.long()
    getrs_bytes = int((8 * m * m + 4 * m + 16 * m + 16).sum().item())
    iter_bytes = 2 * spmv_bytes + 2 * getrs_bytes + 8 * n * (3 + 2 + 3 + 2 + 8)
    line = {"metric": "preconditioned Krylov solves per second (setup + BiCGSTAB to 1e-6)",
            "value": ws / (ms * 1e-3), "unit": "solves/s", "higher_is_better": True,
            "n_gpus": ws, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic (counter-based FEM CSR generated on device)",
            "config": {"workload": CONFIGS["C5K"][4], "block": b, "rows_per_gpu": n, "nnz_per_gpu": nnz,
                       "iterations": it, "relative_residual": res, "l2": "CSR (1.9 GB/GPU) larger than L2"},
            "breakdown_ms": {"setup": setup_ms, "solve": solve_ms, "per_iteration": solve_ms / max(it, 1),
                             "spmv": spmv_ms},
            "iteration_hbm": {"algorithmic_bytes": iter_bytes,
                              "achieved_gbs": iter_bytes / (solve_ms / max(it, 1) * 1e-3) / 1e9},
            "roofline": {"bound": "hbm", "kernel": "bj_spmv (k_spmv + k_spmv_long)", "achieved": achieved,
                         "peak": hbm, "unit": "GB/s", "frac": achieved / hbm, "traffic": None,
                         "peak_source": peak_src, "bytes_per_launch": spmv_bytes},
            "gpu_launches": launches, "clocks": sampler.summary()}
    if rank == 0 and ws == 1 and not args.no_cpu:
        import time
        import bj_synth as S
        import oracle
        rp, ci, va = S.fem_csr_fast(nx, ny, nz)
        t0 = time.perf_counter()
        _, it_o, res_o, *_ = oracle.bicgstab(rp, ci, va, S.uniform_block_ptr(n, b), np.ones(n))
        t_o = time.perf_counter() - t0
        line["cpu_baseline"] = {"value": 1.0 / t_o, "unit": "solves/s", "cores": os.cpu_count(), "kind": "oracle",
                                "sample": f"one full solve incl. oracle extract + getrf ({it_o} iterations, "
                                          f"same matrix); iterations equal: {it_o == it}"}
    if rank == 0:
        print(json.dumps(line), flush=True)


def spawn(n: int) -> int:
    """`bench.py --gpus N` started as a plain process: re-launch it under
    torch.distributed.run with one rank per GPU (the launch the driver uses)."""
    import socket
    import subprocess
    if torch.cuda.device_count() < n:
        print(json.dumps({"error": f"--gpus {n} requested but {torch.cuda.device_count()} GPU(s) visible"}))
        return 2
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C3", choices=sorted(CONFIGS))
    ap.add_argument("--nblocks", type=int, default=0, help="override blocks per GPU")
    ap.add_argument("--block", type=int, default=0, help="C4/C5 diagonal block size (default 24)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-fused", action="store_true", help="skip the extra fused bj_gesv_vbatched measurement")
    ap.add_argument("--kind", default="uniform", choices=["uniform", "int"],
                    help="block values: U[-1,1) (default) or the tie-heavy integer stress set U{-3..3}")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"],
                    help="multi-GPU batched configs: shard the config's batch (strong) or replicate it per GPU (weak)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 0)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn(args.gpus))
    if args.impl == "reference":
        # the CPU oracle arm: rank 0 alone runs it; other ranks exit without work
        ws = int(os.environ.get("WORLD_SIZE", "1"))
        rank = int(os.environ.get("RANK", "0"))
        run_reference(args, ws, rank)
        return
    ws, rank, local = dist_setup(args)
    if args.config == "C5K":
        run_krylov(args, ws, rank, local)
    elif args.config in FEM:
        run_fem(args, ws, rank, local)
    else:
        run_ours(args, ws, rank, local)
    if ws > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
