"""NEXT(4) multi-rank path on CPU (gloo, world size 2 and 3): the halo plan
(bj_halo_plan, host C in libbj.so), the bj_comm exchange over
torch.distributed (bj.TorchComm: one all_to_all_single per halo exchange, one
all_gather_into_tensor per dot phase) and the rank-ordered dot sums of R30.

Each rank owns a z-slab of rows of a small FEM matrix, runs the R29
iteration on its rows with the oracle's SpMV / GETRS building blocks over its
extended vector [own rows | halo], and the gathered solution must equal the
single-process oracle solve with the same shard bounds bit for bit (same
iteration count and residual)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import bj_synth as S
import oracle

GRID = (9, 8, 9)
BLK = 24


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _bounds(world):
    nx, ny, nz = GRID
    plane = 3 * nx * ny
    cuts = [round(nz * r / world) for r in range(world + 1)]
    return np.array([c * plane for c in cuts], np.int64)


def _block_ptr(bounds):
    """Blocks of BLK rows restarting at every shard edge (no block crosses a shard)."""
    edges = []
    for lo, hi in zip(bounds[:-1], bounds[1:]):
        edges.extend(range(int(lo), int(hi), BLK))
    edges.append(int(bounds[-1]))
    return np.unique(np.asarray(edges, np.int32))


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icpp_anztdfq17_b200 import bj
        g = S.FemGrid(*GRID)
        bounds = _bounds(world)
        lo, hi = int(bounds[rank]), int(bounds[rank + 1])
        n = hi - lo
        rp, ci, va = g.csr(lo, hi)                                   # local rows, global columns
        col_local, halo_cols, recv_counts = bj.halo_plan(ci, lo, hi, bounds)
        comm = bj.TorchComm(halo_cols, recv_counts, lo, "cpu")
        nh = comm.nhalo
        # the halo plan: every remote column once, ascending, grouped by owner
        assert np.all(np.diff(halo_cols) > 0) and np.all((halo_cols < lo) | (halo_cols >= hi))
        assert recv_counts.sum() == nh and recv_counts[rank] == 0
        # preconditioner of the own rows (blocks inside the shard)
        bp = _block_ptr(bounds)
        bpl = bp[(bp >= lo) & (bp <= hi)] - lo
        D, sizes, vec, val = oracle.extract(rp, ci, va, bpl, lo)
        LU, perm, info = oracle.getrf_batch(sizes, val, vec, D)

        def apply(u):
            return oracle.getrs_batch(sizes, val, vec, LU, perm, u)

        def halo(u):
            ext = np.zeros(n + nh)
            ext[:n] = u
            comm.send_buf[: comm.nsend] = torch.from_numpy(u[comm.send_idx.numpy()])
            comm.halo_exchange(async_op=True)      # the library's order: start, (interior rows), wait
            comm.halo_wait()
            ext[n:] = comm.recv_buf[:nh].numpy()
            return ext

        def gdot(pairs):
            """R30: rank values (R28 over the own rows), allgather, rank-order sum from +0."""
            comm.gather_buf.zero_()
            for d, (u, w) in enumerate(pairs):
                comm.gather_buf[rank * 4 + d] = oracle.dot(u, w)
            comm.allgather(len(pairs))
            gb = comm.gather_buf.numpy().reshape(world, 4)
            out = []
            for d in range(len(pairs)):
                acc = 0.0
                for r in range(world):
                    acc = acc + gb[r, d]
                out.append(acc)
            return out

        def spmv(u):
            return oracle.spmv(rp, col_local, va, halo(u), col_offset=0)

        # the halo exchange delivers the owners' values
        xg = np.arange(bounds[-1], dtype=np.float64) * 0.5 - 3.0
        ext = halo(xg[lo:hi])
        assert np.array_equal(ext[n:], xg[halo_cols])
        Ag_rows = oracle.spmv(rp, ci, va, xg, col_offset=0)
        assert np.array_equal(spmv(xg[lo:hi]), Ag_rows)

        # R29 on the own rows (the same expressions as the library and the oracle)
        b = np.ones(n)
        x = np.zeros(n)
        r = b.copy()
        rh = b.copy()
        p = np.zeros(n)
        v = np.zeros(n)
        rho_prev = alpha = omega = 1.0
        nb_norm = np.sqrt(gdot([(b, b)])[0])
        res, it, done = 1.0, 0, False
        for it in range(1, 500):
            rho = gdot([(rh, r)])[0]
            beta = (rho / rho_prev) * (alpha / omega)
            p = _fma(beta, _fma(-omega, v, p), r)
            ph = apply(p)
            v = spmv(ph)
            alpha = rho / gdot([(rh, v)])[0]
            s = _fma(-alpha, v, r)
            sh = apply(s)
            t = spmv(sh)
            ts, tt = gdot([(t, s), (t, t)])
            omega = ts / tt
            x = _fma(omega, sh, _fma(alpha, ph, x))
            r = _fma(-omega, t, s)
            res = np.sqrt(gdot([(r, r)])[0])
            if res <= 1e-6 * nb_norm:
                done = True
                break
            rho_prev = rho
        L = int(np.diff(bounds).max())                              # gloo all_gather: equal sizes
        mine = torch.zeros(L, dtype=torch.float64)
        mine[:n] = torch.from_numpy(x)
        allx = [torch.zeros(L, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(allx, mine)
        if rank == 0:
            xs = [allx[i][: int(bounds[i + 1] - bounds[i])] for i in range(world)]
            q.put((torch.cat(xs).numpy(), it if done else -1, res / nb_norm))
    finally:
        dist.destroy_process_group()


def _fma(a, x, y):
    """Elementwise single-rounding fma(a, x, y) through the oracle's C fma
    (numpy has none): a scalar or vector a."""
    a = np.broadcast_to(np.asarray(a, np.float64), np.shape(x))
    return oracle.fma_vec(a, x, y)


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_bicgstab_equals_oracle(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    x, it, res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    g = S.FemGrid(*GRID)
    rp, ci, va = g.csr()
    bounds = _bounds(world)
    x_o, it_o, res_o, *_ = oracle.bicgstab(rp, ci, va, _block_ptr(bounds), np.ones(g.n), bounds=bounds)
    assert it == it_o and res == res_o
    assert np.array_equal(x.view(np.uint64), x_o.view(np.uint64))
