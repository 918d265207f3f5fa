"""Multi-process (world size 2, gloo, CPU) tests of the sharded path's host
logic: the partitioner gives every rank the same contiguous, cost-balanced
ranges; ranks regenerate their shards from the counter generator; the
concatenation of per-rank oracle results equals the unsharded result bit for
bit; max-over-ranks timing."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import bj_synth as S
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, nb, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icpp_anztdfq17_b200 import dist as D
        sizes_all = S.block_sizes(nb, 4, 32)
        first, last = D.shard(sizes_all, world, rank)
        sizes = S.block_sizes(last - first, 4, 32, first=first)          # regenerated locally
        assert np.array_equal(sizes, sizes_all[first:last])
        vec, val = oracle.layout(sizes, 8)
        A = S.block_values(sizes, val, first=first)
        b = S.rhs_values(sizes, first=first)
        LU, piv, info = oracle.getrf_batch(sizes, val, vec, A, nthreads=1)
        x = oracle.getrs_batch(sizes, val, vec, LU, piv, b, nthreads=1)
        xg = D.gather_shards(torch.from_numpy(x))
        pg = D.gather_shards(torch.from_numpy(piv.astype(np.int64)))
        t = D.max_over_ranks(float(rank + 1))
        bounds = torch.tensor([first, last], dtype=torch.int64)
        allb = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allb, bounds)
        if rank == 0:
            q.put((xg.numpy(), pg.numpy(), t, [tuple(x.tolist()) for x in allb]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_sharded_oracle_equals_unsharded(world):
    nb = 3001
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, nb, q)) for r in range(world)]
    for p in procs:
        p.start()
    xg, pg, t, bounds = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    # contiguous cover, balanced cost
    assert bounds[0][0] == 0 and bounds[-1][1] == nb
    assert all(bounds[i][1] == bounds[i + 1][0] for i in range(world - 1))
    sizes = S.block_sizes(nb, 4, 32)
    cost = sizes.astype(np.int64) ** 2
    shares = [cost[a:b].sum() for a, b in bounds]
    assert max(shares) - min(shares) <= 32 * 32
    # bit-identical to the unsharded run
    vec, val = oracle.layout(sizes, 8)
    A = S.block_values(sizes, val)
    b = S.rhs_values(sizes)
    LU, piv, info = oracle.getrf_batch(sizes, val, vec, A)
    x = oracle.getrs_batch(sizes, val, vec, LU, piv, b)
    assert np.array_equal(xg.view(np.uint64), x.view(np.uint64))
    assert np.array_equal(pg, piv.astype(np.int64))
    assert t == float(world)


def test_shard_edges_small_batches():
    from paper_conf_icpp_anztdfq17_b200 import dist as D
    for nb in (0, 1, 2, 5):
        sizes = S.block_sizes(nb, 4, 32)
        ranges = [D.shard(sizes, 8, r) for r in range(8)]
        covered = [i for a, b in ranges for i in range(a, b)]
        assert covered == list(range(nb))
