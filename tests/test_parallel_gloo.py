"""Multi-process plumbing of the multi-GPU driver on CPU (gloo, world_size 2):
tree blob broadcast, warp-aligned sharding, in-place all-gather of results,
max-over-ranks timing.  The traversal itself needs the GPU; this checks that
what every rank receives and assembles is exactly right."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_goldfarbjk13_b200.parallel import balanced_ranges, shard_range


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import ttgen
        import paper_conf_sc_goldfarbjk13_b200 as P
        from paper_conf_sc_goldfarbjk13_b200 import parallel as PAR

        b = ttgen.plummer(4096, seed=300)
        local = P.build_oct(b).pack()  # every rank can pack: used to check the bytes
        blob = PAR.broadcast_blob(local if rank == 0 else None, "cpu")
        ok_blob = bool(np.array_equal(blob.numpy(), local))
        # results: each rank fills its own warp-aligned shard, then all-gather
        n = 64 * world * 50
        full = torch.full((n, 4), -1.0)
        lo, hi = PAR.shard_range(n, rank, world)
        full[lo:hi] = torch.arange(lo, hi, dtype=torch.float32)[:, None] + torch.tensor([0.0, 0.25, 0.5, 0.75])
        PAR.allgather_rows(full, world)
        want = torch.arange(n, dtype=torch.float32)[:, None] + torch.tensor([0.0, 0.25, 0.5, 0.75])
        ok_gather = bool(torch.equal(full, want))
        # int32 id column (the sharded time step's body ids), same row sharding
        ids = torch.full((n,), -1, dtype=torch.int32)
        ids[lo:hi] = torch.arange(lo, hi, dtype=torch.int32) * 3
        PAR.allgather_rows(ids.view(-1, 1), world)
        ok_gather = ok_gather and bool(torch.equal(ids, torch.arange(n, dtype=torch.int32) * 3))
        # cost-balanced unequal shards + padded all-gather
        costs = torch.ones(n)
        costs[: n // 4] = 5.0  # the first quarter costs 5x
        ranges = PAR.balanced_ranges(costs, world)
        lo2, hi2 = ranges[rank]
        full2 = torch.full((n, 3), -1.0)
        full2[lo2:hi2] = torch.arange(lo2, hi2, dtype=torch.float32)[:, None] * torch.tensor([1.0, 2.0, 3.0])
        PAR.allgather_rows_var(full2, ranges)
        ok_gather = ok_gather and bool(torch.equal(
            full2, torch.arange(n, dtype=torch.float32)[:, None] * torch.tensor([1.0, 2.0, 3.0])))
        ok_gather = ok_gather and ranges[0][1] - ranges[0][0] < n // world  # the costly part gets fewer rows
        mx = PAR.max_over_ranks(float(rank + 1) * 1.5, "cpu")
        q.put((rank, ok_blob, ok_gather, mx))
        dist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e), None, None))


def test_broadcast_shard_allgather_world2():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ok_blob, ok_gather, mx in res:
        assert ok_blob is True, (rank, ok_blob)
        assert ok_gather is True
        assert mx == 3.0


@pytest.mark.parametrize("n,world", [(1_000_000, 1), (2_000_000, 2), (8_000_000, 8), (20011, 4), (7, 3)])
def test_shard_range_partitions_warp_aligned(n, world):
    covered = np.zeros(n, np.int32)
    for r in range(world):
        lo, hi = shard_range(n, r, world)
        assert lo % 64 == 0 or lo == n
        covered[lo:hi] += 1
    assert np.all(covered == 1)


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_balanced_ranges_cover_aligned_and_balance(world):
    """Contiguous, warp-aligned, covering; the per-shard cost is within one
    warp of points of total/world (SURVEY §8(e) cost-weighted split)."""
    rng = np.random.default_rng(world)
    n = 64 * 1000 + 37
    c = torch.from_numpy(rng.gamma(0.5, 2.0, n))
    rs = balanced_ranges(c, world)
    covered = np.zeros(n, np.int32)
    for lo, hi in rs:
        assert lo % 64 == 0 or lo == n
        covered[lo:hi] += 1
    assert np.all(covered == 1)
    tot = float(c.sum())
    per = [float(c[lo:hi].sum()) for lo, hi in rs]
    worst = float(torch.topk(c, 64).values.sum())
    assert max(per) - tot / world <= worst
