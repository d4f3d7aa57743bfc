"""Multi-GPU driver: one process per GPU, tree replicated by NCCL broadcast,
points sharded, results all-gathered (north_star).

Points are independent and the tree is read-only during a pass,
so the traversal itself has no exchange step.  The only collectives are:
  * ``broadcast_tree``: rank 0 packs the tree (position-independent int32
    blob, include/tt.h tt_tree_pack) and broadcasts the bytes; every rank
    adopts them with tt_tree_from_blob(mem=DEVICE) -- once per tree;
  * ``allgather_rows``: after the pass each rank holds the results of its
    shard (a contiguous range of point indices) and an in-place
    all_gather_into_tensor assembles the full result on every rank.
The same functions run under the gloo backend with CPU tensors for tests
(the traversal itself needs the GPU; the plumbing does not).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def shard_range(n: int, rank: int, world: int, align: int = 64) -> tuple[int, int]:
    """Contiguous shard [lo, hi) of n points for `rank`, boundaries on multiples
    of `align` (a warp tile: 64 points for BH, 32 otherwise) so every warp of a
    shard is a warp of the unsharded launch: sharded results are then
    bit-identical to one launch."""
    chunk = -(-n // world)
    chunk = -(-chunk // align) * align
    lo = min(rank * chunk, n)
    return lo, min(lo + chunk, n)


def _wire(device, group=None):
    """Device the collectives run on: the tensors' own device under NCCL;
    host memory under gloo (used to exercise the multi-rank flow without
    NVLink, e.g. several ranks on one GPU in tests)."""
    return torch.device("cpu") if dist.get_backend(group) == "gloo" else torch.device(device)


def broadcast_blob(blob: np.ndarray | None, device, src: int = 0, group=None) -> torch.Tensor:
    """Broadcast a packed tree blob (uint8) from `src`; returns it on `device`
    on every rank.  The size travels first as an int64."""
    rank = dist.get_rank(group)
    wire = _wire(device, group)
    size = torch.zeros(1, dtype=torch.int64, device=wire)
    if rank == src:
        size[0] = int(blob.size)
    dist.broadcast(size, src, group=group)
    if rank == src:
        buf = torch.from_numpy(np.ascontiguousarray(blob)).to(wire)
    else:
        buf = torch.empty(int(size.item()), dtype=torch.uint8, device=wire)
    dist.broadcast(buf, src, group=group)
    return buf.to(device)


def broadcast_tree(host_tree, device, src: int = 0, group=None):
    """Rank `src` passes its HostTree (others pass None); every rank gets a
    device Tree adopted from the broadcast blob (tt_tree_from_blob, DEVICE)."""
    from .tt import tt_tree_from_blob  # GPU path only
    blob = host_tree.pack() if dist.get_rank(group) == src else None
    buf = broadcast_blob(blob, device, src, group)
    return tt_tree_from_blob(buf)


def broadcast_device_tree(tree, device, src: int = 0, group=None):
    """Rank `src` passes a device Tree (e.g. built on the GPU with
    tt_build_oct_device), the others None: its packed blob is copied device
    to device into a send buffer (tt_tree_copy_blob), broadcast as bytes and
    adopted on the other ranks (tt_tree_from_blob, DEVICE).  Rank `src`
    keeps its own tree."""
    from .tt import tt_tree_copy_blob, tt_tree_from_blob  # GPU path only
    rank = dist.get_rank(group)
    wire = _wire(device, group)
    size = torch.zeros(1, dtype=torch.int64, device=wire)
    if rank == src:
        size[0] = int(tree.device_bytes)
    dist.broadcast(size, src, group=group)
    if rank == src:
        buf = tt_tree_copy_blob(tree).to(wire)
    else:
        buf = torch.empty(int(size.item()), dtype=torch.uint8, device=wire)
    dist.broadcast(buf, src, group=group)
    return tree if rank == src else tt_tree_from_blob(buf.to(device))


def allgather_rows(full: torch.Tensor, world: int, group=None) -> torch.Tensor:
    """In-place all-gather of equal-size contiguous row shards of `full`
    (rank r owns rows shard_range(n, r, world)); needs n % (64 * world) == 0."""
    n = full.shape[0]
    if n % (64 * world):
        raise ValueError("allgather_rows needs equal warp-aligned shards (n % (64*world) == 0)")
    rank = dist.get_rank(group)
    lo, hi = shard_range(n, rank, world)
    wire = _wire(full.device, group)
    if wire == full.device:
        dist.all_gather_into_tensor(full, full[lo:hi], group=group)  # in place
    else:
        staged = full.to(wire)
        dist.all_gather_into_tensor(staged, staged[lo:hi].clone(), group=group)
        full.copy_(staged)
    return full


def balanced_ranges(costs: torch.Tensor, world: int, align: int = 64) -> list[tuple[int, int]]:
    """Contiguous warp-aligned shards [lo, hi) of len(costs) points with
    (nearly) equal total cost: the boundaries are where the prefix sum of the
    per-point costs crosses r/world of the total, rounded to `align` points
    (SURVEY §8(e)'s cost-weighted split; e.g. costs = the visit counts of a
    previous pass).  Deterministic: every rank computes the same ranges from
    the same costs."""
    n = int(costs.numel())
    c = torch.cumsum(costs.detach().to(torch.float64).cpu(), 0)
    total = float(c[-1]) if n else 0.0
    bounds = [0]
    for r in range(1, world):
        k = int(torch.searchsorted(c, torch.tensor([total * r / world], dtype=torch.float64)).item())
        k = min(max(int(round(k / align)) * align, bounds[-1]), n)
        bounds.append(k)
    bounds.append(n)
    return [(bounds[r], bounds[r + 1]) for r in range(world)]


def allgather_rows_var(full: torch.Tensor, ranges: list[tuple[int, int]], group=None) -> torch.Tensor:
    """All-gather of contiguous row shards of `full` whose lengths differ
    (rank r owns rows ranges[r]): every rank contributes its rows padded to
    the longest shard, one all_gather_into_tensor, then each shard is copied
    to its place.  In place on `full`."""
    world = len(ranges)
    rank = dist.get_rank(group)
    lens = [hi - lo for lo, hi in ranges]
    mx = max(lens)
    wire = _wire(full.device, group)
    row = full.shape[1:]
    mine = torch.zeros((mx, *row), dtype=full.dtype, device=wire)
    lo, hi = ranges[rank]
    mine[:hi - lo] = full[lo:hi].to(wire)
    gathered = torch.empty((world * mx, *row), dtype=full.dtype, device=wire)
    dist.all_gather_into_tensor(gathered, mine, group=group)
    for r, (a, b) in enumerate(ranges):
        if r != rank and b > a:
            full[a:b] = gathered[r * mx:r * mx + (b - a)].to(full.device)
    return full


def max_over_ranks(x: float, device, group=None) -> float:
    t = torch.tensor([x], dtype=torch.float64, device=_wire(device, group))
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
