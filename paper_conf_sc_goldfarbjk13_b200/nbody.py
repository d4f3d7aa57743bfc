"""Barnes-Hut time stepping on the GPU.

The paper's BH workload "ran our inputs for five timesteps": each
time step rebuilds the oct-tree from the moved bodies, recomputes centres of
mass, runs the force traversal and advances the bodies.  Every stage here is
a libtt call on the current stream (no host round trip besides the node
count the GPU build reads back):

    tt_build_oct_device_order -> tt_sort_points (Hilbert; or the build's tree order) -> tt_traverse_bh
    -> tt_kick_drift

Integration is leapfrog kick-drift-kick, with consecutive half kicks merged:
  step 0:     kick(dt/2) + drift(dt), force
  step s > 0: kick(dt)   + drift(dt), force
  end:        kick(dt/2)

``simulate_sharded`` is the multi-GPU form (one process per GPU, DESIGN.md
§9.1): every rank holds all bodies in the order of the last point sort and
rebuilds the same tree (the GPU build is deterministic, so no broadcast);
it computes forces and the kick-drift for its warp-aligned shard of the
sorted order only (tt_kick_drift_permuted writes the shard contiguously),
and one all-gather per state array is the step's exchange.  Per-body results
do not depend on the number of ranks.
"""
from __future__ import annotations

import ctypes as C

import torch

from . import _lib as L
from ._lib import check
from .tt import _dev, _stream_handle, tt_build_oct_device_order, tt_sort_points, tt_traverse_bh


def tt_kick_drift(bodies: torch.Tensor, vel: torch.Tensor, acc: torch.Tensor, dt_kick: float, dt_drift: float,
                  stream=None) -> None:
    """v += acc * dt_kick; x += v * dt_drift (fp32, in place, device rows of 4)."""
    for name, t in (("bodies", bodies), ("vel", vel), ("acc", acc)):
        _dev(t, torch.float32, name, 4)
        if t.shape != bodies.shape or not t.is_contiguous():
            raise ValueError(f"{name} must be a contiguous (n, 4) tensor like bodies")
    check(L.load().tt_kick_drift(bodies.data_ptr(), vel.data_ptr(), acc.data_ptr(), bodies.shape[0],
                                 float(dt_kick), float(dt_drift), C.c_void_p(_stream_handle(stream))),
          "tt_kick_drift")


def tt_kick_drift_permuted(bodies: torch.Tensor, vel: torch.Tensor, acc: torch.Tensor, perm: torch.Tensor,
                           dt_kick: float, dt_drift: float, bodies_out: torch.Tensor, vel_out: torch.Tensor,
                           ids: torch.Tensor | None = None, ids_out: torch.Tensor | None = None, stream=None) -> None:
    """Row j of (bodies_out, vel_out, ids_out) = row perm[j] of the inputs after
    v += acc * dt_kick; x += v * dt_drift (include/tt.h).  len(perm) rows."""
    for name, t in (("bodies", bodies), ("vel", vel), ("acc", acc), ("bodies_out", bodies_out),
                    ("vel_out", vel_out)):
        _dev(t, torch.float32, name, 4)
        if not t.is_contiguous():
            raise ValueError(f"{name} must be a contiguous (n, 4) tensor")
    _dev(perm, torch.int32, "perm")
    n = perm.numel()
    if bodies_out.shape[0] < n or vel_out.shape[0] < n:
        raise ValueError("outputs need len(perm) rows")
    ip = iop = None
    if ids is not None:
        _dev(ids, torch.int32, "ids")
        _dev(ids_out, torch.int32, "ids_out")
        ip, iop = ids.data_ptr(), ids_out.data_ptr()
    check(L.load().tt_kick_drift_permuted(bodies.data_ptr(), vel.data_ptr(), acc.data_ptr(), perm.data_ptr(), ip, n,
                                          float(dt_kick), float(dt_drift), bodies_out.data_ptr(), vel_out.data_ptr(),
                                          iop, C.c_void_p(_stream_handle(stream))), "tt_kick_drift_permuted")


# Traversal order of a time step: "sort" = tt_sort_points' Hilbert order
# (R18b), "build" = the tree (Morton) order the GPU build already produced --
# no extra sort, but less compact warp tiles: 5.25 vs 5.06 ms per 1M-body
# step (bench --workload bhsteps --steps-order, same box), so "sort".
DEFAULT_ORDER = "sort"


def forces(bodies: torch.Tensor, theta: float, eps: float, out: torch.Tensor | None = None, mode="auto",
           stats=None, order: str = DEFAULT_ORDER):
    """One force pass on the current positions: GPU build, sort, traverse."""
    tree, perm = tt_build_oct_device_order(bodies)
    if order == "sort":
        perm = tt_sort_points(tree, bodies, out=perm)
    acc = tt_traverse_bh(tree, bodies, theta, eps, out=out, order=perm, mode=mode, stats=stats)
    return acc, tree


def simulate(bodies: torch.Tensor, vel: torch.Tensor, steps: int, dt: float, theta: float = 0.5,
             eps: float = 0.05, mode="auto", acc: torch.Tensor | None = None):
    """Advance (bodies, vel) in place by `steps` leapfrog steps; returns the
    accelerations at the final positions."""
    if acc is None:
        acc, _ = forces(bodies, theta, eps, mode=mode)
    for s in range(steps):
        tt_kick_drift(bodies, vel, acc, dt * (0.5 if s == 0 else 1.0), dt)
        forces(bodies, theta, eps, out=acc, mode=mode)
    if steps:
        tt_kick_drift(bodies, vel, acc, 0.5 * dt, 0.0)
    return acc


def simulate_sharded(bodies: torch.Tensor, vel: torch.Tensor, ids: torch.Tensor, steps: int, dt: float,
                     theta: float = 0.5, eps: float = 0.05, mode="auto", group=None, final_kick: bool = True,
                     order: str = DEFAULT_ORDER):
    """Leapfrog KDK over `steps` steps with the bodies sharded across the ranks
    of `group` (None and no process group: one rank).  Every rank passes the
    same full (n, 4) bodies / vel and (n,) int32 ids; n must be a multiple of
    64 * world (warp-aligned equal shards).  Returns (bodies, vel, ids), full
    and identical on every rank, in the order of the last point sort (ids
    carries the original body index of every row).

    Step s: tree = build(x); perm = sort(x); a = force(x) for the rank's lanes
    perm[lo:hi]; kick(dt/2 if s == 0 else dt) + drift(dt) gathered through
    perm[lo:hi] into rows [lo, hi); all-gather.  With final_kick, one more
    force pass and the closing kick(dt/2) (drift 0).

    order: the traversal order of a step -- "build": the tree order the GPU
    build has already sorted the bodies into (no extra sort); "sort": the
    Hilbert order of tt_sort_points (R18b: more compact warp tiles, one more
    sort per step)."""
    import torch.distributed as dist
    from .parallel import allgather_rows, shard_range
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    n = bodies.shape[0]
    if n % (64 * world):
        raise ValueError("simulate_sharded needs n % (64 * world) == 0")
    lo, hi = shard_range(n, rank, world)
    x, v, i = bodies, vel, ids
    xo, vo, io = torch.empty_like(x), torch.empty_like(v), torch.empty_like(i)
    acc = torch.empty_like(x)
    order_buf = torch.empty(n, dtype=torch.int32, device=x.device)

    def half(dtk, dtd):
        nonlocal x, v, i, xo, vo, io
        tree, perm = tt_build_oct_device_order(x, order_buf)  # tree order from the build's sort
        if order == "sort":
            perm = tt_sort_points(tree, x, out=order_buf)
        mine = perm[lo:hi]
        tt_traverse_bh(tree, x, theta, eps, out=acc, order=mine, mode=mode)
        tt_kick_drift_permuted(x, v, acc, mine, dtk, dtd, xo[lo:hi], vo[lo:hi], i, io[lo:hi])
        if world > 1:
            allgather_rows(xo, world, group)
            allgather_rows(vo, world, group)
            _allgather_ids(io, world, group)
        x, xo = xo, x
        v, vo = vo, v
        i, io = io, i

    for s in range(steps):
        half(dt * (0.5 if s == 0 else 1.0), dt)
    if steps and final_kick:
        half(0.5 * dt, 0.0)
    return x, v, i


def _allgather_ids(ids: torch.Tensor, world: int, group=None):
    """In-place all-gather of an int32 (n,) id column (rows as for allgather_rows)."""
    from .parallel import allgather_rows
    allgather_rows(ids.view(-1, 1), world, group)
