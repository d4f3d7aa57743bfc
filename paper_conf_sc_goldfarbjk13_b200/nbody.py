"""Barnes-Hut time stepping on the GPU.

The paper's BH workload "ran our inputs for five timesteps": each
time step rebuilds the oct-tree from the moved bodies, recomputes centres of
mass, runs the force traversal and advances the bodies.  Every stage here is
a libtt call on the current stream (no host round trip besides the node
count the GPU build reads back):

    tt_build_oct_device -> tt_sort_points -> tt_traverse_bh -> tt_kick_drift

Integration is leapfrog kick-drift-kick, with consecutive half kicks merged:
  step 0:     kick(dt/2) + drift(dt), force
  step s > 0: kick(dt)   + drift(dt), force
  end:        kick(dt/2)
"""
from __future__ import annotations

import ctypes as C

import torch

from . import _lib as L
from ._lib import check
from .tt import _dev, _stream_handle, tt_build_oct_device, tt_sort_points, tt_traverse_bh


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


def forces(bodies: torch.Tensor, theta: float, eps: float, out: torch.Tensor | None = None, mode="auto",
           stats=None):
    """One force pass on the current positions: GPU build, sort, traverse."""
    tree = tt_build_oct_device(bodies)
    perm = tt_sort_points(tree, bodies)
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
