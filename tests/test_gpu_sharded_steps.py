"""NEXT-4 multi-GPU time stepping on the GPU: the gathered
kick-drift is the fp32 update; a one-rank sharded run equals the in-place
simulate(); a two-rank run (two processes on cuda:0, gloo wire -- the box has
one GPU) is bit-identical to one rank, so per-body results do not depend on
the number of ranks."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import ttgen

pytestmark = pytest.mark.gpu

N, STEPS, DT = 64 * 2 * 160, 3, 1e-3  # 20,480 bodies: 2 equal warp-aligned shards


def dev(a, dtype=torch.float32):
    return torch.from_numpy(np.ascontiguousarray(a)).to("cuda", dtype)


def test_kick_drift_permuted_is_the_gathered_fp32_update():
    from paper_conf_sc_goldfarbjk13_b200.nbody import tt_kick_drift_permuted
    rng = np.random.default_rng(7)
    n = 3000
    x, v, a = (rng.standard_normal((n, 4)).astype(np.float32) for _ in range(3))
    ids = rng.permutation(n).astype(np.int32)
    perm = rng.permutation(n)[:1234].astype(np.int32)
    xo, vo = torch.zeros(1234, 4, device="cuda"), torch.zeros(1234, 4, device="cuda")
    io = torch.zeros(1234, dtype=torch.int32, device="cuda")
    tt_kick_drift_permuted(dev(x), dev(v), dev(a), dev(perm, torch.int32), 0.01, 0.02, xo, vo,
                           dev(ids, torch.int32), io)
    # plain fp32 reference, one rounding per operation (torch CPU elementwise)
    X, V, A = torch.from_numpy(x)[perm], torch.from_numpy(v)[perm], torch.from_numpy(a)[perm]
    v1 = V[:, :3] + A[:, :3] * 0.01
    x1 = X[:, :3] + v1 * 0.02
    assert torch.equal(vo.cpu()[:, :3], v1) and torch.equal(xo.cpu()[:, :3], x1)
    assert torch.equal(xo.cpu()[:, 3], X[:, 3]) and torch.equal(vo.cpu()[:, 3], V[:, 3])
    assert np.array_equal(io.cpu().numpy(), ids[perm])


def _initial():
    b = ttgen.plummer(N, seed=230)
    v = ttgen.plummer_velocities(b, seed=231)
    return b, v


def test_sharded_one_rank_equals_simulate():
    from paper_conf_sc_goldfarbjk13_b200 import nbody
    b, v = _initial()
    B, V = dev(b), dev(v)
    nbody.simulate(B, V, STEPS, DT)
    x, u, ids = nbody.simulate_sharded(dev(b), dev(v), torch.arange(N, dtype=torch.int32, device="cuda"), STEPS, DT)
    ids = ids.cpu().numpy()
    assert np.array_equal(np.sort(ids), np.arange(N))
    xs = np.empty_like(b)
    us = np.empty_like(v)
    xs[ids], us[ids] = x.cpu().numpy(), u.cpu().numpy()
    assert np.array_equal(xs, B.cpu().numpy())
    assert np.array_equal(us, V.cpu().numpy())


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        import torch.distributed as dist
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        from paper_conf_sc_goldfarbjk13_b200 import nbody
        b, v = _initial()
        x, u, ids = nbody.simulate_sharded(dev(b), dev(v), torch.arange(N, dtype=torch.int32, device="cuda"),
                                           STEPS, DT)
        q.put((rank, x.cpu().numpy(), u.cpu().numpy(), ids.cpu().numpy()))
        dist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e), None, None))


def test_two_ranks_bit_identical_to_one():
    from paper_conf_sc_goldfarbjk13_b200 import nbody
    b, v = _initial()
    x1, u1, i1 = nbody.simulate_sharded(dev(b), dev(v), torch.arange(N, dtype=torch.int32, device="cuda"),
                                        STEPS, DT)
    x1, u1, i1 = x1.cpu().numpy(), u1.cpu().numpy(), i1.cpu().numpy()
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, x, u, ids in res:
        assert not isinstance(x, str), x
        assert np.array_equal(ids, i1), rank
        assert np.array_equal(x, x1) and np.array_equal(u, u1), rank


@pytest.mark.parametrize("n,dup", [(1, 0), (3001, 0), (20011, 12), (1_000_000, 0)])
def test_build_tree_order_equals_oracle(n, dup):
    """tt_build_oct_device_order's order = the bodies in leaf preorder: the
    oracle builder's tree order (R8a / R9: depth-32 buckets by index), and a
    traversal in that order matches the oracle."""
    import oracle
    import paper_conf_sc_goldfarbjk13_b200 as P
    b = ttgen.plummer(n, seed=500 + n % 97)
    if dup:
        b[10:10 + dup, :3] = b[2, :3]
    ot = oracle.build_oct(b)
    tree, order = P.tt_build_oct_device_order(dev(b))
    assert np.array_equal(order.cpu().numpy(), ot.tree_order())
    if n == 1:
        assert np.all(P.tt_traverse_bh(tree, dev(b), 0.5, 0.05, order=order).cpu().numpy() == 0)
    elif n <= 20011:
        acc = P.tt_traverse_bh(tree, dev(b), 0.5, 0.05, order=order).cpu().numpy()
        ref = oracle.bh(ot, b, 0.5, 0.05, self_ids=np.arange(n)).out[0]
        err = np.linalg.norm(acc[:, :3] - ref, axis=1) / np.linalg.norm(ref, axis=1)
        assert err.max() <= 1e-4
