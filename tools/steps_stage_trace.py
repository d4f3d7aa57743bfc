"""Per-step, per-stage trace of the NEXT-4 time step (nbody.simulate_sharded's
half step, one rank): device time of build / traverse / kick-drift (CUDA
events) and host time of each call, to locate run-to-run outliers."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import ttgen  # noqa: E402
import paper_conf_sc_goldfarbjk13_b200 as P  # noqa: E402
from paper_conf_sc_goldfarbjk13_b200 import nbody  # noqa: E402

c = ttgen.CONFIGS["bh_1m_plummer"]
n = c["n"] // 64 * 64
b = ttgen.plummer(n, c["seed"])
v = ttgen.plummer_velocities(b, c["seed"] + 1000)
x, vel = torch.from_numpy(b).cuda(), torch.from_numpy(v).cuda()
ids = torch.arange(n, dtype=torch.int32, device="cuda")
xo, vo, io = torch.empty_like(x), torch.empty_like(vel), torch.empty_like(ids)
acc = torch.empty_like(x)
order = torch.empty(n, dtype=torch.int32, device="cuda")
s = torch.cuda.current_stream()
rows = []
for step in range(40):
    E = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    h = []
    t0 = time.perf_counter()
    E[0].record(s)
    tree, perm = P.tt_build_oct_device_order(x, order)
    h.append(time.perf_counter())
    E[1].record(s)
    P.tt_traverse_bh(tree, x, c["theta"], c["eps"], out=acc, order=perm)
    h.append(time.perf_counter())
    E[2].record(s)
    nbody.tt_kick_drift_permuted(x, vel, acc, perm, 1e-3, 1e-3, xo, vo, ids, io)
    E[3].record(s)
    h.append(time.perf_counter())
    del tree
    h.append(time.perf_counter())
    torch.cuda.synchronize()
    h.append(time.perf_counter())
    x, xo, vel, vo, ids, io = xo, x, vo, vel, io, ids
    d = [E[i].elapsed_time(E[i + 1]) for i in range(3)]
    hh = [1e3 * (h[0] - t0)] + [1e3 * (h[i + 1] - h[i]) for i in range(len(h) - 1)]
    rows.append((step, d, hh, 1e3 * (h[-1] - t0)))
print("step | dev build trav kick | host build trav kick free sync | total host")
for st, d, hh, tot in rows:
    print(f"{st:3d} | " + " ".join(f"{x:6.2f}" for x in d) + " | " + " ".join(f"{x:6.2f}" for x in hh) + f" | {tot:6.2f}")
