"""Per-stage timing of one BH time step (simulate vs simulate_sharded)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import ttgen  # noqa: E402
import paper_conf_sc_goldfarbjk13_b200 as P  # noqa: E402
from paper_conf_sc_goldfarbjk13_b200 import nbody  # noqa: E402

n = 1_000_000
b = ttgen.plummer(n, 2)
v = ttgen.plummer_velocities(b, 1002)
B, V = torch.from_numpy(b).cuda(), torch.from_numpy(v).cuda()
ids = torch.arange(n, dtype=torch.int32, device="cuda")


def t(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        r = fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps * 1e3, r


ms, tree = t(lambda: P.tt_build_oct_device(B))
print(f"build {ms:.2f} ms")
ms, perm = t(lambda: P.tt_sort_points(tree, B))
print(f"sort {ms:.2f} ms")
acc = torch.empty_like(B)
ms, _ = t(lambda: P.tt_traverse_bh(tree, B, 0.5, 0.05, out=acc, order=perm))
print(f"traverse {ms:.2f} ms")
ms, _ = t(lambda: P.tt_traverse_bh(tree, B, 0.5, 0.05, out=acc, order=perm[0:n]))
print(f"traverse(slice) {ms:.2f} ms")
xo, vo, io = torch.empty_like(B), torch.empty_like(V), torch.empty_like(ids)
ms, _ = t(lambda: nbody.tt_kick_drift_permuted(B, V, acc, perm, 1e-3, 1e-3, xo, vo, ids, io))
print(f"kick_drift_permuted {ms:.2f} ms")
Bs, Vs = B[perm.long()].contiguous(), V[perm.long()].contiguous()
ms, tree2 = t(lambda: P.tt_build_oct_device(Bs))
print(f"build (sorted input) {ms:.2f} ms")
ms, perm2 = t(lambda: P.tt_sort_points(tree2, Bs))
print(f"sort (sorted input) {ms:.2f} ms")
ms, _ = t(lambda: P.tt_traverse_bh(tree2, Bs, 0.5, 0.05, out=acc, order=perm2))
print(f"traverse (sorted input) {ms:.2f} ms")
ms, _ = t(lambda: nbody.simulate(B, V, 1, 1e-3, acc=acc))
print(f"simulate 1 step {ms:.2f} ms")
ms, _ = t(lambda: nbody.simulate_sharded(Bs, Vs, ids, 1, 1e-3, final_kick=False))
print(f"simulate_sharded 1 step {ms:.2f} ms")
