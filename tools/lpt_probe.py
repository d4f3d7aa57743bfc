"""Upper bound of tile scheduling for BH configs[1]: traversal time with the
in-order Hilbert tiles vs the same tiles dispatched longest-first by their
TRUE cost (warp steps from a stats pass) -- an oracle schedule no cheap
estimator reaches.  Prints both medians (CUDA events, L2 flushed)."""
import os
import statistics
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import ttgen  # noqa: E402
import paper_conf_sc_goldfarbjk13_b200 as P  # noqa: E402

c = ttgen.CONFIGS["bh_1m_plummer"]
b = ttgen.plummer(c["n"], c["seed"])
tree = P.tt_tree_upload(P.build_oct(b))
bd = torch.from_numpy(b).cuda()
perm = P.tt_sort_points(tree, bd)
n = len(b)
T = 64
st = P.Stats.alloc(n, "cuda")
P.tt_traverse_bh(tree, bd, c["theta"], c["eps"], order=perm, stats=st)
torch.cuda.synchronize()
tiles = (n + T - 1) // T
cost = st.warp_steps[:tiles].to(torch.float64).cpu().numpy()
idx = np.argsort(-cost, kind="stable")
pad = np.concatenate([perm.cpu().numpy(), -np.ones(tiles * T - n, dtype=np.int32)]).reshape(tiles, T)
lpt = pad[idx].reshape(-1)
lpt = torch.from_numpy(lpt[lpt >= 0].astype(np.int32)).cuda()  # the one partial tile moves to the end
flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
out = torch.empty((n, 4), dtype=torch.float32, device="cuda")


def timed(order, reps=15):
    ms = []
    for _ in range(3):
        P.tt_traverse_bh(tree, bd, c["theta"], c["eps"], out=out, order=order)
    for _ in range(reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        P.tt_traverse_bh(tree, bd, c["theta"], c["eps"], out=out, order=order)
        e1.record()
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    return statistics.median(ms)


for rep in range(2):
    print(f"in-order {timed(perm):.4f} ms   true-cost LPT {timed(lpt):.4f} ms")
print(f"tile cost: mean {cost.mean():.0f}, max {cost.max():.0f}, tiles {tiles}")
