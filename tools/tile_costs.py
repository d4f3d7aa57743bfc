"""Per-tile (warp) cost distribution and the tail it implies.

  python tools/tile_costs.py [bh knn vp]

For each workload: lockstep warp steps per 32-point tile (tt_stats
warp_steps), and the makespan of greedy in-order tile dispatch (the kernel's
atomic tile counter) over W resident warps, against the ideal sum/W and
against longest-first dispatch -- in units of warp steps.
"""
import heapq
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_goldfarbjk13_b200 as P  # noqa: E402


def greedy(costs, w):
    h = [0.0] * w
    for c in costs:
        t = heapq.heappop(h)
        heapq.heappush(h, t + c)
    return max(h)


def main(names):
    dev = torch.device("cuda:0")
    for name in names:
        w = bench.make_workload(name, 1)
        c = w["cfg"]
        tree = P.tt_tree_upload(bench.host_tree(P, name, w))
        q = torch.from_numpy(w["queries"][: w["m"]]).to(dev)
        m = q.shape[0]
        order = P.tt_sort_points(tree, q)
        st = P.Stats.alloc(m, dev)
        if name == "bh":
            P.tt_traverse_bh(tree, q, c["theta"], c["eps"], order=order, stats=st)
        elif name == "knn":
            P.tt_traverse_knn(tree, q, c["k"], order=order, stats=st)
        else:
            P.tt_traverse_vp(tree, q, order=order, stats=st)
        torch.cuda.synchronize()
        s = st.warp_steps.double().cpu().numpy()
        W = 148 * 32  # 4 CTAs x 8 warps per SM
        ideal = s.sum() / W
        inorder = greedy(s, W)
        lpt = greedy(np.sort(s)[::-1], W)
        rev = greedy(s[::-1], W)
        print(f"{name}: tiles={len(s)} mean={s.mean():.0f} p50={np.median(s):.0f} p99={np.percentile(s, 99):.0f} "
              f"max={s.max():.0f} cv={s.std() / s.mean():.2f} | makespan/ideal in-order={inorder / ideal:.3f} "
              f"reversed={rev / ideal:.3f} longest-first={lpt / ideal:.3f}")
        # cost vs position along the curve (deciles)
        dec = [s[i * len(s) // 10:(i + 1) * len(s) // 10].mean() / s.mean() for i in range(10)]
        print("   cost by decile of tile index:", " ".join(f"{x:.2f}" for x in dec))


if __name__ == "__main__":
    main(sys.argv[1:] or ["bh", "knn", "vp"])
