"""BH tail experiment: per-tile lockstep steps, and the kernel time with tiles
dispatched in-order vs longest-first by their TRUE cost (an upper bound on
what a cost-estimated schedule can gain) and by cheap proxies.
  python tools/bh_tail.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_goldfarbjk13_b200 as P  # noqa: E402

dev = torch.device("cuda:0")
w = bench.make_workload("bh", 1)
c = w["cfg"]
tree = P.tt_tree_upload(bench.host_tree(P, "bh", w))
q = torch.from_numpy(w["queries"][: w["m"]]).to(dev)
m = q.shape[0]
keys = torch.empty(m, dtype=torch.int64, device=dev)
order = P.tt_sort_points(tree, q, keys=keys)
st = P.Stats.alloc(m, dev)
P.tt_traverse_bh(tree, q, c["theta"], c["eps"], order=order, stats=st)
torch.cuda.synchronize()
T = 64
nt = (m + T - 1) // T
s = st.warp_steps.double().cpu().numpy()[:nt]  # BH stats are per 64-body tile
print("tiles", nt, "mean steps", s.mean(), "cv", s.std() / s.mean())


def time_order(o, reps=20):
    out = torch.empty(m, 4, device=dev)
    for _ in range(3):
        P.tt_traverse_bh(tree, q, c["theta"], c["eps"], order=o, out=out)
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    ts = []
    for _ in range(reps):
        ev[0].record()
        P.tt_traverse_bh(tree, q, c["theta"], c["eps"], order=o, out=out)
        ev[1].record()
        torch.cuda.synchronize()
        ts.append(ev[0].elapsed_time(ev[1]))
    return np.median(ts)


def tile_perm(tile_rank):
    full = m // T
    idx = np.argsort(tile_rank[:full], kind="stable")
    o = order.cpu().numpy()
    blocks = o[: full * T].reshape(full, T)[idx].reshape(-1)
    return torch.from_numpy(np.concatenate([blocks, o[full * T:]])).to(dev)


base = time_order(order)
print(f"in-order            {base:.3f} ms")
print(f"true longest-first  {time_order(tile_perm(-s)):.3f} ms")
ht = bench.host_tree(P, "bh", w)
body, level = ht.array("body"), ht.array("level")
leaf_level = np.zeros(m, np.int64)
leaf_level[body[body >= 0]] = level[body >= 0]
o = order.cpu().numpy()
full = m // T
def report(name, key_sorted_bodies, agg):
    kt = agg(key_sorted_bodies[: full * T].reshape(full, T), axis=1)
    kt = np.concatenate([kt, [np.inf] * (nt - full)])
    print(f"corr(steps, {name}) {np.corrcoef(s[:full], kt[:full])[0, 1]:+.3f}  "
          f"{name} ascending {time_order(tile_perm(kt)):.3f} ms")
report("-max leaf level", -leaf_level[o], np.min)
report("-mean leaf level", -leaf_level[o].astype(float), np.mean)
bodies = w["queries"][: w["m"]]
com = ht.array("com")[0, :3]
r = np.linalg.norm(bodies[o, :3] - com, axis=1)
report("min r to root com", r, np.min)
report("mean r to root com", r, np.mean)
report("-min r (cheap first)", -r, np.min)
rng = np.random.default_rng(0)
print(f"random tile order {time_order(tile_perm(rng.permutation(nt).astype(float))):.3f} ms")
print(f"reversed tile order {time_order(tile_perm(-np.arange(nt, dtype=float))):.3f} ms")
print(f"in-order again {time_order(order):.3f} ms")
