"""Small launches of every kernel and mode, for compute-sanitizer (memcheck /
racecheck / synccheck) on the GPU box."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import ttgen
import paper_conf_sc_goldfarbjk13_b200 as P

dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()  # noqa: E731
b = ttgen.plummer(3000, 2)
t = P.tt_tree_upload(P.build_oct(b))
bd = dev(b)
perm = P.tt_sort_points(t, bd)
for m in ("lockstep", "independent", "auto"):
    P.tt_traverse_bh(t, bd, 0.5, 0.05, order=perm, mode=m, stats=P.Stats.alloc(len(b), "cuda"))
p = ttgen.uniform(2000, 3, 1)
t = P.tt_tree_upload(P.build_kd(p, 1))
for m in ("lockstep", "independent"):
    P.tt_traverse_pc(t, dev(p), 0.1, order=P.tt_sort_points(t, dev(p)), mode=m)
p7 = ttgen.gaussian_mixture(3000, 7, 3)
t = P.tt_tree_upload(P.build_kd(p7, 8))
for m in ("lockstep", "independent", "auto"):
    P.tt_traverse_knn(t, dev(p7[:1000]), 8, mode=m, stats=P.Stats.alloc(1000, "cuda"))
for a in (3, 12, 33):  # dynamic L->N switch: in-place warp -> lane stack conversion
    P.tt_traverse_knn(t, dev(p7[:1000]), 8, mode="lockstep", switch_below=a, stats=P.Stats.alloc(1000, "cuda"))
tn = P.tt_tree_upload(P.build_nn(p7))
for m in ("lockstep", "independent", "auto"):
    q = dev(p7[:1000] + 0.01)
    P.tt_traverse_nn(tn, q, order=P.tt_sort_points(tn, q), mode=m, stats=P.Stats.alloc(1000, "cuda"))
p16 = ttgen.gaussian_mixture(2000, 16, 5)
t = P.tt_tree_upload(P.build_vp(p16))
for m in ("lockstep", "independent", "auto"):
    P.tt_traverse_vp(t, dev(p16[:500]), mode=m, stats=P.Stats.alloc(500, "cuda"))
torch.cuda.synchronize()
print("sanitize workload done")
