"""Small launches of every kernel, variant and mode, for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck) on the GPU box
(tools/sanitize_all.sh).  Prints the hash of the CUDA sources it ran."""
import glob
import hashlib
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import ttgen
import paper_conf_sc_goldfarbjk13_b200 as P

h = hashlib.sha256()
for f in sorted(glob.glob(os.path.join(ROOT, "paper_conf_sc_goldfarbjk13_b200", "csrc", "*"))):
    h.update(open(f, "rb").read())
print("csrc sha256", h.hexdigest()[:16], flush=True)

dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()  # noqa: E731
S = lambda n, **kw: P.Stats.alloc(n, "cuda", **kw)  # noqa: E731

# ---- BH: every walk, every mode; eps = 0, no-self ids, foreign ids, buckets
b = ttgen.plummer(3000, 2)
b[100:140, :3] = b[5, :3]  # a depth-32 bucket of 41 coincident bodies (wide groups)
for t in (P.tt_tree_upload(P.build_oct(b)), P.tt_build_oct_device(dev(b))):
    bd = dev(b)
    perm = P.tt_sort_points(t, bd)
    for order in (perm, None):
        for m in ("lockstep", "independent", "auto"):
            for v in ("autoropes", "ropes", "stack"):
                P.tt_traverse_bh(t, bd, 0.5, 0.05, order=order, mode=m, variant=v, stats=S(len(b), hashes=True))
                P.tt_traverse_bh(t, bd, 0.5, 0.05, order=order, mode=m, variant=v)
    P.tt_traverse_bh(t, bd, 0.5, 0.05, mode="independent", variant="recursive", stats=S(len(b), hashes=True))
    P.tt_traverse_bh(t, bd, 0.5, 0.0, order=perm, mode="lockstep")                      # eps = 0
    P.tt_traverse_bh(t, bd, 0.0, 0.05, order=perm, mode="lockstep")                     # theta = 0
    ids = torch.full((len(b),), -1, dtype=torch.int32, device="cuda")
    P.tt_traverse_bh(t, bd * 0.5, 0.5, 0.0, self_ids=ids, order=perm, mode="lockstep")  # no self leaf
    P.tt_traverse_bh(t, bd, 0.5, 0.05, self_ids=torch.roll(torch.arange(len(b), dtype=torch.int32,
                                                                         device="cuda"), 1), mode="lockstep")
b2 = ttgen.plummer(3000, 7)
t2 = P.tt_tree_upload(P.build_oct(b2))  # narrow tree (no bucket)
P.tt_traverse_bh(t2, dev(b2), 0.5, 0.05, order=P.tt_sort_points(t2, dev(b2)), stats=S(len(b2), hashes=True))
P.tt_traverse_bh(t2, dev(b2), 0.5, 0.05, order=P.tt_sort_points(t2, dev(b2)))
v = torch.zeros_like(dev(b2))
a = P.tt_traverse_bh(t2, dev(b2), 0.5, 0.05)
x = dev(b2)
P.tt_kick_drift(x, v, a, 1e-3, 1e-3)

# ---- PC: every variant and mode
p = ttgen.uniform(2000, 3, 1)
p[5:9] = p[1]
for t in (P.tt_tree_upload(P.build_kd(p, 1)), P.tt_build_kd_device(dev(p), 1)):
    pd = dev(p)
    for m in ("lockstep", "independent", "auto"):
        for vv in ("autoropes", "stack", "split"):
            P.tt_traverse_pc(t, pd, 0.1, order=P.tt_sort_points(t, pd), mode=m, variant=vv,
                             stats=S(len(p), hashes=True, point_tests=True))
            P.tt_traverse_pc(t, pd, 0.1, mode=m, variant=vv)
    P.tt_traverse_pc(t, pd, 0.1, mode="independent", variant="recursive", stats=S(len(p), hashes=True))

# ---- kNN: modes, dynamic switch, recursive, LPT schedule
p7 = ttgen.gaussian_mixture(3000, 7, 3)
for t in (P.tt_tree_upload(P.build_kd(p7, 8)), P.tt_build_kd_device(dev(p7), 8)):
    q = dev(p7[:1000])
    perm = P.tt_sort_points(t, q)
    sched = P.tt_schedule_tiles(t, q, perm)
    for m in ("lockstep", "independent", "auto"):
        for order in (sched, None):
            P.tt_traverse_knn(t, q, 8, order=order, mode=m, stats=S(1000, hashes=True, point_tests=True))
            P.tt_traverse_knn(t, q, 8, order=order, mode=m)
    for k in (1, 32):
        P.tt_traverse_knn(t, q, k, mode="auto")
    for sw in (3, 12, 33):  # dynamic L->N switch: in-place warp -> lane stack conversion
        P.tt_traverse_knn(t, q, 8, mode="lockstep", switch_below=sw, stats=S(1000, hashes=True))
    P.tt_traverse_knn(t, q, 8, mode="independent", variant="recursive", stats=S(1000, hashes=True))

# ---- NN (point-per-node kd)
for tn in (P.tt_tree_upload(P.build_nn(p7)), P.tt_build_nn_device(dev(p7))):
    q = dev(p7[:1000] + 0.01)
    for m in ("lockstep", "independent", "auto"):
        P.tt_traverse_nn(tn, q, order=P.tt_sort_points(tn, q), mode=m, stats=S(1000, hashes=True))
        P.tt_traverse_nn(tn, q, mode=m)

# ---- VP
p16 = ttgen.gaussian_mixture(2000, 16, 5)
for t in (P.tt_tree_upload(P.build_vp(p16)), P.tt_build_vp_device(dev(p16))):
    q = dev(p16[:500])
    perm = P.tt_sort_points(t, q)
    P.tt_schedule_tiles(t, q, perm)
    for m in ("lockstep", "independent", "auto"):
        P.tt_traverse_vp(t, q, order=perm, mode=m, stats=S(500, hashes=True))
        P.tt_traverse_vp(t, q, mode=m)
    P.tt_traverse_vp(t, q, mode="independent", variant="recursive", stats=S(500, hashes=True))

# ---- diagnostics
rec = P.chase_records(4096, "cuda")
P.tt_diag_chase(rec, 64, False)
P.tt_diag_chase(rec, 8, True)
torch.cuda.synchronize()
print("sanitize workload done")
