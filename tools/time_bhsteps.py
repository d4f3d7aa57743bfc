import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import ttgen
import paper_conf_sc_goldfarbjk13_b200 as P
from paper_conf_sc_goldfarbjk13_b200 import nbody
b = ttgen.plummer(1_000_000, 2); v = ttgen.plummer_velocities(b, 1002)
B = torch.from_numpy(b).cuda(); V = torch.from_numpy(v).cuda()
acc, _ = nbody.forces(B, 0.5, 0.05)
for it in range(6):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    P.tt_kick_drift(B, V, acc, 1e-3, 1e-3); torch.cuda.synchronize(); t1 = time.perf_counter()
    tree = P.tt_build_oct_device(B); torch.cuda.synchronize(); t2 = time.perf_counter()
    perm = P.tt_sort_points(tree, B); torch.cuda.synchronize(); t3 = time.perf_counter()
    P.tt_traverse_bh(tree, B, 0.5, 0.05, out=acc, order=perm); torch.cuda.synchronize(); t4 = time.perf_counter()
    del tree; torch.cuda.synchronize(); t5 = time.perf_counter()
    print(f"kick {1e3*(t1-t0):.2f} build {1e3*(t2-t1):.2f} sort {1e3*(t3-t2):.2f} force {1e3*(t4-t3):.2f} free {1e3*(t5-t4):.2f} ms")
