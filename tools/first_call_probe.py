import time, sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch, ttgen
import paper_conf_sc_goldfarbjk13_b200 as P
b = ttgen.plummer(1000000, 2)
t0=time.perf_counter(); tree = P.tt_tree_upload(P.build_oct(b)); torch.cuda.synchronize(); print("upload", time.perf_counter()-t0)
q = torch.from_numpy(b[:64]).cuda(); torch.cuda.synchronize()
for i in range(3):
    t0=time.perf_counter(); P.tt_traverse_bh(tree, q, 0.5, 0.05, mode="lockstep"); torch.cuda.synchronize(); print("traverse", i, time.perf_counter()-t0)
