"""Per-step timing of nbody.simulate_sharded (BH time stepping) for the
default BH kernel and the per-node ropes variant."""
import sys
import torch
import ttgen
import paper_conf_sc_goldfarbjk13_b200 as P
from paper_conf_sc_goldfarbjk13_b200 import nbody

c = ttgen.CONFIGS["bh_1m_plummer"]
b = ttgen.plummer(c["n"], c["seed"])
v = ttgen.plummer_velocities(b, c["seed"] + 1000)
orig = nbody.tt_traverse_bh
for variant in ("autoropes", "ropes", "autoropes"):
    nbody.tt_traverse_bh = (lambda *a, _v=variant, **k: orig(*a, variant=_v, **k))
    B, V = torch.from_numpy(b).cuda(), torch.from_numpy(v).cuda()
    ids = torch.arange(len(b), dtype=torch.int32, device="cuda")
    ts = []
    for i in range(14):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        B, V, ids = nbody.simulate_sharded(B, V, ids, 1, 1e-3, c["theta"], c["eps"], final_kick=False)
        e1.record()
        torch.cuda.synchronize()
        ts.append(round(e0.elapsed_time(e1), 2))
    print(variant, ts, flush=True)
