"""Per-step trace of the bhsteps bench loop (device event time and host
enqueue time of every step) to locate run-to-run outliers."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import ttgen
from paper_conf_sc_goldfarbjk13_b200 import nbody
c = ttgen.CONFIGS["bh_1m_plummer"]
b = ttgen.plummer(c["n"], c["seed"]); v = ttgen.plummer_velocities(b, c["seed"] + 1000)
B, V = torch.from_numpy(b).cuda(), torch.from_numpy(v).cuda()
ids = torch.arange(c["n"], dtype=torch.int32, device="cuda")
for _ in range(3):
    B, V, ids = nbody.simulate_sharded(B, V, ids, 1, 1e-3, c["theta"], c["eps"], final_kick=False)
torch.cuda.synchronize()
for rep in range(3):
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(10)]
    host = []
    for i in range(10):
        t0 = time.perf_counter()
        evs[i][0].record()
        B, V, ids = nbody.simulate_sharded(B, V, ids, 1, 1e-3, c["theta"], c["eps"], final_kick=False)
        evs[i][1].record()
        host.append(1e3 * (time.perf_counter() - t0))
    torch.cuda.synchronize()
    print("dev ", " ".join(f"{a.elapsed_time(b_):6.1f}" for a, b_ in evs))
    print("host", " ".join(f"{h:6.1f}" for h in host))
