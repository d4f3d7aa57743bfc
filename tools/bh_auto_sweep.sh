#!/bin/bash
# BH AUTO threshold sweep (shared octant levels), sorted and unsorted
mkdir -p gpurun_out; rm -f gpurun_out/bh_sweep.jsonl
for a in 0 1 2 3 4 5 6; do
  timeout 600 python bench.py --workload bh --mode auto --auto-min-depth $a --steps 5 --warmup 3 --no-cpu-baseline --no-e2e >> gpurun_out/bh_sweep.jsonl 2>>gpurun_out/err.log
done
for a in 1 2 3 4 6; do
  timeout 600 python bench.py --workload bh --mode auto --unsorted --auto-min-depth $a --steps 3 --warmup 2 --no-cpu-baseline --no-e2e >> gpurun_out/bh_sweep.jsonl 2>>gpurun_out/err.log
done
python - <<'PY'
import json
for l in open("gpurun_out/bh_sweep.jsonl"):
    d = json.loads(l); c = d["config"]
    print(f'T={c["auto_min_depth"]} sorted={c["sorted"]!s:5s} kern={d["traverse_ms"]:8.3f} ms lock={d["lockstep_warp_fraction"]:.3f}')
PY
