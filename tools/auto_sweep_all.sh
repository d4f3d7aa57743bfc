#!/bin/bash
# AUTO threshold sweep for kNN / VP / PC with the change-count coherence test
mkdir -p gpurun_out; rm -f gpurun_out/auto_sweep.jsonl
for w in knn vp; do
  for a in 2 4 6; do
    timeout 600 python bench.py --workload $w --mode auto --auto-min-depth $a --steps 3 --warmup 2 --no-cpu-baseline --no-e2e >> gpurun_out/auto_sweep.jsonl 2>>gpurun_out/err.log
    timeout 600 python bench.py --workload $w --mode auto --auto-min-depth $a --unsorted --steps 2 --warmup 1 --no-cpu-baseline --no-e2e >> gpurun_out/auto_sweep.jsonl 2>>gpurun_out/err.log
  done
  timeout 600 python bench.py --workload $w --mode lockstep --steps 3 --warmup 2 --no-cpu-baseline --no-e2e >> gpurun_out/auto_sweep.jsonl 2>>gpurun_out/err.log
done
for a in 2 4 255; do
  timeout 600 python bench.py --workload pc --mode auto --auto-min-depth $a --steps 20 --warmup 5 --no-cpu-baseline --no-e2e >> gpurun_out/auto_sweep.jsonl 2>>gpurun_out/err.log
done
python - <<'PY'
import json
for l in open("gpurun_out/auto_sweep.jsonl"):
    d = json.loads(l); c = d["config"]
    print(f'{c["workload"]:12s} {c["mode"]:9s} T={c["auto_min_depth"]} sorted={c["sorted"]!s:5s} kern={d["traverse_ms"]:9.3f} ms lock={d["lockstep_warp_fraction"]:.4f}')
PY
