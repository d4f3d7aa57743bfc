#!/bin/bash
# A/B of the longest-first tile schedule -> gpurun_out/quick.jsonl
for w in "$@"; do
  timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-schedule 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
  timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
done
