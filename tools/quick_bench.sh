#!/bin/bash
# quick timing of several workloads/modes -> gpurun_out/quick.jsonl
for spec in "$@"; do
  set -- $spec
  timeout 600 python bench.py --workload $1 --mode $2 --steps ${3:-3} --warmup 2 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
done
