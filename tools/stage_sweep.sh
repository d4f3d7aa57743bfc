#!/bin/bash
# sweep the staged-top budget (TT_STAGE_BYTES) per workload -> gpurun_out/stage_sweep.jsonl
# usage: tools/stage_sweep.sh "vp 0 4096 16384" "knn 4096 32768"
for spec in "$@"; do
  set -- $spec
  w=$1; shift
  for b in "$@"; do
    echo "{\"stage_bytes\": $b}" >> gpurun_out/stage_sweep.jsonl
    TT_STAGE_BYTES=$b timeout 600 python bench.py --workload $w --steps 3 --warmup 2 --no-cpu-baseline --no-e2e \
      2>>gpurun_out/quick_err.log >> gpurun_out/stage_sweep.jsonl
  done
done
