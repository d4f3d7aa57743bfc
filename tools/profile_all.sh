#!/bin/bash
# Run on the GPU box (gpurun): launch list of the bench command + one
# `ncu --set full` capture of each traversal kernel.  Outputs in gpurun_out/.
set -x
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_bh.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
for spec in "bh auto 1000000" "pc auto 10000" "knn auto 1000000" "vp auto 1000000" "vp independent 1000000" "knn independent 1000000" "nn auto 1000000"; do
  set -- $spec
  w=$1; m=$2; n=$3
  ncu --set full --clock-control none --import-source on -k regex:$( [ $w = bh ] && echo bh_group_kernel || echo ${w}_kernel ) -s 1 -c 1 \
      -o gpurun_out/prof_${w}_${m} python bench.py --workload $w --mode $m --steps 1 --warmup 1 \
      --no-cpu-baseline --no-e2e --points-per-rank $n > gpurun_out/ncu_${w}_${m}.log 2>&1
done
ls -la gpurun_out
