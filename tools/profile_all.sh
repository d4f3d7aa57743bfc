#!/bin/bash
# Run on the GPU box (gpurun): launch list of the bench command + one
# `ncu --set full` capture of each traversal kernel (configs[0..4]).  Outputs in gpurun_out/.
set -x
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_bh.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-strong > /dev/null 2>&1
# <workload> <mode> <launches to skip: BH: the warm-up launch on a throwaway tree, the group-build trigger, the stats pass and the independent-mode stats pass of Table 2; others: the two stats passes; any larger count lands on a later, identical non-stats launch> <kernel>
for spec in "bh auto 5 bh_group_kernel" "pc auto 1 pc_split_kernel" "knn auto 3 knn_kernel" "vp auto 3 vp_kernel" \
            "vp independent 1 vp_kernel" "knn independent 1 knn_kernel" "nn auto 3 nn_kernel" \
            "bh16m auto 5 bh_group_kernel" "knn16m auto 3 knn_kernel"; do
  set -- $spec
  w=$1; m=$2; sk=$3; k=$4
  extra=""
  case $w in *16m) extra="--device-build";; esac
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$k -s $sk -c 1 \
      -o gpurun_out/prof_${w}_${m} python bench.py --workload $w --mode $m --steps 1 --warmup 1 \
      --no-cpu-baseline --no-e2e --no-chase --no-strong $extra > gpurun_out/ncu_${w}_${m}.log 2>&1
done
ls -la gpurun_out
