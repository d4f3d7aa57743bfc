#!/bin/bash
# ncu --set full captures of the configs[4] traversal kernels (16M points)
mkdir -p gpurun_out
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:knn_kernel -s 1 -c 1 \
    -o gpurun_out/prof_knn16m python bench.py --workload knn16m --steps 1 --warmup 1 \
    --no-cpu-baseline --no-e2e --no-chase --device-build > gpurun_out/ncu_knn16m.log 2>&1
echo "knn16m ncu rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bh_group_kernel -s 1 -c 1 \
    -o gpurun_out/prof_bh16m python bench.py --workload bh16m --steps 1 --warmup 1 \
    --no-cpu-baseline --no-e2e --no-chase --device-build > gpurun_out/ncu_bh16m.log 2>&1
echo "bh16m ncu rc=$?"
