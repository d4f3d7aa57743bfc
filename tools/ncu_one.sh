#!/bin/bash
# One `ncu --set full` capture of a traversal kernel (run under gpurun).
# usage: tools/ncu_one.sh <workload> <mode> <points> <tag>
mkdir -p gpurun_out
w=$1; m=$2; n=$3; tag=${4:-$1_$2}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${w}_kernel -s 1 -c 1 \
    -o gpurun_out/prof_${tag} python bench.py --workload $w --mode $m --steps 1 --warmup 1 \
    --no-cpu-baseline --no-e2e --points-per-rank $n > gpurun_out/ncu_${tag}.log 2>&1
echo "ncu rc=$?"
