#!/bin/bash
# ncu --set full of bh_group_kernel for abtest libs: tools/ncu_ab.sh A B ...
mkdir -p gpurun_out
cp paper_conf_sc_goldfarbjk13_b200/libtt.so /tmp/libtt_orig.so
for v in "$@"; do
  cp abtest/libtt_$v.so paper_conf_sc_goldfarbjk13_b200/libtt.so
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:bh_group_kernel -s 1 -c 1 \
      -o gpurun_out/prof_ab_$v python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-chase --no-strong \
      > gpurun_out/ncu_ab_$v.log 2>&1
  echo "$v ncu rc=$?"
done
cp /tmp/libtt_orig.so paper_conf_sc_goldfarbjk13_b200/libtt.so
