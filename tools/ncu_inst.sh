#!/bin/bash
# Executed warp instructions and duration of one non-stats BH launch for each
# abtest/libtt_<name>.so: tools/ncu_inst.sh A B ...
cp paper_conf_sc_goldfarbjk13_b200/libtt.so /tmp/libtt_orig.so
for v in "$@"; do
  cp abtest/libtt_$v.so paper_conf_sc_goldfarbjk13_b200/libtt.so
  r=$(timeout 600 ncu --metrics smsp__inst_executed.sum,gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:bh_group_kernel -s 5 -c 1 --csv \
      python bench.py --workload bh --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-chase --no-strong 2>/dev/null | grep -E "inst_executed|time_duration|issue_active" | awk -F'","' '{print $(NF-2)"="$NF}' | tr -d '"' | tr '\n' ' ')
  echo "$v: $r"
done
cp /tmp/libtt_orig.so paper_conf_sc_goldfarbjk13_b200/libtt.so
