#!/bin/bash
# A/B on one box for any workload: tools/ab_w.sh "<bench args>" A B ... (abtest/libtt_X.so), 2 rounds
args=$1; shift
cp paper_conf_sc_goldfarbjk13_b200/libtt.so /tmp/libtt_orig.so
for rep in 1 2; do for v in "$@"; do
  cp abtest/libtt_$v.so paper_conf_sc_goldfarbjk13_b200/libtt.so
  r=$(timeout 900 python bench.py $args --no-cpu-baseline --no-e2e --no-chase --no-strong 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['traverse_ms'],4), round(d['ms_per_step'],4))")
  echo "$v: $r"
done; done
cp /tmp/libtt_orig.so paper_conf_sc_goldfarbjk13_b200/libtt.so
