#!/bin/bash
# BH A/B on one box: tools/ab_bh.sh A B ... (abtest/libtt_X.so), 3 rounds, traversal ms
cp paper_conf_sc_goldfarbjk13_b200/libtt.so /tmp/libtt_orig.so
for rep in 1 2 3; do for v in "$@"; do
  cp abtest/libtt_$v.so paper_conf_sc_goldfarbjk13_b200/libtt.so
  r=$(timeout 600 python bench.py --no-cpu-baseline --no-e2e --no-chase --no-strong --steps 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['traverse_ms'],4), round(d['ms_per_step'],4))")
  echo "$v: $r"
done; done
cp /tmp/libtt_orig.so paper_conf_sc_goldfarbjk13_b200/libtt.so
