#!/bin/bash
# A/B libtt builds on one box: tools/ab_libs.sh "<bench args>" A B C ...  (abtest/libtt_X.so)
args=$1; shift
cp paper_conf_sc_goldfarbjk13_b200/libtt.so /tmp/libtt_orig.so
for rep in 1 2; do for v in "$@"; do
  cp abtest/libtt_$v.so paper_conf_sc_goldfarbjk13_b200/libtt.so
  r=$(timeout 600 python bench.py $args --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['traverse_ms'],3), d.get('lockstep_warp_fraction'))")
  echo "$v: $r"
done; done
cp /tmp/libtt_orig.so paper_conf_sc_goldfarbjk13_b200/libtt.so
