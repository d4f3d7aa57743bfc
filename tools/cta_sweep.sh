#!/bin/bash
# resident CTAs per SM sweep (TT_CTAS_PER_SM, tuning only) -> gpurun_out/cta_sweep.txt
for w in bh knn nn vp; do for c in 2 3 4; do
  st=5; [ $w = vp ] && st=2
  r=$(TT_CTAS_PER_SM=$c timeout 600 python bench.py --workload $w --steps $st --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['traverse_ms'],3))")
  echo "$w ctas=$c kern_ms=$r" | tee -a gpurun_out/cta_sweep.txt
done; done
