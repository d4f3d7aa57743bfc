#!/bin/bash
# staged-top budget sweep (TT_STAGE_BYTES, tuning only) -> gpurun_out/stage2.txt
for w in bh knn nn vp; do for sb in 32 4096 16384 32768; do
  st=5; [ $w = vp ] && st=2
  r=$(TT_STAGE_BYTES=$sb timeout 600 python bench.py --workload $w --steps $st --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['traverse_ms'],3))")
  echo "$w stage_bytes=$sb kern_ms=$r" | tee -a gpurun_out/stage2.txt
done; done
