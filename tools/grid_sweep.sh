#!/bin/bash
for g in 444 466 488 500 510 521 532 554 576 592; do
  r=$(TT_BH_GRID=$g timeout 600 python bench.py --workload bh --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['traverse_ms'],3))")
  echo "grid=$g kern_ms=$r" | tee -a gpurun_out/grid_sweep.txt
done
