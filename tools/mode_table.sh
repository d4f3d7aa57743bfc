#!/bin/bash
# Mode x order table of every workload (DESIGN.md §4.5 / §7) -> gpurun_out/modes.jsonl
mkdir -p gpurun_out
for w in bh knn pc vp; do
  for o in "" "--unsorted"; do
    for m in auto lockstep independent; do
      st=5; [ $w = vp ] && st=2
      timeout 600 python bench.py --workload $w --mode $m $o --steps $st --warmup 3 --no-cpu-baseline --no-e2e \
        2>>gpurun_out/modes_err.log >> gpurun_out/modes.jsonl
    done
  done
done
for w in bh16m knn16m bhsteps; do
  timeout 900 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-e2e \
    2>>gpurun_out/modes_err.log >> gpurun_out/modes.jsonl
done
python tools/show_quick.py gpurun_out/modes.jsonl
