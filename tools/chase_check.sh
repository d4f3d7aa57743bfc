#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k diag > gpurun_out/pytest_diag.txt 2>&1; tail -1 gpurun_out/pytest_diag.txt
for w in bh knn nn vp pc; do
  st=5; [ $w = vp ] && st=2
  timeout 600 python bench.py --workload $w --steps $st --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/chase_err.log | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; c=r.get('chase')
print('$w', round(d['traverse_ms'],3), 'ms lock', d['lockstep_warp_fraction'], 'chase', c)"
done
for w in bh knn; do
  timeout 600 python bench.py --workload $w --unsorted --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/chase_err.log | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; c=r.get('chase')
print('$w unsorted', round(d['traverse_ms'],3), 'ms lock', d['lockstep_warp_fraction'], 'chase', c)"
done
