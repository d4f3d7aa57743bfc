#!/bin/bash
# after the oct-build change: GPU tests touching the builders / time stepping, bhsteps x5 fresh processes
mkdir -p gpurun_out
python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "oct or steps or sharded or recycled or order or blob" > gpurun_out/r02_pt2.txt 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r02_pt2.txt
for i in 1 2 3 4 5; do
  python bench.py --workload bhsteps --steps 10 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('bhsteps', round(d['ms_per_step'],3))"
done
