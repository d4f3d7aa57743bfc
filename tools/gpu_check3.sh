#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nn.py tests/test_gpu_parity.py -x -q -k "nn or switch or knn" > gpurun_out/pytest_k.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_k.txt
rm -f gpurun_out/sw.jsonl
for a in 0 2 4 8 12 16; do
  timeout 600 python bench.py --workload knn --mode lockstep --switch-below $a --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/sw_err.log >> gpurun_out/sw.jsonl
done
for a in 4 8 16; do
  timeout 600 python bench.py --workload knn --mode lockstep --unsorted --switch-below $a --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/sw_err.log >> gpurun_out/sw.jsonl
done
bash tools/ab_libs.sh "--workload bh --steps 10 --warmup 3" b4 m6 s5 s6 > gpurun_out/ab_regs.txt 2>&1
tail -3 gpurun_out/pytest_k.txt
python - <<'PY'
import json
for l in open("gpurun_out/sw.jsonl"):
    d=json.loads(l); c=d["config"]
    print(c["workload"], c["sorted"], c.get("switch_below",0), round(d["traverse_ms"],3), d["visits_per_point"])
PY
cat gpurun_out/ab_regs.txt
