#!/bin/bash
# NEXT-3 NN kernel: GPU parity + bench in every mode -> gpurun_out/
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_nn.py -x -q > gpurun_out/pytest_nn.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_nn.txt
for o in "" "--unsorted"; do for m in auto lockstep independent; do
  timeout 600 python bench.py --workload nn --mode $m $o --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/nn_err.log >> gpurun_out/nn_modes.jsonl
done; done
timeout 600 python bench.py --workload nn --steps 10 --warmup 3 > gpurun_out/bench_nn.json 2>>gpurun_out/nn_err.log
tail -3 gpurun_out/pytest_nn.txt
python tools/show_quick.py gpurun_out/nn_modes.jsonl
