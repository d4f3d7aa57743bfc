#!/bin/bash
# NEXT-4 sharded time stepping: GPU tests + bhsteps bench at 1 rank and 2 ranks on one GPU (gloo wire)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sharded_steps.py -m gpu -x -q > gpurun_out/pytest_steps.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_steps.txt
timeout 600 python bench.py --workload bhsteps --steps 5 --warmup 3 > gpurun_out/bhsteps_1.json 2> gpurun_out/bhsteps_1.err
TT_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
   bench.py --gpus 2 --workload bhsteps --steps 5 --warmup 3 > gpurun_out/bhsteps_2gloo.json 2> gpurun_out/bhsteps_2gloo.err
tail -3 gpurun_out/pytest_steps.txt; cat gpurun_out/bhsteps_1.json gpurun_out/bhsteps_2gloo.json | cut -c1-300; tail -3 gpurun_out/bhsteps_2gloo.err
