#!/bin/bash
# Full round check on the GPU box: gpu tests, smoke, default bench, quick
# benches of every workload, launch list + ncu --set full captures.
bash tools/gpu_validate.sh
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
bash tools/profile_all.sh
