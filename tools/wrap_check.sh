#!/bin/bash
# Last check of the round: all GPU tests, smoke, default bench (roofline keys),
# time stepping, and the Table 1/2 analogue.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 python bench.py --workload bhsteps --steps 5 --warmup 3 > gpurun_out/bench_bhsteps.json 2>> gpurun_out/bench_err.log
timeout 1500 python tools/paper_tables.py > gpurun_out/paper_tables.log 2>&1
tail -2 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt
