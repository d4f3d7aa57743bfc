#!/bin/bash
# End-of-session check on the committed sources: pytest -m gpu, smoke, the
# default bench line, the checked build run.  Outputs in gpurun_out/final/.
mkdir -p gpurun_out/final
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/final/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/final/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/final/smoke.txt
timeout 900 python bench.py > gpurun_out/final/bench_default.json 2> gpurun_out/final/bench_default.err
timeout 900 python bench.py --impl reference > gpurun_out/final/bench_reference.json 2> gpurun_out/final/bench_reference.err
bash tools/checked_run.sh > gpurun_out/final/checked.txt 2>&1
tail -2 gpurun_out/final/pytest_gpu.txt; tail -2 gpurun_out/final/smoke.txt; tail -c 600 gpurun_out/final/bench_default.json; cat gpurun_out/final/checked.txt
