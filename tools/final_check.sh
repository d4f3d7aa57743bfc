#!/bin/bash
# End-of-round check on the GPU box: tests, smoke, bench lines (every
# workload, with the oracle baseline), reference arm, paper tables, ncu.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for w in knn vp pc nn bh16m knn16m; do
  timeout 900 python bench.py --workload $w > gpurun_out/bench_$w.json 2>> gpurun_out/bench_err.log
done
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
timeout 1500 python tools/paper_tables.py > gpurun_out/paper_tables.log 2>&1
bash tools/profile_all.sh
tail -2 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; cat gpurun_out/bench_default.json
