#!/bin/bash
# End-of-session check on the GPU box: tests, smoke, ncu captures of every
# traversal kernel + counts refresh (make_profiles.py on the box), then the
# bench lines that read those counts.  Copies for profiles/ land in
# gpurun_out/refresh/.
mkdir -p gpurun_out/refresh
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
bash tools/profile_all.sh > gpurun_out/profile_all.log 2>&1
python tools/make_profiles.py r01 > gpurun_out/make_profiles.log 2>&1
cp profiles/ncu_counts.json profiles/r01/ncu_*.md profiles/r01/launches_bh.md gpurun_out/refresh/
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for w in knn vp pc nn bh16m knn16m; do
  timeout 900 python bench.py --workload $w > gpurun_out/bench_$w.json 2>> gpurun_out/bench_err.log
done
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
rm -f gpurun_out/prof_*.ncu-rep.tmp
tail -2 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; cat gpurun_out/bench_default.json
