#!/bin/bash
# Round-2 refresh on the GPU box: tests, smoke, ncu capture of every traversal
# kernel + counts (make_profiles.py on the box), bench line of every
# workload (reading those counts), reference arm, paper tables.
# gpurun brings back <= 64 MiB of gpurun_out/: the .ncu-rep files are
# summarised here and moved out (the BH and kNN source pages kept, gzipped).
mkdir -p gpurun_out/refresh
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
bash tools/profile_all.sh > gpurun_out/profile_all.log 2>&1
python tools/make_profiles.py r02 > gpurun_out/make_profiles.log 2>&1
cp profiles/ncu_counts.json profiles/r02/ncu_*.md profiles/r02/launches_bh.md gpurun_out/refresh/
for t in bh_auto knn_auto bh16m_auto knn16m_auto; do
  ncu -i gpurun_out/prof_$t.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/refresh/src_$t.csv.gz
  ncu -i gpurun_out/prof_$t.ncu-rep --page raw --csv 2>/dev/null | gzip > gpurun_out/refresh/raw_$t.csv.gz
done
mkdir -p /tmp/reps && mv gpurun_out/prof_*.ncu-rep /tmp/reps/ 2>/dev/null
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for w in knn vp pc nn bh16m knn16m bhsteps; do
  extra=""
  case $w in *16m) extra="--device-build";; esac
  timeout 1200 python bench.py --workload $w $extra > gpurun_out/bench_$w.json 2>> gpurun_out/bench_err.log
done
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
timeout 1800 python tools/paper_tables.py --out gpurun_out/paper_tables.md > gpurun_out/paper_tables.log 2>&1
du -sh gpurun_out
tail -2 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; cat gpurun_out/bench_default.json
