#!/bin/bash
# After a BH kernel change (round 2): tests, smoke, the BH launch list and
# ncu captures (configs[1] and configs[4]'s 16M), counts merged by
# make_profiles.py, the BH bench lines, the reference arm, paper tables and
# the checked build.  Outputs in gpurun_out/ (summaries in gpurun_out/refresh/).
mkdir -p gpurun_out/refresh
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_bh.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-strong > /dev/null 2>&1
for spec in "bh auto 5" "bh16m auto 5"; do
  set -- $spec
  w=$1; m=$2; sk=$3
  extra=""
  case $w in *16m) extra="--device-build";; esac
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bh_group_kernel -s $sk -c 1 \
      -o gpurun_out/prof_${w}_${m} python bench.py --workload $w --mode $m --steps 1 --warmup 1 \
      --no-cpu-baseline --no-e2e --no-chase --no-strong $extra > gpurun_out/ncu_${w}_${m}.log 2>&1
done
python tools/make_profiles.py r02 > gpurun_out/make_profiles.log 2>&1
cp profiles/ncu_counts.json profiles/r02/ncu_bh_auto.md profiles/r02/ncu_bh16m_auto.md profiles/r02/launches_bh.md gpurun_out/refresh/
ncu -i gpurun_out/prof_bh_auto.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/refresh/src_bh_auto.csv.gz
ncu -i gpurun_out/prof_bh_auto.ncu-rep --page raw --csv 2>/dev/null | gzip > gpurun_out/refresh/raw_bh_auto.csv.gz
mkdir -p /tmp/reps && mv gpurun_out/prof_*.ncu-rep /tmp/reps/ 2>/dev/null
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 1200 python bench.py --workload bh16m --device-build > gpurun_out/bench_bh16m.json 2>> gpurun_out/bench_err.log
timeout 900 python bench.py --workload bhsteps > gpurun_out/bench_bhsteps.json 2>> gpurun_out/bench_err.log
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
timeout 1800 python tools/paper_tables.py --out gpurun_out/paper_tables.md > gpurun_out/paper_tables.log 2>&1
bash tools/checked_run.sh > gpurun_out/checked.txt 2>&1
tail -2 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; tail -c 400 gpurun_out/bench_default.json; cat gpurun_out/checked.txt
