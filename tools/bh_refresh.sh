#!/bin/bash
# After a BH kernel change, on the GPU box: tests, smoke, BH launch list and
# ncu capture, counts refresh (make_profiles.py, run on the box), then the
# bench lines that read those counts.  Everything lands in gpurun_out/.
mkdir -p gpurun_out/refresh
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.txt
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_bh.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:bh_group_kernel -s 1 -c 1 \
    -o gpurun_out/prof_bh_auto python bench.py --workload bh --mode auto --steps 1 --warmup 1 \
    --no-cpu-baseline --no-e2e --points-per-rank 1000000 > gpurun_out/ncu_bh_auto.log 2>&1
python tools/make_profiles.py r01 > gpurun_out/make_profiles.log 2>&1
cp profiles/ncu_counts.json profiles/r01/ncu_bh_auto.md profiles/r01/launches_bh.md gpurun_out/refresh/
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 python bench.py --workload bh16m > gpurun_out/bench_bh16m.json 2>> gpurun_out/bench_default.err
timeout 600 python bench.py --workload bhsteps > gpurun_out/bench_bhsteps.json 2>> gpurun_out/bench_default.err
tail -2 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; cat gpurun_out/bench_default.json
