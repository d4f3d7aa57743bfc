#!/bin/bash
# round-2 interim check: default bench line, 2-rank torchrun test, PC line
mkdir -p gpurun_out
python bench.py > gpurun_out/r02_bench_bh.json 2> gpurun_out/r02_bench_bh.err; echo "bench rc=$?"
python -m pytest tests/test_bench_multirank.py -m gpu -q -p no:cacheprovider > gpurun_out/r02_multirank.txt 2>&1; echo "multirank rc=$?"
python bench.py --workload pc --no-strong > gpurun_out/r02_bench_pc.json 2> gpurun_out/r02_bench_pc.err; echo "pc rc=$?"
python bench.py --workload knn16m --device-build --steps 3 --no-cpu-baseline > gpurun_out/r02_bench_knn16m.json 2> gpurun_out/r02_bench_knn16m.err; echo "knn16m rc=$?"
