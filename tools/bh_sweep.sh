for a in 2 4 6; do timeout 600 python bench.py --workload bh --mode auto --auto-min-depth $a --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl; done
timeout 600 python bench.py --workload bh --mode independent --unsorted --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
for a in 0 2 4 6; do timeout 600 python bench.py --workload bh --mode auto --unsorted --auto-min-depth $a --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl; done
