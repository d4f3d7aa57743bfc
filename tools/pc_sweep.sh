for m in lockstep independent; do timeout 600 python bench.py --workload pc --mode $m --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl; done
for a in 2 4 6 8; do timeout 600 python bench.py --workload pc --mode auto --auto-min-depth $a --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl; done
timeout 600 python bench.py --workload pc --mode lockstep --unsorted --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
timeout 600 python bench.py --workload pc --mode independent --unsorted --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
timeout 600 python bench.py --workload bh --mode auto --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
timeout 600 python bench.py --workload bh --mode auto --unsorted --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
