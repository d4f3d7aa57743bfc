for w in bh knn vp pc; do
  timeout 900 python bench.py --workload $w --mode independent --variant recursive --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
  timeout 900 python bench.py --workload $w --mode independent --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>>gpurun_out/quick_err.log >> gpurun_out/quick.jsonl
done
