set -x
timeout 900 python -m pytest tests -m "gpu" -x -q -k "vp or knn" 2>&1 | tail -3
for w in knn vp; do
 for m in lockstep independent; do timeout 600 python bench.py --workload $w --mode $m --steps 3 --warmup 1 --no-cpu-baseline --no-e2e 2>>gpurun_out/err.log | tee -a gpurun_out/sweep.jsonl; done
 for a in 2 4 6 8 10 12; do timeout 600 python bench.py --workload $w --mode auto --auto-min-depth $a --steps 3 --warmup 1 --no-cpu-baseline --no-e2e 2>>gpurun_out/err.log | tee -a gpurun_out/sweep.jsonl; done
done
for a in 0 2 4 6 8; do timeout 600 python bench.py --workload knn --mode auto --unsorted --auto-min-depth $a --steps 3 --warmup 1 --no-cpu-baseline --no-e2e 2>>gpurun_out/err.log | tee -a gpurun_out/sweep.jsonl; done
for a in 2 4 8; do timeout 600 python bench.py --workload vp --mode auto --unsorted --auto-min-depth $a --steps 2 --warmup 1 --no-cpu-baseline --no-e2e 2>>gpurun_out/err.log | tee -a gpurun_out/sweep.jsonl; done
