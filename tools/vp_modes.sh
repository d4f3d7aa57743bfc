rm -f gpurun_out/vpu.jsonl
for m in independent auto; do
timeout 900 python bench.py --workload vp --mode $m --unsorted --steps 2 --warmup 1 --no-cpu-baseline --no-e2e >> gpurun_out/vpu.jsonl 2>>gpurun_out/err.log
done
timeout 900 python bench.py --workload vp --mode independent --steps 2 --warmup 1 --no-cpu-baseline --no-e2e >> gpurun_out/vpu.jsonl 2>>gpurun_out/err.log
timeout 900 python bench.py --workload vp --mode independent --no-schedule --steps 2 --warmup 1 --no-cpu-baseline --no-e2e >> gpurun_out/vpu.jsonl 2>>gpurun_out/err.log
python - <<'PY'
import json
for l in open("gpurun_out/vpu.jsonl"):
    d = json.loads(l); c = d["config"]
    print(f'{c["workload"]:12s} {c["mode"]:12s} sorted={c["sorted"]!s:5s} sched={c["tile_schedule"]} kern={d["traverse_ms"]:9.3f} ms lock={d["lockstep_warp_fraction"]:.4f}')
PY
