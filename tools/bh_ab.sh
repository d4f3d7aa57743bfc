rm -f gpurun_out/ab.jsonl
for a in 1 0 1 0 3 0 3; do
  timeout 600 python bench.py --workload bh --mode auto --auto-min-depth $a --steps 10 --warmup 3 --no-cpu-baseline --no-e2e >> gpurun_out/ab.jsonl 2>>gpurun_out/err.log
done
timeout 600 python bench.py --workload bh --mode lockstep --steps 10 --warmup 3 --no-cpu-baseline --no-e2e >> gpurun_out/ab.jsonl 2>>gpurun_out/err.log
python - <<'PY'
import json
for l in open("gpurun_out/ab.jsonl"):
    d = json.loads(l); c = d["config"]
    print(f'mode={c["mode"]} T={c["auto_min_depth"]} kern={d["traverse_ms"]:8.3f} ms lock={d["lockstep_warp_fraction"]:.3f} clk={d["clocks"]["sm_mhz"]}')
PY
