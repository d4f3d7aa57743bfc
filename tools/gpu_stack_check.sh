#!/bin/bash
# NEXT-3 stack variant: parity tests + timings vs the method's kernels
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "stack or recursive" > gpurun_out/pytest_stack.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_stack.txt
rm -f gpurun_out/variants.jsonl
for spec in "bh lockstep stack" "bh independent stack" "bh lockstep autoropes" "bh independent autoropes" \
            "pc lockstep stack" "pc independent stack" "pc lockstep autoropes" "pc independent autoropes"; do
  set -- $spec
  timeout 600 python bench.py --workload $1 --mode $2 --variant $3 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e \
     >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err
  timeout 600 python bench.py --workload $1 --mode $2 --variant $3 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --unsorted \
     >> gpurun_out/variants.jsonl 2>> gpurun_out/variants.err
done
tail -3 gpurun_out/pytest_stack.txt
python - <<'PY'
import json
for l in open("gpurun_out/variants.jsonl"):
    d = json.loads(l); c = d["config"]
    print(f'{c["workload"]:14s} {c["mode"]:12s} {c["variant"]:10s} sorted={c["sorted"]!s:5s} kern={d["traverse_ms"]:9.3f} ms  fetch/visit={d.get("work_expansion_fetch_over_visits")}')
PY
