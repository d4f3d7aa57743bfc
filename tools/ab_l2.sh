#!/bin/bash
# L2 persisting window A/B on the configs[4] trees (TT_L2_PERSIST_MB, tt_api.cu L2Window):
# off / 64 / max MiB, 2 rounds, traversal ms of bh16m and knn16m (device-built trees)
cp abtest/libtt_l2.so paper_conf_sc_goldfarbjk13_b200/libtt.so
python - <<'PY'
import torch
p = torch.cuda.get_device_properties(0)
print("persistingL2CacheMaxSize", getattr(p, "persisting_l2_cache_max_size", None), "L2", p.L2_cache_size)
PY
for rep in 1 2; do for w in bh16m knn16m; do for mb in 0 64 1000; do
  r=$(TT_L2_PERSIST_MB=$mb timeout 900 python bench.py --workload $w --device-build --steps 3 --no-cpu-baseline --no-e2e --no-chase --no-strong 2>>gpurun_out/ab_l2.err | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['traverse_ms'],3))")
  echo "$w mb=$mb: $r"
done; done; done
