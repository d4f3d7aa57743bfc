#!/bin/bash
# repeat the 2-rank gloo bench run to catch an intermittent hang (phase trace in gpurun_out/mrd_*.err);
# each run in its own session, killed by process group on timeout
mkdir -p gpurun_out
for i in 1 2 3 4; do
  port=$((29600 + i))
  TT_BENCH_TRACE=1 TT_DIST_BACKEND=gloo GLOO_SOCKET_IFNAME=lo setsid python -m torch.distributed.run --nnodes=1 \
     --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=$port bench.py --gpus 2 --steps 2 --warmup 3 \
     --points-per-rank 64000 --strong-points 256000 --no-cpu-baseline --no-e2e --no-chase \
     > gpurun_out/mrd_$i.out 2> gpurun_out/mrd_$i.err &
  pid=$!
  for t in $(seq 1 90); do kill -0 $pid 2>/dev/null || break; sleep 1; done
  if kill -0 $pid 2>/dev/null; then kill -9 -- -$pid; echo "run $i: killed after 90 s"; fi
  wait $pid; echo "run $i rc=$? $(grep -c '\[bench' gpurun_out/mrd_$i.err) trace lines"
done
