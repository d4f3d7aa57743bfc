mkdir -p gpurun_out
timeout 600 python bench.py --workload bhsteps --steps 10 --warmup 3 > gpurun_out/bhsteps_1.json 2> gpurun_out/bhsteps_1.err
TT_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
   bench.py --gpus 2 --workload bhsteps --steps 10 --warmup 3 > gpurun_out/bhsteps_2gloo.json 2> gpurun_out/bhsteps_2gloo.err
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for f in bhsteps_1 bhsteps_2gloo bench_default; do python -c "import json,sys; d=json.loads(open('gpurun_out/$f.json').read().strip().splitlines()[-1]); print('$f', d['value'], d['ms_per_step'], d.get('clocks'))"; done
