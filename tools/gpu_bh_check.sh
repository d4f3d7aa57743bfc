#!/bin/bash
# BH-focused GPU check: BH parity tests + timing (run under gpurun)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "bh or plummer or two_body or sharded" > gpurun_out/pytest_bh.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_bh.txt
rm -f gpurun_out/quick.jsonl
bash tools/quick_bench.sh "bh auto 5" "bh auto 5" "bh lockstep 5"
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
python tools/show_quick.py < gpurun_out/quick.jsonl
tail -2 gpurun_out/pytest_bh.txt
