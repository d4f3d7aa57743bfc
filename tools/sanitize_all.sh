#!/bin/bash
# compute-sanitizer over tools/sanitize.py (every kernel, variant and mode);
# logs in gpurun_out/sanitizer/ (copied to profiles/<round>/sanitizer/).
mkdir -p gpurun_out/sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > gpurun_out/sanitizer/$tool.txt 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer/$tool.txt
  tail -3 gpurun_out/sanitizer/$tool.txt
done
