#!/bin/bash
mkdir -p gpurun_out/sanitizer
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > gpurun_out/sanitizer/$tool.txt 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer/$tool.txt
  tail -3 gpurun_out/sanitizer/$tool.txt
done
