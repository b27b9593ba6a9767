#!/bin/bash
mkdir -p gpurun_out/sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/sanitizer/$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer/summary.txt
done
cat gpurun_out/sanitizer/summary.txt
