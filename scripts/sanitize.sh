#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck over every kernel (C1-sized)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 \
      python scripts/sanitize_driver.py > gpurun_out/sanitizer/$tool.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/sanitizer/$tool.log | tail -1)"
done
