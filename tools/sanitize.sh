#!/bin/bash
# compute-sanitizer over every library kernel at small n (run under gpurun, one GPU).
# Logs: gpurun_out/sanitize/{memcheck,racecheck,synccheck}.log
cd "$(dirname "$0")/.."
o=${OUT:-gpurun_out/sanitize}; mkdir -p $o
for tool in memcheck racecheck synccheck; do
  timeout 2400 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 \
    python tools/sanitize_driver.py ${SIZES:-10 12} > $o/$tool.log 2>&1
  echo "$tool rc=$?" >> $o/summary.txt
done
cat $o/summary.txt
