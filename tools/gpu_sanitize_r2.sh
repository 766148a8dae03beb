#!/bin/bash
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_r2.py > gpurun_out/sanitize_r2_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize_r2_$tool.log
  tail -n 4 gpurun_out/sanitize_r2_$tool.log
done
