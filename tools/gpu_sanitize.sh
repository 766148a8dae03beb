#!/bin/bash
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize_$tool.log
done
timeout 600 python -m pytest tests/test_gpu_leaf.py -x -q -k v2_ldg > gpurun_out/tv2.log 2>&1
for f in gpurun_out/sanitize_*.log gpurun_out/tv2.log; do tail -n 3 $f; done
