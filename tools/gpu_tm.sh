#!/bin/bash
# v3 (A' in TMEM) bring-up: parity tests, then timing and profile vs v1.2
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_leaf.py -x -q -k "v3" > gpurun_out/tm_test.log 2>&1; tail -3 gpurun_out/tm_test.log
for v in 2 4; do
  NORTHUP_LEAF=$v SZS=8192,16384,32768 timeout 300 python tools/variant_perf.py >> gpurun_out/tm_perf.log 2>&1
  LEAF_VARIANT=$v timeout 200 python tools/mma_prof.py >> gpurun_out/tm_perf.log 2>&1
done
cat gpurun_out/tm_perf.log
