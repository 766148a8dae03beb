#!/bin/bash
# v3 tuning sweep: each build/variants/*.so (NORTHUP_LIB_PATH), leaf variant 4
mkdir -p gpurun_out
: > gpurun_out/variants4.log
timeout 300 python -m pytest tests/test_gpu_leaf.py -x -q -k "v3" > gpurun_out/tm_test.log 2>&1; tail -2 gpurun_out/tm_test.log
for so in build/variants/*.so; do
  echo "== $so" >> gpurun_out/variants4.log
  NORTHUP_LEAF=4 NORTHUP_LIB_PATH=$PWD/$so SZS=8192,32768 timeout 300 python tools/variant_perf.py >> gpurun_out/variants4.log 2>&1
  LEAF_VARIANT=4 NORTHUP_LIB_PATH=$PWD/$so timeout 200 python tools/mma_prof.py >> gpurun_out/variants4.log 2>&1
done
cat gpurun_out/variants4.log
