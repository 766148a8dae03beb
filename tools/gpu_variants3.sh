#!/bin/bash
mkdir -p gpurun_out
: > gpurun_out/variants.log
for so in build/variants/*.so; do
  echo "== $so" >> gpurun_out/variants.log
  NORTHUP_LEAF=3 NORTHUP_LIB_PATH=$PWD/$so SZS=8192 timeout 300 python tools/npass2_check.py 2>&1 | grep tflops >> gpurun_out/variants.log
  LEAF_VARIANT=3 NORTHUP_LIB_PATH=$PWD/$so timeout 200 python tools/mma_prof.py >> gpurun_out/variants.log 2>&1
done
