#!/bin/bash
mkdir -p gpurun_out
SZ=${1:-8192}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_gemm -s 2 -c 1 \
    -o gpurun_out/prof_leaf_$SZ -f python tools/ncu_leaf.py $SZ > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log
