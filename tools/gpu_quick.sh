#!/bin/bash
mkdir -p gpurun_out
timeout 120 python tools/debug_leaf.py > gpurun_out/dbg.log 2>&1; echo rc=$? >> gpurun_out/dbg.log
timeout 600 python -m pytest tests/test_gpu_leaf.py tests/test_gpu_tree.py -x -q > gpurun_out/tg.log 2>&1; tail -3 gpurun_out/tg.log
timeout 300 python tools/perf_leaf.py > gpurun_out/perf2.log 2>&1
if [ "$1" == "ncu" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:leaf_gemm -s 2 -c 1 \
    -o gpurun_out/prof_leaf2 -f python tools/ncu_leaf.py 8192 > gpurun_out/ncu_full.log 2>&1
fi
