#!/bin/bash
mkdir -p gpurun_out
NORTHUP_LEAF=3 timeout 600 python tools/npass2_check.py > gpurun_out/np2_v3.log 2>&1
LEAF_VARIANT=3 timeout 300 python tools/mma_prof.py > gpurun_out/mma_prof_v3.log 2>&1
NORTHUP_LEAF=3 timeout 900 python -m pytest tests/test_gpu_leaf.py tests/test_gpu_tree.py -x -q > gpurun_out/tg_v3.log 2>&1; tail -2 gpurun_out/tg_v3.log
