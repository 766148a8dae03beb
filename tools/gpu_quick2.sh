#!/bin/bash
mkdir -p gpurun_out
timeout 600 python tools/npass2_check.py > gpurun_out/np2.log 2>&1
timeout 300 python tools/mma_prof.py > gpurun_out/mma_prof.log 2>&1
timeout 900 python -m pytest tests/test_gpu_leaf.py tests/test_gpu_tree.py tests/test_gpu_file.py -x -q > gpurun_out/tg.log 2>&1; tail -2 gpurun_out/tg.log
