#!/bin/bash
mkdir -p gpurun_out
( nvidia-smi --query-gpu=clocks.sm,power.draw --format=csv,noheader -lms 500 > gpurun_out/clk_sweep.csv ) &
SMI=$!
timeout 300 python tools/sweep.py prec > gpurun_out/sweep.log 2>&1
for band in 4 16 32; do for pan in 0 1 4; do
  NORTHUP_RASTER_BAND=$band NORTHUP_PANEL_CHUNKS=$pan timeout 300 python tools/sweep.py perf >> gpurun_out/sweep.log 2>&1
done; done
kill $SMI
timeout 600 python -m pytest tests/test_gpu_leaf.py tests/test_gpu_tree.py -x -q > gpurun_out/tg.log 2>&1; tail -2 gpurun_out/tg.log
