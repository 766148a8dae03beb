#!/bin/bash
# Closing run: smoke, full GPU suite, default bench, HotSpot bench, launch list of the default bench command.
bash tools/gpu_final_r2c.sh
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/launches_cfg3.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/b_under_ncu.log 2>&1; echo "launch list rc=$?"
python tools/launch_summary.py gpurun_out/launches_cfg3.csv > gpurun_out/launches_cfg3_summary.txt; head -8 gpurun_out/launches_cfg3_summary.txt
