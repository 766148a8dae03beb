#!/bin/bash
# Round-1 refresh of the judged profiles: launch list of the default bench command, one --set full capture of
# the dominant kernel (a cfg3 K-panel reduce launch), the FILE-root bench (staging vs FILE->HBM bounce).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_cfg3.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/b_under_ncu.log 2>&1; echo "launch list rc=$?"
python tools/launch_summary.py gpurun_out/launches_cfg3.csv > gpurun_out/launches_cfg3_summary.txt; cat gpurun_out/launches_cfg3_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_gemm -s 1 -c 1 \
    -o gpurun_out/leaf_v3_cfg3 -f python tools/ncu_leaf.py 32768 > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
timeout 600 python tools/gds_bench.py 16384 > gpurun_out/gds.log 2>&1; echo "gds rc=$?"; tail -3 gpurun_out/gds.log | cut -c1-400
