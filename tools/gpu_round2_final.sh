#!/bin/bash
# Round-2 evidence: full GPU suite, smoke, the default bench line, and the launch list of the
# same bench command under ncu (per-launch times, cold-cache and serialised: shares only).
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 > gpurun_out/gputest.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_cfg3.log 2>&1; echo "bench rc=$?"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/launches_cfg3.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/b_under_ncu.log 2>&1; echo "launch list rc=$?"
python tools/launch_summary.py gpurun_out/launches_cfg3.csv > gpurun_out/launches_cfg3_summary.txt; head -20 gpurun_out/launches_cfg3_summary.txt
