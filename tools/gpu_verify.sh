#!/bin/bash
# Re-entry check: build + smoke, all GPU tests, the default bench line.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tg.log 2>&1; tail -3 gpurun_out/tg.log
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -c 600 gpurun_out/bench_full.json
nvidia-smi -q | grep -i -A3 "nvme\|Product Name" | head; lsblk 2>/dev/null | head -20
