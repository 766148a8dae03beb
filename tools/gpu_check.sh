#!/bin/bash
# Re-entry check: smoke, all GPU tests, default bench line, hotspot bench line.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu -rf > gpurun_out/tg.log 2>&1; tail -8 gpurun_out/tg.log
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench rc=$?"
timeout 900 python bench.py --config hotspot > gpurun_out/bench_hs.json 2> gpurun_out/bench_hs.err; echo "hs rc=$?"
timeout 300 python tools/gds_bench.py > gpurun_out/gds.log 2>&1; echo "gds rc=$?"; tail -5 gpurun_out/gds.log
