#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_hotspot.py -q -x > gpurun_out/tg_hs.log 2>&1; tail -30 gpurun_out/tg_hs.log | cut -c1-400
timeout 900 python tools/hotspot_perf.py 32768 64 8 > gpurun_out/hs_perf.log 2>&1; cat gpurun_out/hs_perf.log | cut -c1-600
