#!/bin/bash
# HotSpot leaf check: GPU tests (v3 default, v1), in-HBM throughput of v3 variants vs v1, out-of-core 32768^2 x 64.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x > gpurun_out/tg_hs.log 2>&1; tail -3 gpurun_out/tg_hs.log | cut -c1-300
NORTHUP_HS_LEAF=1 timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x 2>&1 | tail -1
echo "v1:"; NORTHUP_HS_LEAF=1 HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | cut -c1-700
for f in build/hsvar/*.so; do echo "$f:"; NORTHUP_LIB_PATH=$f HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | cut -c1-700; done
timeout 600 python tools/hotspot_perf.py 32768 64 8 > gpurun_out/hs_perf.log 2>&1; cat gpurun_out/hs_perf.log | cut -c1-600
