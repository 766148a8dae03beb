#!/bin/bash
# HotSpot leaf v4 (packed fp32x2): bitwise tests of all leaves, in-HBM throughput v3 vs v4, bench line with v4.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_hotspot.py -q -x > gpurun_out/tg_hs.log 2>&1; tail -3 gpurun_out/tg_hs.log | cut -c1-300
NORTHUP_HS_LEAF=4 timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x 2>&1 | tail -1
for v in 3 4; do echo "v$v:"; NORTHUP_HS_LEAF=$v HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | cut -c1-700; done
NORTHUP_HS_LEAF=4 timeout 900 python bench.py --config hotspot > gpurun_out/bench_hs_v4.json 2> gpurun_out/bench_hs_v4.err; echo "hs v4 rc=$?"
