#!/bin/bash
# HotSpot leaf v5 (4x4 register blocks): bitwise tests of every leaf, in-HBM throughput v3 vs v5, ncu of v5.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x -k variants > gpurun_out/tg_hs5.log 2>&1; tail -3 gpurun_out/tg_hs5.log | cut -c1-300
NORTHUP_HS_LEAF=5 timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x 2>&1 | tail -1
for v in 3 5; do echo "v$v:"; NORTHUP_HS_LEAF=$v HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print({k:round(v['gcups'],1) for k,v in d.items() if isinstance(v,dict)})"; done
NORTHUP_HS_LEAF=5 timeout 400 ncu --set full --clock-control none --import-source on -k regex:hotspot_kernel -s 2 -c 1 \
   -o gpurun_out/hs_v5_li8 -f python tools/hs_ncu.py 8 > gpurun_out/hs_ncu_v5.log 2>&1; tail -1 gpurun_out/hs_ncu_v5.log
