#!/bin/bash
# HotSpot leaf v6 (persistent v3, staged T loads): bitwise tests, tree tests with v6, in-HBM throughput v3 vs v6.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x -k variants 2>&1 | tail -1
NORTHUP_HS_LEAF=6 timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x 2>&1 | tail -1
for v in 3 6 3 6; do echo "v$v:"; NORTHUP_HS_LEAF=$v HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print({k:round(v['gcups'],1) for k,v in d.items() if isinstance(v,dict)})"; done
