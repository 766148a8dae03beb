#!/bin/bash
# HotSpot v3 with the iteration loop unrolled by 2: bitwise tests + in-HBM throughput vs default.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for so in default build/hsu/u2.so default build/hsu/u2.so; do
  echo "== $so"
  if [ "$so" = default ]; then unset NORTHUP_LIB_PATH; else export NORTHUP_LIB_PATH=$PWD/$so; fi
  timeout 300 python -m pytest tests/test_gpu_hotspot.py -q -x -k "variants_bitwise and 3 or whole_grid" 2>&1 | tail -1
  HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print({k:round(v['gcups'],1) for k,v in d.items() if isinstance(v,dict)})"
done
