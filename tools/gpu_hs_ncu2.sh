#!/bin/bash
# ncu --set full of the HotSpot leaf v3 (product) and v4 (packed fp32x2), 8 iterations per launch on 16384^2.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for v in 3 4; do
NORTHUP_HS_LEAF=$v timeout 400 ncu --set full --clock-control none --import-source on -k regex:hotspot_kernel -s 2 -c 1 \
   -o gpurun_out/hs_v${v}_li8 -f python tools/hs_ncu.py 8 > gpurun_out/hs_ncu_v${v}.log 2>&1; tail -1 gpurun_out/hs_ncu_v${v}.log
done
ls -la gpurun_out/*.ncu-rep
