#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for v in 1 2; do for li in 1 8; do
NORTHUP_HS_LEAF=$v timeout 300 ncu --set full --clock-control none --import-source on -k regex:hotspot_kernel -s 2 -c 1 \
   -o gpurun_out/hs_v${v}_li${li} -f python tools/hs_ncu.py $li > gpurun_out/hs_ncu_v${v}_li${li}.log 2>&1; tail -1 gpurun_out/hs_ncu_v${v}_li${li}.log
done; done
ls gpurun_out/*.ncu-rep
