#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hotspot_kernel_tma -s 2 -c 1 \
    -o gpurun_out/hs_tma -f python tools/hs_ncu.py 8 > gpurun_out/ncu_hs.log 2>&1; echo "ncu hs rc=$?"
ncu -i gpurun_out/hs_tma.ncu-rep --page details > gpurun_out/hotspot_tma_ncu.txt 2>&1
ncu -i gpurun_out/hs_tma.ncu-rep --page raw --csv > gpurun_out/hotspot_tma_raw.csv 2>&1
ncu -i gpurun_out/hs_tma.ncu-rep --page source --csv --print-source sass > gpurun_out/hotspot_tma_sass.csv 2>&1
rm -f gpurun_out/hs_tma.ncu-rep
