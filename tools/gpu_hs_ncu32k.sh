#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
HS_N=32768 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:hotspot_kernel_tma -s 2 -c 1 --csv \
    python tools/hs_ncu.py 8 > gpurun_out/hs_ncu32k.csv 2> gpurun_out/hs_ncu32k.err; echo "ncu rc=$?"
cat gpurun_out/hs_ncu32k.csv | tail -4
