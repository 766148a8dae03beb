#!/bin/bash
# ncu evidence for the round: HotSpot v3 leaf (full set), GEMM leaf cfg3 panel launch (full set),
# launch lists of the default bench and of the HotSpot bench.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hotspot_kernel_v3 -s 2 -c 1 \
    -o gpurun_out/hs_v3_li8 -f python tools/hs_ncu.py 8 > gpurun_out/hs_ncu_v3.log 2>&1; tail -1 gpurun_out/hs_ncu_v3.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_gemm -s 20 -c 1 \
    -o gpurun_out/prof_leaf_32768 -f python tools/ncu_leaf.py 32768 > gpurun_out/ncu_full.log 2>&1; tail -1 gpurun_out/ncu_full.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1; tail -1 gpurun_out/ncu_bench.log
