#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python bench.py --config hotspot --steps 3 --warmup 3 > gpurun_out/bench_hotspot.json 2> gpurun_out/bench_hotspot.err; tail -3 gpurun_out/bench_hotspot.err; tail -c 2500 gpurun_out/bench_hotspot.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
    --log-file gpurun_out/hs_launches.csv python bench.py --config hotspot --quick --steps 1 --warmup 3 > gpurun_out/hs_ncu_bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hotspot_kernel -s 5 -c 1 \
    -o gpurun_out/hs_v3_li8 -f python tools/hs_ncu.py 8 > gpurun_out/hs_ncu_v3.log 2>&1; tail -1 gpurun_out/hs_ncu_v3.log
