#!/bin/bash
# bench (full cfg3) + ncu launch list of the same command + ncu --set full of one cfg3 leaf launch
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
if [ "$1" == "ncu" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_cfg3.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline \
    > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_gemm -s 20 -c 1 \
    -o gpurun_out/prof_cfg3 -f python tools/ncu_leaf.py 32768 > gpurun_out/ncu_cfg3.log 2>&1
fi
