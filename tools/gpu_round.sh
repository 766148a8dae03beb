#!/bin/bash
# One GPU session: tests, bench (quick + full), ncu launch list + full profile of the leaf.
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python bench.py --quick > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err
timeout 600 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches.csv python bench.py --quick --steps 2 --warmup 3 --no-cpu-baseline \
    > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_gemm -s 2 -c 1 \
    -o gpurun_out/prof_leaf -f python tools/ncu_leaf.py 8192 > gpurun_out/ncu_full.log 2>&1
ls -la gpurun_out
