#!/bin/bash
# Full session after a leaf change: build+smoke, all GPU tests, default bench,
# ncu launch list of the bench command, ncu --set full of one cfg3 panel launch.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tg.log 2>&1; tail -3 gpurun_out/tg.log
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -c 300 gpurun_out/bench_full.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline \
    > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_gemm -s 20 -c 1 \
    -o gpurun_out/prof_leaf_32768 -f python tools/ncu_leaf.py 32768 > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log
