#!/bin/bash
# full validation: smoke, every -m gpu test, default bench, cfg4 bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tg.log 2>&1; tail -3 gpurun_out/tg.log
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -c 600 gpurun_out/bench_full.json
timeout 900 python bench.py --config cfg4 --steps 3 --warmup 3 --cpu-budget 5 > gpurun_out/bench_cfg4.json 2> gpurun_out/bench_cfg4.err
