#!/bin/bash
# out-of-core check after a planner change: timeline, tree/config tests, bench cfg3 + cfg5
mkdir -p gpurun_out
timeout 600 python tools/ooc_timeline.py 32768 > gpurun_out/ooc_tl.json 2>&1; cat gpurun_out/ooc_tl.json | head -12
timeout 1200 python -m pytest tests/test_gpu_tree.py tests/test_gpu_file.py tests/test_gpu_configs.py -q -x > gpurun_out/tg_ooc.log 2>&1; tail -2 gpurun_out/tg_ooc.log
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
timeout 900 python bench.py --config cfg5 --steps 3 --warmup 3 --cpu-budget 5 > gpurun_out/bench_cfg5.json 2> gpurun_out/bench_cfg5.err
timeout 900 python bench.py --config cfg2 --steps 5 --warmup 3 --cpu-budget 5 > gpurun_out/bench_cfg2.json 2> gpurun_out/bench_cfg2.err
for f in bench_full bench_cfg5 bench_cfg2; do python -c "
import json,sys; d=json.loads(open('gpurun_out/$f.json').read().strip().splitlines()[-1]); print('$f', d['value'], d['e2e']['value'], d['slowdown_pct_vs_in_hbm'], d['roofline']['frac'], d['clocks']['sm_mhz'])"; done
