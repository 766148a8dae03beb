#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x > gpurun_out/tg_hs.log 2>&1; tail -3 gpurun_out/tg_hs.log | cut -c1-400
NORTHUP_HS_LEAF=1 timeout 600 python -m pytest tests/test_gpu_hotspot.py -q -x 2>&1 | tail -1
HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | cut -c1-700
timeout 900 python bench.py --config hotspot --steps 3 --warmup 3 > gpurun_out/bench_hotspot.json 2> gpurun_out/bench_hotspot.err; tail -2 gpurun_out/bench_hotspot.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_hotspot.json').read().strip().splitlines()[-1]); print('hs', d['value'], d['e2e']['value'], d['slowdown_pct_vs_in_hbm'], d['roofline']['frac'], d['parity'], d['clocks'])"
timeout 600 python tools/hotspot_perf.py 32768 64 8 > gpurun_out/hs_perf.log 2>&1; tail -1 gpurun_out/hs_perf.log | cut -c1-600
