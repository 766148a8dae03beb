#!/bin/bash
# Full GPU suite + smoke + default bench line.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 2000 python -m pytest tests -q -m gpu -rf --durations=10 -p no:cacheprovider > gpurun_out/tg.log 2>&1; echo "pytest rc=$?"; tail -16 gpurun_out/tg.log | cut -c1-200
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench_full.json').read().strip().splitlines()[-1]); print('bench', d['value'], d['e2e']['value'], d['slowdown_pct_vs_in_hbm'], d['roofline']['frac'], d['e2e_roofline']['frac'], d['cfg2_in_hbm_tflops'], d['slowdown_pct_vs_cfg2_in_hbm'], d['staging']['copy_hidden_pct'], d['clocks'])"
