#!/bin/bash
# NEXT-1 session: tree tests (shared staging incl.), virtual-sibling shared-staging bench + PCIe probe,
# cfg3 out-of-core timeline and the default bench line (slowdown variance check).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_tree.py -q -x > gpurun_out/tg_tree.log 2>&1; tail -3 gpurun_out/tg_tree.log
timeout 900 python tools/shared_bench.py > gpurun_out/shared_bench.log 2>&1; cat gpurun_out/shared_bench.log | cut -c1-600
timeout 600 python tools/ooc_timeline.py 32768 > gpurun_out/ooc_tl.json 2>&1; head -c 1500 gpurun_out/ooc_tl.json
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_full.json').read().strip().splitlines()[-1]); print('bench', d['value'], d['e2e']['value'], d['slowdown_pct_vs_in_hbm'], d['roofline']['frac'], d['clocks'])"
