#!/bin/bash
# Closing run after the HotSpot update rewrite: smoke, full GPU suite, default bench, HotSpot bench.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 > gpurun_out/gputest.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/gputest.log
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "default rc=$?"
timeout 900 python bench.py --config hotspot --steps 5 --warmup 3 > gpurun_out/bench_hotspot.json 2> gpurun_out/bench_hotspot.err; echo "hotspot rc=$?"
python -c "
import json
for f in ['gpurun_out/bench_default.json','gpurun_out/bench_hotspot.json']:
    d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, d['value'], d['e2e']['value'], d['in_hbm']['value'], d['roofline']['frac'], d['clocks'])
"
