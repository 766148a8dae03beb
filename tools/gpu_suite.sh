#!/bin/bash
# Full GPU suite (names + durations), then cfg5 / cfg2 bench lines with the out-of-core roofline.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 2000 python -m pytest tests -q -m gpu -rf --durations=25 -p no:cacheprovider > gpurun_out/tg.log 2>&1; echo "pytest rc=$?"; tail -40 gpurun_out/tg.log | cut -c1-200
for c in cfg5 cfg2; do timeout 600 python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo "$c rc=$?"; done
