#!/bin/bash
# Round-end check: smoke, full GPU suite, the default bench line, HotSpot and cfg1 lines, reference arm.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 2000 python -m pytest tests -q -m gpu -rf -p no:cacheprovider > gpurun_out/tg.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/tg.log | cut -c1-200
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench rc=$?"
timeout 900 python bench.py --config hotspot > gpurun_out/bench_hs.json 2> gpurun_out/bench_hs.err; echo "hs rc=$?"
timeout 900 python bench.py --config cfg1 > gpurun_out/bench_cfg1.json 2> gpurun_out/bench_cfg1.err; echo "cfg1 rc=$?"
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$?"
