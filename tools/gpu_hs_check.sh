#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 300 python tools/hs_perlaunch.py
timeout 300 python tools/hs_block_seq.py
timeout 900 python -m pytest tests/test_gpu_hotspot.py -q -x -p no:cacheprovider > gpurun_out/tg_hs.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/tg_hs.log
HS_VARIANTS=tma HS_N=32768 timeout 300 python tools/hs_variants.py | tail -1
timeout 600 python bench.py --config hotspot > gpurun_out/bench_hotspot.json 2> gpurun_out/bench_hotspot.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/bench_hotspot.json'));print(d['value'],d['in_hbm'],d['slowdown_pct_vs_in_hbm'],d['e2e_roofline'],d['breakdown'],d['roofline']['frac'],d['clocks'])"
