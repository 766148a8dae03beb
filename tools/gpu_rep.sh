#!/bin/bash
# replicate_result pushes (GPU tree tests) and the HotSpot bench line (measured link rates, breakdown).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_tree.py tests/test_gpu_hotspot.py -q -x -p no:cacheprovider > gpurun_out/tg_tree.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/tg_tree.log | cut -c1-400
timeout 600 python bench.py --config hotspot > gpurun_out/bench_hotspot.json 2> gpurun_out/bench_hotspot.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/bench_hotspot.json'));print(d['value'],d['e2e_roofline'],d['breakdown'])"
