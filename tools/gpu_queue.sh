#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_tree.py -q -x > gpurun_out/tg_tree.log 2>&1; tail -15 gpurun_out/tg_tree.log | cut -c1-400
timeout 900 python tools/queue_bench.py 16384 16384 > gpurun_out/queue_bench.log 2>&1; cat gpurun_out/queue_bench.log | cut -c1-400
