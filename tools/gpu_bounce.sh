#!/bin/bash
# Pipelined pinned-bounce FILE <-> HBM edge: FILE tests, GDS bench (staging vs direct), bench contract test.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 python -m pytest tests/test_gpu_file.py tests/test_bench_contract.py -q -x -rf > gpurun_out/tg_file.log 2>&1; tail -3 gpurun_out/tg_file.log | cut -c1-300
timeout 600 python tools/gds_bench.py 16384 > gpurun_out/gds.log 2>&1; echo "gds rc=$?"; tail -2 gpurun_out/gds.log | cut -c1-300
