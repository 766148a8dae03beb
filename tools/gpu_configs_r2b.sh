#!/bin/bash
# Bench lines of the other workloads with the closing code (one GPU).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in cfg1 cfg2 cfg4 cfg5 file; do
  timeout 1500 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/bench_$c.log 2>&1
  echo "$c rc=$?"
  tail -1 gpurun_out/bench_$c.log > gpurun_out/bench_$c.json
done
