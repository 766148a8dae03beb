#!/bin/bash
# Round-2 bench lines of every workload (one GPU), each into gpurun_out/bench_<cfg>.json.
mkdir -p gpurun_out
for c in cfg3 cfg1 cfg2 cfg4 cfg5 hotspot file; do
  timeout 1500 python bench.py --config $c --steps 3 --warmup 3 > gpurun_out/bench_$c.log 2>&1
  echo "$c rc=$?"
  tail -1 gpurun_out/bench_$c.log > gpurun_out/bench_$c.json
done
