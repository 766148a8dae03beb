#!/bin/bash
mkdir -p gpurun_out
for c in cfg1 cfg2 cfg5 cfg4; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --cpu-budget 5 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
