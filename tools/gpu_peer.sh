#!/bin/bash
# Multi-process siblings on the 1-GPU pool: IPC peer test, bench N=2 (two ranks share cuda:0, gloo)
# with and without NVLink-shared staging (cfg4 at /4 sizes), reference arm line.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 python -m pytest tests/test_gpu_peer.py -q -x > gpurun_out/tg_peer.log 2>&1; tail -30 gpurun_out/tg_peer.log | cut -c1-300
for mode in shared noshared; do
  extra=""; [ $mode = noshared ] && extra="--no-shared-staging"
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
     --master-port 29512 bench.py --gpus 2 --quick --steps 3 --warmup 3 --dist-backend gloo --device-mod 1 \
     --replicate $extra > gpurun_out/bench_n2_$mode.json 2> gpurun_out/bench_n2_$mode.err
  echo "$mode rc=$?"; tail -3 gpurun_out/bench_n2_$mode.err | cut -c1-300
  python -c "
import json; d=json.loads(open('gpurun_out/bench_n2_$mode.json').read().strip().splitlines()[-1]); print('$mode', d['value'], d['e2e'], d['config']['shared_staging'], d['parity'], d.get('replicate'))" 2>&1 | cut -c1-600
done
