#!/bin/bash
# Multi-process siblings with kernel-written flag words: peer tests (2/4 processes, dead peer), N=2 and N=4 bench on one GPU.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_peer.py -q -rf 2>&1 | tail -2
for n in 2 4; do
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 \
   --master-port 2951$n bench.py --gpus $n --quick --steps 3 --warmup 3 --dist-backend gloo --device-mod 1 \
   > gpurun_out/bench_n${n}.json 2> gpurun_out/bench_n${n}.err; echo "n$n rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench_n${n}.json').read().strip().splitlines()[-1]); print('n$n', d['value'], d['e2e']['value'], d['config']['shared_staging'], d['config']['shared_staging_peers'], d['e2e']['p2p_bytes_per_step'], d['parity'])" 2>&1 | cut -c1-400
done
