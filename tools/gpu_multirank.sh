#!/bin/bash
# N=2 bench path on ONE GPU: two ranks share cuda:0, gloo process group (test mode)
mkdir -p gpurun_out
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
   --master-port 29512 bench.py --gpus 2 --quick --steps 3 --warmup 3 --dist-backend gloo --device-mod 1 \
   --replicate > gpurun_out/bench_n2.json 2> gpurun_out/bench_n2.err
echo rc=$? >> gpurun_out/bench_n2.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 --ref-step-s 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
