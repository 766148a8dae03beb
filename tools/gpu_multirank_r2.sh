#!/bin/bash
# Round-2 code on the N > 1 bench path, ranks sharing the one GPU (gloo process group):
# N = 2 at full cfg4 size, N = 4 and 8 at quick size with --replicate; the reference arm.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_hotspot.py -q -x -p no:cacheprovider -k concurrent > gpurun_out/tg_hs2.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/tg_hs2.log
timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
   --master-port 29512 bench.py --gpus 2 --steps 3 --warmup 3 --dist-backend gloo --device-mod 1 \
   > gpurun_out/bench_n2_full.json 2> gpurun_out/bench_n2_full.err; echo "n2 full rc=$?"
for n in 4 8; do
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 \
   --master-port 2952$n bench.py --gpus $n --quick --steps 3 --warmup 3 --dist-backend gloo --device-mod 1 \
   --replicate > gpurun_out/bench_n${n}_quick.json 2> gpurun_out/bench_n${n}_quick.err; echo "n$n quick rc=$?"
done
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 --ref-step-s 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$?"
for f in gpurun_out/bench_n2_full.json gpurun_out/bench_n4_quick.json gpurun_out/bench_n8_quick.json gpurun_out/bench_ref.json; do
  python -c "import json,sys;d=json.loads(open('$f').read().strip().splitlines()[-1]);print('$f',d.get('value'),d.get('n_gpus'),d.get('e2e',{}).get('value'),d.get('parity'),d.get('replicate'))" 2>&1 | cut -c1-400
done
