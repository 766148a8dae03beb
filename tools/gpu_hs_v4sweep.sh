#!/bin/bash
# HotSpot v4 CTA-shape sweep (2 CTAs/SM variants), bitwise tests per variant; N=2 multi-process bench check.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for v in 3 4; do echo "default v$v:"; NORTHUP_HS_LEAF=$v HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | cut -c1-420; done
for f in build/hsvar4/*.so; do echo "$f:"; NORTHUP_LIB_PATH=$f NORTHUP_HS_LEAF=4 timeout 300 python -m pytest tests/test_gpu_hotspot.py -q -x -k "variants_bitwise and 4" 2>&1 | tail -1
  NORTHUP_LIB_PATH=$f NORTHUP_HS_LEAF=4 HS_IN_HBM_ONLY=1 timeout 300 python tools/hotspot_perf.py 16384 64 2>&1 | tail -1 | cut -c1-420; done
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
   --master-port 29512 bench.py --gpus 2 --quick --steps 3 --warmup 3 --dist-backend gloo --device-mod 1 \
   > gpurun_out/bench_n2_shared.json 2> gpurun_out/bench_n2_shared.err; echo "n2 rc=$?"; tail -c 1500 gpurun_out/bench_n2_shared.json
