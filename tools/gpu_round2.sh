#!/bin/bash
# Full check after the peer-protocol change: smoke, all GPU tests, N=2 bench (shared), default bench line.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/tg.log 2>&1; tail -3 gpurun_out/tg.log
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
   --master-port 29512 bench.py --gpus 2 --quick --steps 3 --warmup 3 --dist-backend gloo --device-mod 1 \
   > gpurun_out/bench_n2_shared.json 2> gpurun_out/bench_n2_shared.err; echo "n2 rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/bench_n2_shared.json').read().strip().splitlines()[-1]); print('n2', d['value'], d['e2e'], d['config']['shared_staging'], d['config']['shared_staging_peers'], d['parity'])" 2>&1 | cut -c1-600
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_full.json').read().strip().splitlines()[-1]); print('bench', d['value'], d['e2e']['value'], d['slowdown_pct_vs_in_hbm'], d['roofline']['frac'], d['clocks'])"
