#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_leaf.py tests/test_gpu_tree.py tests/test_gpu_configs.py -q -x -p no:cacheprovider 2>&1 | tail -2
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/launches_cfg3.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/b_under_ncu.log 2>&1; echo "launch list rc=$?"
python tools/launch_summary.py gpurun_out/launches_cfg3.csv > gpurun_out/launches_cfg3_summary.txt; head -8 gpurun_out/launches_cfg3_summary.txt
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "default rc=$?"
python -c "
import json
d=json.loads(open('gpurun_out/bench_default.json').read().strip().splitlines()[-1]); print(d['value'], d['in_hbm']['value'], d['roofline']['frac'], d['clocks']['sm_mhz'], d['config']['links_at_finalize']['pcie_gbs'])"
