#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_tree.py -q -x -p no:cacheprovider -k "finalize_measures" 2>&1 | tail -1
for i in 1 2 3; do
python - <<'PY'
import paper_conf_ipps_chey19_b200 as nu, time
t0 = time.perf_counter()
t, _ = nu.host_tree(1, 8 << 30); t.finalize()
print("links", t.link_info(), "finalize_s", round(time.perf_counter() - t0, 2), "plan r1", t.plan(32768, 32768, 32768).stats()["bfirst_rows"])
t.destroy()
PY
done
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "default rc=$?"
python -c "
import json
d=json.loads(open('gpurun_out/bench_default.json').read().strip().splitlines()[-1]); print(d['value'], d['config']['links_at_finalize'], d['config'].get('bfirst_rows'), d['clocks']['sm_mhz'])"
