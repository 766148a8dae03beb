#!/bin/bash
# Round-2 closing evidence (second session): smoke, full GPU suite, the sanitizer paths run
# plainly (compute-sanitizer is closed on the pool), bench lines of every workload, the launch
# list of the default bench command, an ncu --set full capture of the HotSpot leaf.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 > gpurun_out/gputest.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/gputest.log
timeout 300 python tools/sanitize_r2.py > gpurun_out/sanitize_paths.log 2>&1; echo "paths rc=$?"; tail -1 gpurun_out/sanitize_paths.log
for c in cfg3 cfg1 cfg2 cfg4 cfg5 hotspot file; do
  timeout 1500 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/bench_$c.log 2>&1
  echo "$c rc=$?"
  tail -1 gpurun_out/bench_$c.log > gpurun_out/bench_$c.json
done
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "default rc=$?"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/launches_cfg3.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/b_under_ncu.log 2>&1; echo "launch list rc=$?"
python tools/launch_summary.py gpurun_out/launches_cfg3.csv > gpurun_out/launches_cfg3_summary.txt; head -8 gpurun_out/launches_cfg3_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hotspot_kernel_tma -s 2 -c 1 \
    -o gpurun_out/hs_tma -f python tools/hs_ncu.py 8 > gpurun_out/ncu_hs.log 2>&1; echo "ncu hs rc=$?"
ncu -i gpurun_out/hs_tma.ncu-rep --page details > gpurun_out/hotspot_tma_ncu.txt 2>&1
ncu -i gpurun_out/hs_tma.ncu-rep --page raw --csv > gpurun_out/hotspot_tma_raw.csv 2>&1
rm -f gpurun_out/hs_tma.ncu-rep
