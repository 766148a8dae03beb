#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
for v in 3 1 2; do for tool in memcheck racecheck synccheck; do
  NORTHUP_HS_LEAF=$v timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize2.py > gpurun_out/sanitize2_v${v}_$tool.log 2>&1
  echo "v$v $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize2 run ok' gpurun_out/sanitize2_v${v}_$tool.log | tr '\n' ' ')"
done; done
