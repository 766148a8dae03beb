#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for tool in memcheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize3.py > gpurun_out/sanitize3_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize3_$tool.log
  tail -n 4 gpurun_out/sanitize3_$tool.log
done
