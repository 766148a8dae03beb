#!/bin/bash
# Leaf v3 L2 cache-policy variants: parity subset, TF/s, DRAM bytes of one cfg3 K-panel reduce launch.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
: > gpurun_out/l2hint.log
for so in default build/variants_l2/h1.so build/variants_l2/h2.so build/variants_l2/h3.so; do
  echo "== $so" >> gpurun_out/l2hint.log
  if [ "$so" = default ]; then unset NORTHUP_LIB_PATH; else export NORTHUP_LIB_PATH=$PWD/$so; fi
  timeout 300 python -m pytest tests/test_gpu_leaf.py -x -q -k "v3 or integer" 2>&1 | tail -1 >> gpurun_out/l2hint.log
  NORTHUP_LEAF=4 SZS=8192,32768 timeout 300 python tools/variant_perf.py >> gpurun_out/l2hint.log 2>&1
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
     --clock-control none -k regex:leaf_gemm -s 1 -c 1 --csv python tools/ncu_leaf.py 32768 2>/dev/null | grep -E "dram__|gpu__time|lts__" >> gpurun_out/l2hint.log
done
unset NORTHUP_LIB_PATH
cat gpurun_out/l2hint.log
