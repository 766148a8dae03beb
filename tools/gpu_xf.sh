#!/bin/bash
# Leaf v3 split-warp variants: parity subset, TF/s at 8192^3 / 32768^3, profile-mode breakdown.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
: > gpurun_out/xf.log
for so in default build/variants_xf/x16e4.so build/variants_xf/x16e8.so build/variants_xf/x16e8_rs4b1.so default; do
  echo "== $so" >> gpurun_out/xf.log
  if [ "$so" = default ]; then unset NORTHUP_LIB_PATH; else export NORTHUP_LIB_PATH=$PWD/$so; fi
  timeout 300 python -m pytest tests/test_gpu_leaf.py -x -q -k "v3 or integer" 2>&1 | tail -1 >> gpurun_out/xf.log
  NORTHUP_LEAF=4 SZS=8192,32768 timeout 300 python tools/variant_perf.py >> gpurun_out/xf.log 2>&1
  LEAF_VARIANT=4 timeout 200 python tools/mma_prof.py 2>&1 | tail -1 | cut -c1-260 >> gpurun_out/xf.log
done
unset NORTHUP_LIB_PATH
cat gpurun_out/xf.log
