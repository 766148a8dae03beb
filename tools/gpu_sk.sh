#!/bin/bash
# Leaf v3 skewed issue variant: leaf tests, TF/s, profile-mode breakdown vs default.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
: > gpurun_out/sk.log
for so in default build/variants_sk/sk1.so default build/variants_sk/sk1.so; do
  echo "== $so" >> gpurun_out/sk.log
  if [ "$so" = default ]; then unset NORTHUP_LIB_PATH; else export NORTHUP_LIB_PATH=$PWD/$so; fi
  timeout 300 python -m pytest tests/test_gpu_leaf.py -q -rf 2>&1 | tail -4 >> gpurun_out/sk.log
  NORTHUP_LEAF=4 SZS=8192,32768 timeout 300 python tools/variant_perf.py >> gpurun_out/sk.log 2>&1
  LEAF_VARIANT=4 timeout 200 python tools/mma_prof.py 2>&1 | tail -1 | cut -c1-260 >> gpurun_out/sk.log
done
unset NORTHUP_LIB_PATH
cat gpurun_out/sk.log
