#!/bin/bash
# Leaf v3 epilogue variants (register-direct st/red vs TMA staging): v3 parity tests and in-HBM TF/s per variant.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
: > gpurun_out/red.log
echo "== default" >> gpurun_out/red.log
NORTHUP_LEAF=4 SZS=8192,32768 timeout 300 python tools/variant_perf.py >> gpurun_out/red.log 2>&1
for so in build/variants_red/*.so; do
  echo "== $so" >> gpurun_out/red.log
  NORTHUP_LIB_PATH=$PWD/$so timeout 300 python -m pytest tests/test_gpu_leaf.py -x -q -k "v3 or integer or closed or accumulate or strided or degenerate" 2>&1 | tail -1 >> gpurun_out/red.log
  NORTHUP_LEAF=4 NORTHUP_LIB_PATH=$PWD/$so SZS=8192,32768 timeout 300 python tools/variant_perf.py >> gpurun_out/red.log 2>&1
done
echo "== default again" >> gpurun_out/red.log
NORTHUP_LEAF=4 SZS=8192,32768 timeout 300 python tools/variant_perf.py >> gpurun_out/red.log 2>&1
cat gpurun_out/red.log
