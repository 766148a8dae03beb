#!/bin/bash
# Leaf v3 with A_hi in TMEM (NU_LEAF3_AHI_TMEM): bitwise vs the default build, leaf tests, TF/s, profile mode.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
NORTHUP_LEAF=4 timeout 300 python tools/presplit_probe.py v3 2048 2304 4096
NORTHUP_LEAF=4 NORTHUP_LIB_PATH=$PWD/build/ah/ah.so timeout 300 python tools/presplit_probe.py ah 2048 2304 4096
python -c "
import numpy as np
a, b = (np.load(f'gpurun_out/C_{t}.npy') for t in ('v3', 'ah'))
print('ah==v3', np.array_equal(a, b), float(np.abs(a - b).max()))"
NORTHUP_LIB_PATH=$PWD/build/ah/ah.so timeout 300 python -m pytest tests/test_gpu_leaf.py -q 2>&1 | tail -1
for so in default build/ah/ah.so; do echo "== $so"; if [ $so = default ]; then unset NORTHUP_LIB_PATH; else export NORTHUP_LIB_PATH=$PWD/$so; fi
LEAF_VARIANT=4 timeout 200 python tools/mma_prof.py 2>&1 | tail -1 | cut -c1-250; done
