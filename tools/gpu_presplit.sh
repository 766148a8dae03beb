#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
NORTHUP_LEAF=4 timeout 300 python tools/presplit_probe.py v3 2048 2304 4096
NORTHUP_LEAF=2 timeout 300 python tools/presplit_probe.py v12 2048 2304 4096
NORTHUP_LEAF=2 NORTHUP_LIB_PATH=$PWD/build/ps/ps.so timeout 300 python tools/presplit_probe.py ps 2048 2304 4096
python -c "
import numpy as np
a, b, c = (np.load(f'gpurun_out/C_{t}.npy') for t in ('v3', 'v12', 'ps'))
print('v3==v12', np.array_equal(a, b), 'ps==v12', np.array_equal(c, b), 'max|ps-v12|', float(np.abs(c - b).max()))"
