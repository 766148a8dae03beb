#!/bin/bash
# HotSpot out-of-core block-size sweep (32768^2 x 256, 8 GiB cap).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for b in 0 10944 16384; do echo "block $b:"; HS_BLOCK=$b timeout 600 python tools/hotspot_perf.py 32768 256 8 2>&1 | grep "'block'" | cut -c1-400; done
