#!/bin/bash
# HotSpot: iterations per launch with the q-in-registers 16 x 8 leaf (limit raised for the run only).
H=paper_conf_ipps_chey19_b200/csrc/northup_internal.h
cp $H /tmp/h_orig.h
sed -i 's/constexpr int kHotspotMaxIters = 8; /constexpr int kHotspotMaxIters = 16;/' $H
python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1 || tail -3 /tmp/b.log
LIS=6,8,10,12,8 timeout 600 python tools/hs_leaf_iters.py
cp /tmp/h_orig.h $H
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
