#!/bin/bash
# HotSpot TMA leaf: warps x rows-per-lane variants built on the box (q in registers).
F=paper_conf_ipps_chey19_b200/csrc/hotspot.cu
cp $F /tmp/hotspot_orig.cu
for shape in "12 10" "12 11" "16 8" "16 7" "8 15"; do
  set -- $shape
  sed -i "s/constexpr int kPW = [0-9]*, kPV = [0-9]*, kPRH/constexpr int kPW = $1, kPV = $2, kPRH/" $F
  python -c "import __graft_entry__ as g; g.build()" > /tmp/b.log 2>&1 || { echo "build $shape failed"; tail -3 /tmp/b.log; continue; }
  echo "$shape: $(HS_VARIANTS=tma HS_N=32768 timeout 300 python tools/hs_variants.py | tail -1)"
done
cp /tmp/hotspot_orig.cu $F
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
