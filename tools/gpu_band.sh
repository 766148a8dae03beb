#!/bin/bash
# Raster band width of the x3 leaf: time (x3_prof) and DRAM bytes of one reduce-add panel launch (ncu).
mkdir -p gpurun_out
for band in 16 32 64; do
  sed -i "s/constexpr int kRasterBand = [0-9]*;/constexpr int kRasterBand = $band;/" paper_conf_ipps_chey19_b200/csrc/northup_internal.h
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
  echo "band $band: $(timeout 300 python tools/x3_prof.py 2>/dev/null | tail -1)"
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:leaf_x3 -s 1 -c 1 python tools/ncu_x3.py 2>/dev/null | grep -E "dram__bytes|gpu__time" 
done
