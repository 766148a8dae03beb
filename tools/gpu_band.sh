#!/bin/bash
mkdir -p gpurun_out; : > gpurun_out/band.log
for b in 8 16 32 64 128; do
  echo "band $b" >> gpurun_out/band.log
  NORTHUP_RASTER_BAND=$b SZS=32768 timeout 300 python tools/variant_perf.py >> gpurun_out/band.log 2>&1
done
for pc in 2 4; do
  echo "panel_chunks $pc" >> gpurun_out/band.log
  NORTHUP_PANEL_CHUNKS=$pc SZS=32768 timeout 300 python tools/variant_perf.py >> gpurun_out/band.log 2>&1
done
cat gpurun_out/band.log
