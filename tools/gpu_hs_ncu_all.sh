#!/bin/bash
mkdir -p gpurun_out
bash tools/gpu_hs_ncu.sh
bash tools/gpu_hs_ncu32k.sh
