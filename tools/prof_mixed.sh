#!/bin/bash
# ncu --set full of the fused step's kernels on CONUS (tag = $1), one launch each
T=${1:-mix}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_mixed_cells|k_fused_pure|k_parity" -c 3 \
  -o gpurun_out/full_$T -f python tools/prof_step.py conus 256 1 fused > gpurun_out/full_$T.log 2>&1
