#!/bin/bash
# Profiling recipe (run under gpurun, 1 GPU).  Usage: tools/profile.sh <tag>
#   1. launch list of the bench command (ncu --metrics gpu__time_duration.sum, cold-cache and
#      serialised: compare per-kernel SHARES of the step, not absolutes)
#   2. ncu --set full of the step kernels on the CONUS config (one launch each, source-correlated)
set -u
TAG=${1:-r01}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > gpurun_out/launches_${TAG}.log 2>&1
#    (step 1 four-step: k_tile_hist, k_aggregate, k_parity, k_pip_cells; step 2 fused: k_fused_pure,
#    k_parity, k_pip_cells)
timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"k_tile_hist|k_aggregate|k_parity|k_pip_cells|k_fused_pure|k_mixed_cells|k_touch" \
    -c 7 -o gpurun_out/full_${TAG} -f python tools/prof_step.py conus 256 2 four_fused > gpurun_out/full_${TAG}.log 2>&1
echo profile done
