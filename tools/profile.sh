#!/bin/bash
# Profiling recipe (run under gpurun).  Usage: tools/profile.sh <tag> [config]
#   1. launch list of the bench command (cold-cache, serialised: compare shares, not absolutes)
#   2. ncu --set full of the step kernels (one launch each) with source correlation
set -u
TAG=${1:-r01}; CFG=${2:-conus}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --config ${CFG} --steps 2 --warmup 1 --no-e2e --no-cpu > gpurun_out/launches_${TAG}.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_tile_hist|k_pip|k_aggregate" -s 3 -c 3 \
    -o gpurun_out/full_${TAG} -f python bench.py --config ${PROF_CFG:-state} --steps 1 --warmup 1 --no-e2e --no-cpu \
    > gpurun_out/full_${TAG}.log 2>&1
echo profile done
