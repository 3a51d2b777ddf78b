#!/bin/bash
# PIP-stress config (BASELINE.json configs[4]): 50k jagged polygons over the CONUS raster, tile sweep.
# Usage (under gpurun): bash tools/pip_stress_sweep.sh <tag>
TAG=${1:-r01}
mkdir -p gpurun_out
for T in 64 128 256 512 1024; do
  OTHER=""
  if [ "$T" = "64" ]; then OTHER="--no-other"; fi   # the four-step path would need 98.8 GB of tile histograms
  timeout 900 python bench.py --config pip-stress --tile $T --steps 5 --warmup 3 --no-e2e --no-cpu $OTHER \
     > gpurun_out/pipstress_${TAG}_T${T}.json 2> gpurun_out/pipstress_${TAG}_T${T}.err
  echo "T=$T rc=$?"
done
