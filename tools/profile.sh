#!/bin/bash
# Profiling recipe (run under gpurun, 1 GPU).  Usage: tools/profile.sh <tag>
#   1. launch list of the bench command (ncu --metrics gpu__time_duration.sum, cold-cache and
#      serialised: compare per-kernel SHARES of the step, not absolutes)
#   2. ncu --set full of the step kernels (one launch each, source-correlated): CONUS fused and
#      four-step (T = 256), state fused, PIP-stress fused (T = 256)
set -u
TAG=${1:-r02}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/launches_${TAG}.log 2>&1
K='k_tile_hist|k_aggregate|k_parity|k_pip_cells|k_fused_pure|k_mixed_cells|k_mbb_edges|k_classify|k_mark|k_poly_bands'
for spec in "conus 256 fused" "conus 256 four_step" "state 256 fused" "pip-stress 256 fused"; do
  set -- $spec
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$K" -c 12 \
      -o gpurun_out/full_${TAG}_$1_$3 -f python tools/prof_step.py $1 $2 1 $3 > gpurun_out/full_${TAG}_$1_$3.log 2>&1
done

# summaries on the box (the reports are large; gpurun copies back at most 64 MiB)
for spec in "conus 256 fused" "conus 256 four_step" "state 256 fused" "pip-stress 256 fused"; do
  set -- $spec
  R=gpurun_out/full_${TAG}_$1_$3.ncu-rep
  { python tools/ncu_summary.py $R
    for k in k_fused_pure k_mixed_cells k_parity k_tile_hist k_aggregate k_pip_cells k_mbb_edges k_classify; do
      echo "### $k"; python tools/src_hotspots.py $R $k 12 2>/dev/null; done; } > gpurun_out/ncu_full_${TAG}_$1_$3.txt
  ZH_TRAFFIC_JSON=gpurun_out/ncu_traffic_${TAG}.json python tools/ncu_traffic.py $R $1 $2 $3
done
python tools/launch_summary.py gpurun_out/launches_${TAG}.csv 'zhs_fill|FillFunctor' > gpurun_out/launches_summary_${TAG}.txt
rm -f gpurun_out/full_${TAG}_conus_four_step.ncu-rep gpurun_out/full_${TAG}_state_fused.ncu-rep gpurun_out/full_${TAG}_pip-stress_fused.ncu-rep
echo summaries done
