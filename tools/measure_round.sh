#!/bin/bash
# Round measurement recipe (under gpurun, 1 GPU).  Usage: bash tools/measure_round.sh <tag>
#   1. profiles (tools/profile.sh: launch list + ncu --set full summaries + DRAM bytes per kernel),
#      whose traffic table then feeds the bench lines' roofline.traffic
#   2. bench lines: CONUS (default command), state, reference arm, shared-GPU 2-rank path
#   3. PIP-stress tile sweep
set -u
TAG=${1:-r02}
mkdir -p gpurun_out
bash tools/profile.sh $TAG > gpurun_out/profile_${TAG}.log 2>&1
[ -f gpurun_out/ncu_traffic_${TAG}.json ] && cp gpurun_out/ncu_traffic_${TAG}.json profiles/ncu_traffic.json
timeout 900 python bench.py > gpurun_out/bench_conus_${TAG}.json 2> gpurun_out/bench_conus_${TAG}.err
timeout 900 python bench.py --config state > gpurun_out/bench_state_${TAG}.json 2> gpurun_out/bench_state_${TAG}.err
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference_${TAG}.json 2> gpurun_out/bench_reference_${TAG}.err
ZH_BENCH_SHARED_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29517 bench.py --gpus 2 --steps 5 --warmup 3 --no-e2e --no-cpu --no-other \
  > gpurun_out/bench_shared2_${TAG}.json 2> gpurun_out/bench_shared2_${TAG}.err
bash tools/pip_stress_sweep.sh $TAG > gpurun_out/sweep_${TAG}.log 2>&1
echo measure done
