#!/bin/bash
# A/B of libzh builds on the bench step (no e2e / CPU / other path).  Usage: tools/ab_bench.sh tag lib1 [lib2 ...]
# ("default" = the in-tree build; BENCH_ARGS="--config pip-stress" etc. passed to bench.py).
# Lines go to gpurun_out/ab_<tag>.txt.
TAG=$1; shift
mkdir -p gpurun_out
for L in "$@"; do
  if [ "$L" = default ]; then unset ZH_LIBZH; else export ZH_LIBZH=$PWD/$L; fi
  timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu --no-other $BENCH_ARGS > gpurun_out/ab_tmp.json 2>gpurun_out/ab_tmp.err
  python - "$L" <<'PY' >> gpurun_out/ab_${TAG}.txt
import json, sys
try:
    d = json.loads(open("gpurun_out/ab_tmp.json").read().strip().splitlines()[-1])
    s = d["steps_detail"]
    print(sys.argv[1], "ms/step %.3f" % d["ms_per_step"], " ".join("%s=%.3f" % (k, v["ms"]) for k, v in s.items()))
except Exception as e:
    print(sys.argv[1], "FAILED", e, open("gpurun_out/ab_tmp.err").read()[-500:])
PY
done
