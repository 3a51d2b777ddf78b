"""Simulate the N-GPU decomposition on one GPU: time each shard's step (the bench's: pair_tiles +
fused update replayed from the context's CUDA graph, over the polygons whose bounding box meets the
strip — dist.strip_polygons) separately and report max / mean per N, for equal and work-balanced
(zh_plan_rows) strips.  The max over shards is the compute part of an N-GPU step (the NCCL reduce
is not included).  python tools/shard_sim.py [config]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangw14_b200 import zh  # noqa: E402
from paper_conf_ipps_zhangw14_b200.dist import plan_shards, strip_polygons  # noqa: E402
from synth.configs import CONFIGS  # noqa: E402
from synth.dem import fill_device  # noqa: E402

cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "conus"]
P = cfg.polygons()
pitch = (cfg.cols + 7) // 8 * 8
r = torch.empty((cfg.rows, pitch), dtype=torch.int16, device="cuda")
fill_device(cfg.dem, cfg.cols, r.data_ptr(), 0, 0, cfg.rows, cfg.cols, pitch, torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
res = {}
for n in (1, 2, 4, 8):
    for mode in ("equal", "balanced"):
        if n == 1 and mode == "balanced":
            continue
        b = plan_shards(cfg.rows, cfg.cols, cfg.gt, P, cfg.tile, n, balanced=(mode == "balanced"))
        times = []
        for s in range(n):
            if b[s + 1] == b[s]:
                times.append(0.0)
                continue
            Ps = P.subset(strip_polygons(P, cfg.gt, b[s], b[s + 1])) if n > 1 else P
            with zh.ZonalHistogram(r[b[s]:b[s + 1]], cfg.gt, Ps, cfg.nbins, tile=cfg.tile, rows=cfg.rows,
                                   cols=cfg.cols, row0=b[s], nodata=cfg.nodata) as z:
                best = 1e9
                for _ in range(2):  # direct (learns the sizes), captured
                    z.zh_step_graph()
                for _ in range(3):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    torch.cuda.synchronize()
                    e0.record()
                    z.zh_step_graph()
                    e1.record()
                    torch.cuda.synchronize()
                    best = min(best, e0.elapsed_time(e1))
                times.append(best)
        res[f"{n}_{mode}"] = {"bounds": b, "ms": times, "max_ms": max(times), "mean_ms": sum(times) / n}
        print(n, mode, "max %.3f mean %.3f" % (max(times), sum(times) / n), [round(t, 2) for t in times], flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/shard_sim.json", "w"), indent=1)
