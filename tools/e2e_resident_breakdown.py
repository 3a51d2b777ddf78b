"""Where SURVEY.md §8d's end-to-end time goes (raster resident in HBM, host polygons -> host
histogram): zh_create (validation + polygon H2D), zh_run (step 2 + fused update + result D2H),
zh_destroy.  python tools/e2e_resident_breakdown.py [config]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangw14_b200 import zh  # noqa: E402
from synth.configs import CONFIGS  # noqa: E402
from synth.dem import fill_device  # noqa: E402

cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "conus"]
P = cfg.polygons()
pitch = (cfg.cols + 7) // 8 * 8
dev = torch.empty((cfg.rows, pitch), dtype=torch.int16, device="cuda")
fill_device(cfg.dem, cfg.cols, dev.data_ptr(), 0, 0, cfg.rows, cfg.cols, pitch, torch.cuda.current_stream().cuda_stream)
cudart = torch.cuda.cudart()
for a in (P.x, P.y):
    cudart.cudaHostRegister(a.ctypes.data, a.nbytes, 0)
res_pin = torch.empty((P.n_poly, cfg.nbins), dtype=torch.int64, pin_memory=True)
out = res_pin.numpy().view(np.uint64)
stream = torch.cuda.current_stream()
res = {}
for it in range(5):
    ph = {}
    torch.cuda.synchronize()
    t = time.perf_counter()
    z = zh.ZonalHistogram(dev, cfg.gt, P, cfg.nbins, lo=cfg.lo, width=cfg.width, nodata=cfg.nodata,
                          oor_drop=cfg.oor_drop, tile=cfg.tile, rows=cfg.rows, cols=cfg.cols, stream=stream)
    ph["create_ms"] = 1e3 * (time.perf_counter() - t)
    t1 = time.perf_counter()
    z.zh_pair_tiles()
    z.zh_fused_update()
    torch.cuda.synchronize()
    ph["step_ms"] = 1e3 * (time.perf_counter() - t1)
    t1 = time.perf_counter()
    h = z.output_device()
    res_pin.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    ph["d2h_ms"] = 1e3 * (time.perf_counter() - t1)
    t1 = time.perf_counter()
    z.close()
    ph["destroy_ms"] = 1e3 * (time.perf_counter() - t1)
    ph["total_ms"] = 1e3 * (time.perf_counter() - t)
    res[f"e2e_{it}"] = ph
print(json.dumps(res, indent=1))
