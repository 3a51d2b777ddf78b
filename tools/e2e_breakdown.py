"""Where the end-to-end seconds go (CONUS, one GPU): H2D bandwidth of the pinned host raster by
chunking / streams, and the phases of one e2e step through the public API.
python tools/e2e_breakdown.py [config]"""
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
res = {}
dev = torch.empty((cfg.rows, pitch), dtype=torch.int16, device="cuda")
fill_device(cfg.dem, cfg.cols, dev.data_ptr(), 0, 0, cfg.rows, cfg.cols, pitch, torch.cuda.current_stream().cuda_stream)
host = np.empty((cfg.rows, pitch), dtype=np.int16)
cudart = torch.cuda.cudart()
t0 = time.perf_counter()
cudart.cudaHostRegister(host.ctypes.data, host.nbytes, 0)
res["host_register_s"] = time.perf_counter() - t0
th = torch.from_numpy(host)
th.copy_(dev)
torch.cuda.synchronize()
nbytes = host.nbytes


def h2d(nchunks, nstreams):
    streams = [torch.cuda.Stream() for _ in range(nstreams)]
    rows = (cfg.rows + nchunks - 1) // nchunks
    torch.cuda.synchronize()
    t = time.perf_counter()
    for i in range(nchunks):
        s = streams[i % nstreams]
        with torch.cuda.stream(s):
            dev[i * rows:(i + 1) * rows].copy_(th[i * rows:(i + 1) * rows], non_blocking=True)
    torch.cuda.synchronize()
    return nbytes / (time.perf_counter() - t) / 1e9


for nc, ns in [(1, 1), (1, 1)]:
    res[f"h2d_GBps_{nc}chunks_{ns}streams"] = h2d(nc, ns)

del dev
torch.cuda.empty_cache()
res_pin = torch.empty((P.n_poly, cfg.nbins), dtype=torch.int64, pin_memory=True)
out = res_pin.numpy().view(np.uint64)
stream = torch.cuda.current_stream()
for it in range(4):
    ph = {}
    torch.cuda.synchronize()
    t = time.perf_counter()
    z = zh.ZonalHistogram(host, cfg.gt, P, cfg.nbins, lo=cfg.lo, width=cfg.width, nodata=cfg.nodata,
                          oor_drop=cfg.oor_drop, tile=cfg.tile, rows=cfg.rows, cols=cfg.cols, stream=stream)
    torch.cuda.synchronize()
    ph["create"] = time.perf_counter() - t
    t1 = time.perf_counter()
    z.zh_run(out)
    ph["zh_run"] = time.perf_counter() - t1
    st = z.stats()
    t1 = time.perf_counter()
    z.close()
    ph["destroy"] = time.perf_counter() - t1
    ph["total"] = time.perf_counter() - t
    ph["h2d_bytes"] = st["h2d_bytes"]
    ph["h2d_floor_s"] = st["h2d_bytes"] / (res["h2d_GBps_1chunks_1streams"] * 1e9)
    res[f"e2e_{it}"] = ph
print(json.dumps(res, indent=1))
