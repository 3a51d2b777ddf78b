"""One hot-path step of a config, for ncu (python tools/prof_step.py [config] [tile])."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangw14_b200 import zh  # noqa: E402
from synth.configs import CONFIGS  # noqa: E402
from synth.dem import fill_device  # noqa: E402

cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "conus"]
T = int(sys.argv[2]) if len(sys.argv) > 2 else cfg.tile
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
path = sys.argv[4] if len(sys.argv) > 4 else "four_step"
P = cfg.polygons()
pitch = (cfg.cols + 7) // 8 * 8
r = torch.empty((cfg.rows, pitch), dtype=torch.int16, device="cuda")
fill_device(cfg.dem, cfg.cols, r.data_ptr(), 0, 0, cfg.rows, cfg.cols, pitch, torch.cuda.current_stream().cuda_stream)
z = zh.ZonalHistogram(r, cfg.gt, P, cfg.nbins, tile=T, cols=cfg.cols, nodata=cfg.nodata)
for i in range(steps):
    z.zh_pair_tiles()
    if path == "fused" or (path == "four_fused" and i % 2 == 1):
        z.zh_fused_update()
    else:
        z.zh_tile_hist()
        z.zh_aggregate()
        z.zh_pip_update()
torch.cuda.synchronize()
print("stats", z.stats())
