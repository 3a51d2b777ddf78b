"""Mixed-tile statistics of a config's step-2 pair lists (how many cell-in-polygon pairs share a tile).
python tools/mixed_stats.py [config] [tile]"""
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangw14_b200 import zh  # noqa: E402
from synth.configs import CONFIGS  # noqa: E402

cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "conus"]
T = int(sys.argv[2]) if len(sys.argv) > 2 else cfg.tile
P = cfg.polygons()
pitch = (cfg.cols + 7) // 8 * 8
r = torch.empty((cfg.rows, pitch), dtype=torch.int16, device="cuda")  # geometry only: values never read
z = zh.ZonalHistogram(r, cfg.gt, P, cfg.nbins, tile=T, rows=cfg.rows, cols=cfg.cols, nodata=cfg.nodata)
z.zh_pair_tiles()
inside, isect = z.pairs_host()
mixed = collections.Counter(np.asarray(isect)[:, 0].tolist())
ins_mixed = sum(1 for t in np.asarray(inside)[:, 0].tolist() if t in mixed)
dist = collections.Counter(mixed.values())
print({"config": cfg.name if hasattr(cfg, "name") else sys.argv[1], "tile": T, "n_isect": len(isect),
       "n_inside": len(inside), "mixed_tiles": len(mixed), "inside_pairs_of_mixed_tiles": ins_mixed,
       "pairs_per_mixed_tile": dict(sorted(dist.items())),
       "groups_of_2": sum((c + 1) // 2 for c in mixed.values())})
