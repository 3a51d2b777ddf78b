"""Small end-to-end runs for compute-sanitizer (memcheck / racecheck / synccheck): tiny config,
both paths, a ragged tile size, the CUDA-graph step, the zonal statistics / summary and the
histogram distances (pair lists and all pairs, both product widths).  python tools/sanitize.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangw14_b200 import zh  # noqa: E402
from synth.configs import TINY as cfg  # noqa: E402
from synth.dem import fill_device  # noqa: E402

P = cfg.polygons()
t = torch.empty((cfg.rows, cfg.cols), dtype=torch.int16, device="cuda")
fill_device(cfg.dem, cfg.cols, t.data_ptr(), 0, 0, cfg.rows, cfg.cols, cfg.cols, torch.cuda.current_stream().cuda_stream)
res = []
for tile, fused in ((128, False), (128, True), (100, True), (100, False)):
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=tile, nodata=cfg.nodata, fused=fused) as z:
        res.append(z.run())
        z.zh_zonal_stats()
        z.zh_zonal_summary()
        for kind in ("l1", "emd", "chi2"):
            z.zh_hist_distance(kind)
            z.zh_hist_distance(kind, [0, 3, 15], [1, 3, 2])
        for _ in range(3):  # direct, captured, replayed
            z.zh_step_graph()
        res.append(z.output_device().cpu().numpy().view(np.uint64).copy())
os.environ["ZH_DIST_WIDE"] = "1"
with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=128, nodata=cfg.nodata) as z:
    z.run()
    for kind in ("l1", "emd", "chi2"):
        z.zh_hist_distance(kind)
del os.environ["ZH_DIST_WIDE"]
assert all((r == res[0]).all() for r in res)
cov = []
for tile, fused in ((128, True), (100, False)):  # cover mode (R15): k_touch on top of the split step 4
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=tile, nodata=cfg.nodata, fused=fused, cover=True) as z:
        cov.append(z.run())
assert (cov[0] == cov[1]).all() and (cov[0] >= res[0]).all()
print("sanitize run ok", int(res[0].sum()))
