"""Size of the sparse histogram reduction (dist.SparseReducer) of the N-GPU decomposition, from the
real step-2 pairs of each work-balanced strip (one GPU; only step 2 runs, the raster is not read):
polygons spanning strips, rows put on the fabric per step (sparse vs dense), and the bytes rank 0
receives.  python tools/sparse_reduce_plan.py [config] > profiles/r01/sparse_reduce_plan_conus.json"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangw14_b200 import zh  # noqa: E402
from paper_conf_ipps_zhangw14_b200.dist import plan_shards, sparse_plan, touched_polygons  # noqa: E402
from synth.configs import CONFIGS  # noqa: E402

cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "conus"]
P = cfg.polygons()
pitch = (cfg.cols + 7) // 8 * 8
r = torch.empty((cfg.rows, pitch), dtype=torch.int16, device="cuda")  # contents unused (step 2 only)
row_bytes = cfg.nbins * 8
res = {"config": cfg.name, "n_poly": P.n_poly, "row_bytes": row_bytes}
for n in (2, 4, 8):
    b = plan_shards(cfg.rows, cfg.cols, cfg.gt, P, cfg.tile, n, balanced=True)
    t = np.zeros((n, P.n_poly), bool)
    for s in range(n):
        if b[s + 1] > b[s]:
            with zh.ZonalHistogram(r[b[s]:b[s + 1]], cfg.gt, P, cfg.nbins, tile=cfg.tile, rows=cfg.rows,
                                   cols=cfg.cols, row0=b[s], nodata=cfg.nodata) as z:
                z.zh_pair_tiles()
                t[s, touched_polygons(z)] = True
    shared, owned = sparse_plan(t)
    # reduce form: shared rows go through an NCCL reduce over all ranks, owned rows of ranks != 0
    # are sent to rank 0 once; the dense reduce moves all n_poly rows through every link.
    rank0_in = (len(shared) + sum(len(o) for o in owned[1:])) * row_bytes
    res[str(n)] = {"bounds": [int(x) for x in b], "shared_polys": int(len(shared)),
                   "owned_per_rank": [int(len(o)) for o in owned],
                   "untouched": int(P.n_poly - len(shared) - sum(len(o) for o in owned)),
                   "sparse_reduce_bytes": int(len(shared) * row_bytes),
                   "p2p_bytes_to_rank0": int(sum(len(o) for o in owned[1:]) * row_bytes),
                   "dense_reduce_bytes": int(P.n_poly * row_bytes),
                   "rank0_ingress_bytes_sparse_upper": int(rank0_in)}
print(json.dumps(res, indent=1))
