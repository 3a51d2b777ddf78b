"""Full-size GPU parity (BASELINE.json state-scale and CONUS-scale configs, the bench's launch
configuration): sampled per-polygon histograms vs the oracle (computed one polygon at a time on
the polygon's raster window; BASELINE.json configs [1], [2] and [4]), plus properties that hold at any size — tile-size invariance,
force-all-intersect invariance, and (state tiling covers the extent) the partition identity
sum_k H_k == global histogram of the mapped raster."""
import numpy as np
import pytest

import oracle
from synth.configs import CONUS, PIPSTRESS, STATE
from synth.dem import fill_device, fill_host

pytestmark = pytest.mark.gpu


def _raster(cfg):
    import torch
    pitch = (cfg.cols + 7) // 8 * 8
    t = torch.empty((cfg.rows, pitch), dtype=torch.int16, device="cuda")
    fill_device(cfg.dem, cfg.cols, t.data_ptr(), 0, 0, cfg.rows, cfg.cols, pitch,
                torch.cuda.current_stream().cuda_stream)
    return t


def _run(t, cfg, P, **kw):
    """Four-step path and fused path; both must agree; returns the fused result and stats."""
    from paper_conf_ipps_zhangw14_b200 import zh
    tile = kw.pop("tile", cfg.tile)
    res = []
    for fused in (False, True):
        with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=tile, cols=cfg.cols, nodata=cfg.nodata,
                               fused=fused, **kw) as z:
            res.append(z.run())
            st = z.stats()
    assert (res[0] == res[1]).all(), "fused path differs from the four-step path"
    return res[1], st


def _sample_polys(P, n, seed):
    rng = np.random.default_rng(seed)
    nv = np.diff(P.ring_vert_off)[P.poly_ring_off[:-1]]  # first ring sizes
    nr = np.diff(P.poly_ring_off)
    picks = {int(np.argmax(nv)), int(np.argmin(nv)), P.n_poly - 1}  # biggest, smallest, an enclave
    holed = np.nonzero(nr > 1)[0]
    if holed.size:
        picks.add(int(holed[0]))
    while len(picks) < n:
        picks.add(int(rng.integers(0, P.n_poly)))
    return sorted(picks)


def _oracle_poly(cfg, P, k):
    r0, r1, c0, c1 = oracle.polygon_window(P, k, cfg.gt, cfg.rows, cfg.cols)
    one = P.subset([k])
    if r1 <= r0 or c1 <= c0:
        return np.zeros(cfg.nbins, np.uint64)
    win = fill_host(cfg.dem, cfg.cols, r0, c0, r1 - r0, c1 - c0)
    return oracle.o1(win, cfg.gt, one, oracle.make_bins(cfg.nbins, nodata=cfg.nodata), row0=r0, col0=c0)[0]


def test_state_full_size(cuda_device):
    import torch
    cfg = STATE
    P = cfg.polygons()
    t = _raster(cfg)
    G, st = _run(t, cfg, P)
    assert st["n_inside"] > 0 and st["n_isect"] > 0
    for k in _sample_polys(P, 6, 1):
        assert (G[k] == _oracle_poly(cfg, P, k)).all(), k
    # partition identity: the state tiling covers the whole extent
    v = t[:, :cfg.cols].reshape(-1).to(torch.int32)
    v = v[v != cfg.nodata].clamp(0, cfg.nbins - 1)
    glob = torch.bincount(v, minlength=cfg.nbins).cpu().numpy().astype(np.uint64)
    assert (G.sum(axis=0) == glob).all()
    G2, _ = _run(t, cfg, P, tile=100)
    assert (G2 == G).all()
    G3, _ = _run(t, cfg, P, force_isect=True)
    assert (G3 == G).all()


def test_conus_full_size(cuda_device):
    import torch
    cfg = CONUS
    P = cfg.polygons()
    t = _raster(cfg)
    G, st = _run(t, cfg, P)
    assert st["n_tiles"] == 366 * 844
    for k in _sample_polys(P, 5, 2):
        assert (G[k] == _oracle_poly(cfg, P, k)).all(), k
    torch.cuda.empty_cache()
    G2, _ = _run(t, cfg, P, tile=360)  # the paper's 0.1 degree tile
    assert (G2 == G).all()
    # every counted cell is a real, non-nodata cell
    assert G.sum() <= cfg.cells


def test_pipstress_full_size(cuda_device):
    """BASELINE.json configs[4]: the CONUS raster with 50k small jagged polygons (mostly
    intersecting tiles) over the tile-size sweep.  Fused and four-step paths at T = 256; the fused
    path alone at T = 64 (the four-step path would need 98.8 GB of tile histograms)
    and T = 1024 (no inside tile at all).  Every tile size gives the same histograms; sampled
    polygons equal the oracle."""
    import torch
    from paper_conf_ipps_zhangw14_b200 import zh
    cfg = PIPSTRESS
    P = cfg.polygons()
    t = _raster(cfg)
    G, st = _run(t, cfg, P)
    assert st["n_isect"] > 10 * st["n_inside"] > 0
    for k in _sample_polys(P, 8, 3):
        assert (G[k] == _oracle_poly(cfg, P, k)).all(), k
    torch.cuda.empty_cache()
    for tile in (64, 1024):
        with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=tile, cols=cfg.cols, nodata=cfg.nodata,
                               fused=True) as z:
            Gt = z.run()
            if tile == 1024:
                assert z.stats()["n_inside"] == 0
        assert (Gt == G).all(), tile
        torch.cuda.empty_cache()
    assert G.sum() <= cfg.cells
