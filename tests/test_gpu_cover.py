"""GPU parity of the "geometrically intersect" variant (options.cover = 1, reading R15,
PAPER.md:12 §III ¶1): a cell counts in P_k when its closed rectangle meets the closed polygon.
libzh (k_parity + k_touch + k_pip_cells, both the four-step and the fused path) vs the oracle's
zho_cover_o0 (pinned in tests/test_oracle_cover.py), bit-exact.
"""
import numpy as np
import pytest

import oracle
from synth.configs import STATE, TINY, TINY_LONLAT
from synth.dem import fill_device, fill_host
from synth.polygons import from_rings

pytestmark = pytest.mark.gpu


def device_raster(spec, rows, cols, row0=0, nrows=None):
    import torch
    nrows = rows - row0 if nrows is None else nrows
    pitch = (cols + 7) // 8 * 8
    t = torch.full((nrows, pitch), 12345, dtype=torch.int16, device="cuda")
    fill_device(spec, cols, t.data_ptr(), row0, 0, nrows, cols, pitch, torch.cuda.current_stream().cuda_stream)
    return t


def gpu_hist(t, gt, P, nbins, tile, cols, rows=None, row0=0, **kw):
    """Both libzh paths (four steps and fused), required equal; returns the result."""
    from paper_conf_ipps_zhangw14_b200 import zh
    res = []
    for fused in (False, True):
        with zh.ZonalHistogram(t, gt, P, nbins, tile=tile, cols=cols, rows=rows, row0=row0, fused=fused,
                               **kw) as z:
            res.append(z.run())
    assert (res[0] == res[1]).all(), "fused path differs from the four-step path"
    return res[1]


@pytest.fixture(scope="module")
def tiny_cover():
    cfg = TINY
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    H = oracle.cover_o0(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    return cfg, P, R, H


@pytest.mark.parametrize("tile", [7, 64, 100, 128, 256, 1024])
def test_tiny_cover_bit_exact(tiny_cover, cuda_device, tile):
    cfg, P, R, H = tiny_cover
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    got = gpu_hist(t, cfg.gt, P, cfg.nbins, tile, cfg.cols, nodata=cfg.nodata, cover=True)
    assert (got == H).all()
    centre = gpu_hist(t, cfg.gt, P, cfg.nbins, tile, cfg.cols, nodata=cfg.nodata)
    assert (got >= centre).all() and got.sum() > centre.sum()


def test_tiny_cover_force_isect_and_u32(tiny_cover, cuda_device):
    cfg, P, R, H = tiny_cover
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    assert (gpu_hist(t, cfg.gt, P, cfg.nbins, 128, cfg.cols, nodata=cfg.nodata, cover=True,
                     force_isect=True) == H).all()
    assert (gpu_hist(t, cfg.gt, P, cfg.nbins, 128, cfg.cols, nodata=cfg.nodata, cover=True,
                     out_u64=False) == H).all()


def test_tiny_cover_shards_sum_to_whole(tiny_cover, cuda_device):
    cfg, P, R, H = tiny_cover
    T = 128
    acc = np.zeros_like(H)
    for r0, r1 in ((0, 384), (384, 768), (768, cfg.rows)):
        t = device_raster(cfg.dem, cfg.rows, cfg.cols, row0=r0, nrows=r1 - r0)
        acc += gpu_hist(t, cfg.gt, P, cfg.nbins, T, cfg.cols, rows=cfg.rows, row0=r0, nodata=cfg.nodata,
                        cover=True)
    assert (acc == H).all()


def test_tiny_lonlat_cover(cuda_device):
    cfg = TINY_LONLAT
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    H = oracle.cover_o0(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    for tile in (128, 256):
        assert (gpu_hist(t, cfg.gt, P, cfg.nbins, tile, cfg.cols, nodata=cfg.nodata, cover=True) == H).all()


@pytest.mark.parametrize("flip", ["x", "y"])
def test_cover_flipped_geotransform_and_grid_aligned_polygons(cuda_device, flip):
    """Axis-aligned rectangles on grid lines (touching sides/corners count), a diagonal through
    cell corners, a hole, a long straight edge, under mirrored geotransforms."""
    from synth.dem import KIND_LINMOD, DemSpec
    rows, cols = 300, 520
    spec = DemSpec(seed=3, kind=KIND_LINMOD)
    gt = [0.0, 1.0, 0.0, float(rows), 0.0, -1.0]
    if "x" in flip:
        gt = [float(cols), -1.0, 0.0, float(rows), 0.0, -1.0]
    if "y" in flip:
        gt = [gt[0], gt[1], 0.0, 0.0, 0.0, 1.0]

    def rect(x0, y0, x1, y1):
        return [(np.array([x0, x1, x1, x0]), np.array([y0, y0, y1, y1]))]
    polys = [rect(10, 10, 130, 70), rect(200.5, 20.25, 260.75, 290.5),
             [(np.array([300.0, 500, 300]), np.array([10.0, 210, 210]))],
             rect(20, 100, 180, 280) + rect(60, 150, 120, 200),
             [(np.array([0.0, 519.6, 519.6, 0.0]), np.array([295.0, 280.0, 299.9, 299.9]))]]
    P = from_rings(polys)
    R = fill_host(spec, cols, 0, 0, rows, cols)
    H = oracle.cover_o0(R, gt, P, oracle.make_bins(64, nodata=None))
    t = device_raster(spec, rows, cols)
    for tile in (32, 100, 256):
        assert (gpu_hist(t, gt, P, 64, tile, cols, cover=True) == H).all()


def test_state_window_cover(cuda_device):
    """Jagged state-scale polygons (~1.3k vertices) on a 1024 x 1024 window of the state raster."""
    cfg = STATE
    P = cfg.polygons()
    r0, c0, n = 12288, 14336, 1024  # window (tile aligned for T = 256)
    R = fill_host(cfg.dem, cfg.cols, r0, c0, n, n)
    gt = (cfg.gt[0] + c0 * cfg.gt[1], cfg.gt[1], 0.0, cfg.gt[3] + r0 * cfg.gt[5], 0.0, cfg.gt[5])
    H = oracle.cover_o0(R, gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    assert H.sum() > 0
    import torch
    t = torch.zeros((n, n), dtype=torch.int16)
    t[:] = torch.from_numpy(np.ascontiguousarray(R))
    t = t.cuda()
    got = gpu_hist(t, gt, P, cfg.nbins, 256, n, nodata=cfg.nodata, cover=True)
    assert (got == H).all()


def test_cover_requires_centre(cuda_device):
    from paper_conf_ipps_zhangw14_b200 import zh
    cfg = TINY
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    with pytest.raises(zh.ZhError):
        zh.ZonalHistogram(t, cfg.gt, cfg.polygons(), cfg.nbins, cover=True, rep=(0.0, 0.0))
