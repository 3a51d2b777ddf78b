"""Full-size GPU parity (BASELINE.json configs [1] state-scale, [2] CONUS-scale, [4] PIP-stress; the
bench's launch configuration): EVERY row of the P x B matrix against the oracle O1 over the whole
raster (§III ¶1 definition, centres PAPER.md:18 §III.D, Fig. 5 predicate PAPER.md:20),
bit-exact, for both libzh paths and several tile sizes; plus what holds at any size (partition
identity of the state tiling, force-all-intersect invariance) and the §8f-4 summary / distances
on the full-size histograms.

The oracle is fed band by band (rows are independent: O1 accumulates each band into the same
matrix).  Its raster is the synth generator's: the device fill (synth/dem_dev.cu, input
generation, not libzh) copied to the host band by band, checked equal to the host generator
(synth/dem_host.c) on sampled bands in the same test."""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle import features as F
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


def _oracle_full(cfg, P, t, band=4096):
    """O1 over the whole raster, fed in bands of rows from the generator's device fill."""
    bins = oracle.make_bins(cfg.nbins, lo=cfg.lo, width=cfg.width, nodata=cfg.nodata, oor_drop=cfg.oor_drop)
    H = np.zeros((P.n_poly, cfg.nbins), dtype=np.uint64)
    rng = np.random.default_rng(cfg.rows)
    checks = set(int(v) for v in rng.integers(0, cfg.rows // band, 2))
    for i, r0 in enumerate(range(0, cfg.rows, band)):
        n = min(band, cfg.rows - r0)
        host = t[r0:r0 + n, :cfg.cols].cpu().numpy()
        if i in checks:  # the device generator equals the host generator the oracle is pinned with
            assert np.array_equal(host[:64], fill_host(cfg.dem, cfg.cols, r0, 0, min(64, n), cfg.cols))
        oracle.o1(host, cfg.gt, P, bins, row0=r0, out=H)
    return H


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


def _fused(t, cfg, P, tile):
    from paper_conf_ipps_zhangw14_b200 import zh
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=tile, cols=cfg.cols, nodata=cfg.nodata, fused=True) as z:
        G = z.run()
        st = z.stats()
    return G, st


def _assert_equal(G, H, what):
    if not np.array_equal(G, H):
        bad = np.nonzero((G != H).any(axis=1))[0]
        raise AssertionError(f"{what}: {bad.size} polygon rows differ from the oracle, first {bad[:8].tolist()}")


def _features(t, cfg, P, H):
    """§8f-4 on the full-size histogram: summary bit-exact to zh.h's sequence on the oracle's
    integers, and L1 / EMD / chi^2 on sampled polygon pairs against the exact definitions."""
    from paper_conf_ipps_zhangw14_b200 import zh
    rng = np.random.default_rng(11)
    a = rng.integers(0, P.n_poly, 60)
    b = rng.integers(0, P.n_poly, 60)
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=cfg.tile, cols=cfg.cols, nodata=cfg.nodata) as z:
        z.run()
        S = z.zh_zonal_summary()
        D = {k: z.zh_hist_distance(k, a, b) for k in ("l1", "emd", "chi2")}
    n = H.sum(axis=1)
    for k in range(P.n_poly):
        if n[k] == 0:
            assert S[k, 0] == 0 and np.isnan(S[k, 4])
            continue
        row = H[k].astype(object)
        s1 = int(np.dot(np.arange(cfg.nbins, dtype=object), row))
        s2 = int(np.dot(np.arange(cfg.nbins, dtype=object) ** 2, row))
        nk = int(n[k])
        assert S[k, 0] == nk
        assert S[k, 4] == float(cfg.lo) + float(cfg.width) * (float(s1) / float(nk))
        assert S[k, 5] == float(cfg.width) * (math.sqrt(float(nk * s2 - s1 * s1)) / float(nk))
    U = 2.0 ** -53
    for kind, g in D.items():
        for i, (x, y) in enumerate(zip(a, b)):
            e = F.distance_exact(H, kind, int(x), int(y))
            if e is None:
                assert math.isnan(g[i])
            elif kind == "chi2":
                assert abs(Fraction(g[i]) - e) <= (cfg.nbins + 8) * U * e
            else:
                N = e * int(n[x]) * int(n[y])
                n1, n2 = sorted((int(n[x]), int(n[y])))
                assert g[i] == float(N.numerator) / float(n1) / float(n2)


def test_state_full_size(cuda_device):
    import torch
    cfg = STATE
    P = cfg.polygons()
    t = _raster(cfg)
    H = _oracle_full(cfg, P, t)
    G, st = _run(t, cfg, P)
    assert st["n_inside"] > 0 and st["n_isect"] > 0
    _assert_equal(G, H, "state T=256")
    # partition identity: the state tiling covers the whole extent
    v = t[:, :cfg.cols].reshape(-1).to(torch.int32)
    v = v[v != cfg.nodata].clamp(0, cfg.nbins - 1)
    glob = torch.bincount(v, minlength=cfg.nbins).cpu().numpy().astype(np.uint64)
    assert (H.sum(axis=0) == glob).all()
    G2, _ = _run(t, cfg, P, tile=100)
    _assert_equal(G2, H, "state T=100")
    G3, _ = _run(t, cfg, P, force_isect=True)
    _assert_equal(G3, H, "state force-intersect")
    _features(t, cfg, P, H)


def test_conus_full_size(cuda_device):
    import torch
    cfg = CONUS
    P = cfg.polygons()
    t = _raster(cfg)
    H = _oracle_full(cfg, P, t)
    G, st = _run(t, cfg, P)
    assert st["n_tiles"] == 366 * 844
    _assert_equal(G, H, "CONUS T=256")
    torch.cuda.empty_cache()
    G2, _ = _run(t, cfg, P, tile=360)  # the paper's 0.1 degree tile
    _assert_equal(G2, H, "CONUS T=360")
    torch.cuda.empty_cache()
    _features(t, cfg, P, H)


def test_pipstress_full_size(cuda_device):
    """BASELINE.json configs[4]: the CONUS raster with 50k small jagged polygons (mostly
    intersecting tiles) over the tile-size sweep.  Fused and four-step paths at T = 256; the fused
    path alone at T = 64 (the four-step path would need 98.8 GB of tile histograms),
    T = 512 and T = 1024 (no inside tile at all).  Every result is the whole oracle matrix."""
    import torch
    cfg = PIPSTRESS
    P = cfg.polygons()
    t = _raster(cfg)
    H = _oracle_full(cfg, P, t)
    G, st = _run(t, cfg, P)
    assert st["n_isect"] > 10 * st["n_inside"] > 0
    _assert_equal(G, H, "PIP-stress T=256")
    del G
    torch.cuda.empty_cache()
    for tile in (64, 512, 1024):
        Gt, stt = _fused(t, cfg, P, tile)
        if tile == 1024:
            assert stt["n_inside"] == 0
        _assert_equal(Gt, H, f"PIP-stress T={tile}")
        del Gt
        torch.cuda.empty_cache()
