"""GPU parity of SURVEY.md §8f-4 (§I ¶1): zh_zonal_summary and zh_hist_distance against
oracle/features.py (exact rational definitions), on the tiny config's oracle histograms.

Two checks per value: (1) bit-exact equality with the rounding sequence zh.h states, applied in
Python floats (IEEE binary64, round-to-nearest) to the exact integers the oracle defines; (2) the
distance to the exact rational value within the bound that sequence implies."""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle import features as F
from synth.configs import TINY
from synth.dem import fill_device, fill_host

pytestmark = pytest.mark.gpu
U = 2.0 ** -53


@pytest.fixture(scope="module")
def tiny_gpu():
    import torch
    cfg = TINY
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    t = torch.empty((cfg.rows, cfg.cols), dtype=torch.int16, device="cuda")
    fill_device(cfg.dem, cfg.cols, t.data_ptr(), 0, 0, cfg.rows, cfg.cols, cfg.cols,
                torch.cuda.current_stream().cuda_stream)
    return cfg, P, R, t


def _summary_ref(row, lo, width):
    """zh.h's stated sequence for mean / std on the exact integers of one histogram row."""
    n = sum(row)
    s1 = sum(b * v for b, v in enumerate(row))
    s2 = sum(b * b * v for b, v in enumerate(row))
    mean = float(lo) + float(width) * (float(s1) / float(n))
    std = float(width) * (math.sqrt(float(n * s2 - s1 * s1)) / float(n))
    return mean, std


@pytest.mark.parametrize("lo,width,nbins", [(0, 1, 256), (-400, 3, 400)])
@pytest.mark.parametrize("out_u64", [True, False])
def test_zonal_summary(tiny_gpu, cuda_device, lo, width, nbins, out_u64):
    from paper_conf_ipps_zhangw14_b200 import zh
    cfg, P, R, t = tiny_gpu
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(nbins, lo=lo, width=width, nodata=cfg.nodata))
    with zh.ZonalHistogram(t, cfg.gt, P, nbins, lo=lo, width=width, tile=cfg.tile, nodata=cfg.nodata,
                           out_u64=out_u64) as z:
        G = z.run()
        S = z.zh_zonal_summary()
        d = z.zonal_stats()
    assert (G == H).all()
    want = F.summary_exact(H, lo, width)
    for k in range(P.n_poly):
        n, mn, mx, med, mean, var = want[k]
        assert S[k, 0] == n
        if n == 0:
            assert np.isnan(S[k, 1:]).all()
            continue
        assert (S[k, 1], S[k, 2], S[k, 3]) == (mn, mx, med)
        m_ref, s_ref = _summary_ref([int(v) for v in H[k]], lo, width)
        assert S[k, 4] == m_ref and S[k, 5] == s_ref, k  # bit-exact: the stated rounding sequence
        # within the bound of that sequence around the exact values (4 roundings, 5 for std)
        assert abs(Fraction(S[k, 4]) - mean) <= 4 * U * (abs(mean) + abs(mean - lo))
        sd = F.sqrt_fraction(var)
        assert abs(Fraction(S[k, 5]) - sd) <= 5 * U * sd + Fraction(1, 10 ** 30)
    assert (d["count"] == S[:, 0]).all() and np.array_equal(d["std"], S[:, 5], equal_nan=True)


def _pairs(n):
    a, b = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    return a.ravel(), b.ravel()


@pytest.mark.parametrize("kind", ["l1", "emd", "chi2"])
@pytest.mark.parametrize("wide", [False, True])
def test_hist_distances(tiny_gpu, cuda_device, monkeypatch, kind, wide):
    from paper_conf_ipps_zhangw14_b200 import zh
    cfg, P, R, t = tiny_gpu
    if wide:
        monkeypatch.setenv("ZH_DIST_WIDE", "1")
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=cfg.tile, nodata=cfg.nodata) as z:
        z.run()
        a, b = _pairs(P.n_poly)
        L = z.zh_hist_distance(kind, a, b)
        M = z.zh_hist_distance(kind)
        few = z.zh_hist_distance(kind, [3], [3])
    L = L.reshape(P.n_poly, P.n_poly)
    if kind == "chi2":  # the two modes sum the bins in different orders
        assert np.allclose(L, M, rtol=(cfg.nbins + 8) * 2 * U, atol=0, equal_nan=True)
    else:
        assert np.array_equal(L, M, equal_nan=True)
    assert np.array_equal(M, M.T, equal_nan=True)
    n = H.sum(axis=1).astype(object)
    for i, j in zip(a, b):
        e = F.distance_exact(H, kind, int(i), int(j))
        g = M[i, j]
        if e is None:
            assert math.isnan(g)
            continue
        if kind == "chi2":
            assert abs(Fraction(g) - e) <= (cfg.nbins + 8) * U * e
        else:
            N = e * n[i] * n[j]
            assert N.denominator == 1
            n1, n2 = sorted((int(n[i]), int(n[j])))
            assert g == float(N.numerator) / float(n1) / float(n2), (i, j)  # bit-exact
            assert abs(Fraction(g) - e) <= 3 * U * e
    assert few[0] == 0.0 and (np.diag(M)[n > 0] == 0).all()


def test_distance_rejects_bad_ids(tiny_gpu, cuda_device):
    from paper_conf_ipps_zhangw14_b200 import zh
    cfg, P, R, t = tiny_gpu
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=cfg.tile, nodata=cfg.nodata) as z:
        with pytest.raises(zh.ZhError):
            z.zh_hist_distance("l1")  # no histogram yet
        z.run()
        with pytest.raises(zh.ZhError):
            z.zh_hist_distance("l1", [0], [P.n_poly])


def test_distances_with_empty_and_no_polygons(tiny_gpu, cuda_device):
    """Polygons with no counted cell give NaN distances (R17) and NaN summaries; no polygons at all
    give empty results."""
    from paper_conf_ipps_zhangw14_b200 import zh
    from synth.polygons import from_rings
    cfg, P, R, t = tiny_gpu
    sq = (np.array([5.0, 30, 30, 5]), np.array([5.0, 5, 30, 30]))
    off = (sq[0] + 5000, sq[1])  # far off the raster: no cell
    Q = from_rings([[sq], [off], [(sq[0] + 100, sq[1] + 100)]])
    with zh.ZonalHistogram(t, cfg.gt, Q, cfg.nbins, tile=64, nodata=cfg.nodata) as z:
        z.run()
        M = z.zh_hist_distance("l1")
        S = z.zh_zonal_summary()
    assert np.isnan(M[1]).all() and np.isnan(M[:, 1]).all()
    assert M[0, 0] == 0 and M[0, 2] == M[2, 0] and not np.isnan(M[0, 2])
    assert S[1, 0] == 0 and np.isnan(S[1, 1:]).all()
    E = from_rings([])
    with zh.ZonalHistogram(t, cfg.gt, E, cfg.nbins, tile=64) as z:
        z.run()
        assert z.zh_hist_distance("emd").shape == (0, 0)
        assert z.zh_zonal_summary().shape == (0, 6)


def test_step_graph_on_host_raster(tiny_gpu, cuda_device):
    """zh_step_graph on a context whose raster lives in host memory: after the upload (zh_run) the
    graph replays the step on the device copy."""
    import torch
    from paper_conf_ipps_zhangw14_b200 import zh
    cfg, P, R, t = tiny_gpu
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    pinned = torch.from_numpy(R.copy()).pin_memory()
    for fused in (True, False):
        with zh.ZonalHistogram(pinned, cfg.gt, P, cfg.nbins, tile=cfg.tile, nodata=cfg.nodata, fused=fused) as z:
            with pytest.raises(zh.ZhError):
                z.zh_step_graph()  # nothing uploaded yet
            assert (z.run() == H).all()
            for _ in range(3):
                z.zh_step_graph()
                assert (z.output_device().cpu().numpy().view(np.uint64) == H).all()
