"""Input generators: determinism, window consistency, recipe statistics (no method arithmetic)."""
import numpy as np

from synth.configs import CONUS, TINY
from synth.dem import NODATA, fill_host
from synth.polygons import voronoi_tiling


def test_dem_window_consistency_and_determinism():
    a = fill_host(CONUS.dem, CONUS.cols, 40000, 100000, 300, 500)
    b = fill_host(CONUS.dem, CONUS.cols, 40100, 100200, 100, 200)
    assert (a[100:200, 200:400] == b).all()
    c = fill_host(CONUS.dem, CONUS.cols, 40000, 100000, 300, 500, nthreads=1)
    assert (a == c).all()


def test_dem_srtm_like_statistics():
    a = fill_host(CONUS.dem, CONUS.cols, 30000, 100000, 1024, 2048)
    v = a[a != NODATA]
    assert 0.005 < (a == NODATA).mean() < 0.06          # clustered voids
    eq = (a[:, 1:] == a[:, :-1]).mean()
    assert 0.15 < eq < 0.6                              # runs of equal neighbours
    assert v.min() > -1000 and v.max() < 9000


def test_tiny_value_range_exercises_clamping():
    a = fill_host(TINY.dem, TINY.cols, 0, 0, TINY.rows, TINY.cols)
    v = a[a != NODATA]
    assert (v < 0).any() and (v >= TINY.nbins).any() and (a == NODATA).any()


def test_voronoi_tiling_shared_borders_exact():
    P = voronoi_tiling(1000, 800, (0, 1, 0, 800, 0, -1), 30, 5, 9, n_holes=2)
    # every undirected border edge is used by exactly two rings (the two neighbours, or a hole
    # ring and its enclave) with bit-identical endpoints; only extent-boundary edges by one
    from collections import Counter
    edges = Counter()
    for k in range(P.n_poly):
        for rx, ry in P.rings(k):
            n = len(rx)
            for i in range(n):
                j = (i + 1) % n
                a, b = (rx[i], ry[i]), (rx[j], ry[j])
                edges[(min(a, b), max(a, b))] += 1
    border = 0
    on = lambda p: min(abs(p[0]), abs(p[0] - 1000), abs(p[1]), abs(p[1] - 800)) < 1e-6
    for (a, b), m in edges.items():
        assert m in (1, 2)
        if m == 1:
            assert on(a) and on(b)
            border += 1
    assert border > 0
    assert P.meta["n_holes"] == 2 and P.n_poly == 32
