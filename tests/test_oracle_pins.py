"""Pins of the CPU oracle against what the paper and the mathematics fix (not against itself).

Each pin is chosen so that a plausible slip in oracle/zh_oracle.c fails at least one:
  - dropped/transposed terms in the intercept, wrong sign of a comparison, closed vs
    half-open rule  -> hand-worked counts with edges/vertices on centres, Fig. 5 counts;
  - rows/cols transposed, geotransform sign handling  -> non-square raster, flipped gt;
  - bin mapping (lo, width, clamp/drop, nodata)  -> closed-form histograms, np.bincount;
  - ring bookkeeping (offsets, holes, implicit closure)  -> hole/island cases, partition;
  - O1 hoisting  -> O0 == O1 on every cell of tiny (dyadic and lon/lat geotransforms).
"""
import os

import numpy as np
import pytest

import oracle
from synth.configs import TINY, TINY_LONLAT
from synth.dem import KIND_COLMOD, DemSpec, fill_host
from synth.polygons import from_rings

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _parse_rings(s):
    rings = []
    for part in s.split("/"):
        pts = [tuple(map(float, p.split(","))) for p in part.split()]
        rings.append((np.array([p[0] for p in pts]), np.array([p[1] for p in pts])))
    return rings


def _hand_cases():
    out = []
    for line in open(os.path.join(GOLD, "hand_counts.txt")):
        if line.startswith("#") or not line.strip():
            continue
        name, rings, count, _ = [f.strip() for f in line.split("|")]
        out.append((name, _parse_rings(rings), int(count)))
    return out


HAND = _hand_cases()
GT_HAND = (0.0, 1.0, 0.0, 20.0, 0.0, -1.0)


@pytest.mark.parametrize("mode", ["o0", "o0p", "o1"])
def test_hand_worked_counts(mode):
    R = np.zeros((20, 24), np.int16)
    P = from_rings([rings for _, rings, _ in HAND])
    bins = oracle.make_bins(1)
    if mode == "o1":
        H = oracle.o1(R, GT_HAND, P, bins)
    else:
        H = oracle.o0(R, GT_HAND, P, bins, prefilter=(mode == "o0p"))
    got = {name: int(H[k, 0]) for k, (name, _, _) in enumerate(HAND)}
    want = {name: c for name, _, c in HAND}
    assert got == want


@pytest.mark.parametrize("flip", ["x", "y", "xy"])
def test_hand_counts_flipped_geotransform(flip):
    """Same geometry under a mirrored geotransform: x' = 24 - x (gt1 < 0) and/or y' = -y... the
    cells are relabelled but the set of centres and the polygon are mirrored together.
    Mirroring x maps the half-open rule left<->right, so only cases symmetric under the rule's
    boundary handling (no edges through centres) are compared."""
    sx = -1.0 if "x" in flip else 1.0
    sy = -1.0 if "y" in flip else 1.0
    # mirrored gt: centre of (r, c) is (sx*(c+.5) + ox, sy*(19.5 - r)...)
    gt = (24.0 if sx < 0 else 0.0, sx * 1.0, 0.0, -20.0 if sy < 0 else 20.0, 0.0, -1.0 * sy)
    R = np.zeros((20, 24), np.int16)
    names = ["square_hole", "tall_rect", "wide_rect", "two_islands", "off_raster", "degenerate_two_vertex"]
    cases = [(n, r, c) for n, r, c in HAND if n in names]
    # mirror polygons the same way the geotransform mirrors centres: x -> ox + sx*x, y -> sy*y (+shift)
    polys = []
    for _, rings, _ in cases:
        mr = []
        for rx, ry in rings:
            mx = (24.0 - rx) if sx < 0 else rx
            my = (-ry) if sy < 0 else ry
            mr.append((mx, my))
        polys.append(mr)
    P = from_rings(polys)
    bins = oracle.make_bins(1)
    for H in (oracle.o0(R, gt, P, bins), oracle.o1(R, gt, P, bins)):
        assert [int(h) for h in H[:, 0]] == [c for _, _, c in cases]


def test_fig5_crossing_counts():
    """PAPER.md:20 Fig. 5: 2 / 4 / 3 / 1 crossings for a polygon with a hole."""
    rows = [l.split() for l in open(os.path.join(GOLD, "fig5_crossings.txt")) if not l.startswith("#")]
    P = from_rings([[(np.array([0., 10, 10, 0]), np.array([0., 0, 10, 10])),
                     (np.array([3., 7, 7, 3]), np.array([3., 3, 7, 7]))]])
    for x, y, n, inside in rows:
        got = oracle.crossings(P, 0, float(x), float(y))
        assert got == int(n)
        assert (got & 1) == int(inside)


def test_franklin_textbook_single_ring_random():
    """Crossing parity == winding-number insideness for random points off the boundary of a
    random simple (star-shaped) polygon — the textbook equivalence of PNPOLY [16]."""
    rng = np.random.default_rng(0)
    th = np.sort(rng.uniform(0, 2 * np.pi, 40))
    rad = rng.uniform(2, 5, 40)
    px, py = rad * np.cos(th), rad * np.sin(th)
    P = from_rings([[(px, py)]])
    pts = rng.uniform(-6, 6, size=(400, 2))

    def winding(x, y):
        ang = np.arctan2(py - y, px - x)
        d = np.diff(np.concatenate([ang, ang[:1]]))
        d = (d + np.pi) % (2 * np.pi) - np.pi
        return int(round(d.sum() / (2 * np.pi)))

    for x, y in pts:
        assert (oracle.crossings(P, 0, x, y) & 1) == (winding(x, y) != 0)


def test_closed_form_histogram_colmod():
    """v(r,c) = c mod 7; rectangle [10.5,41.5) x [5.5,29.5) on a 64x64 dyadic raster:
    24 rows x 31 cols, residues 3,4,5 appear 5 times, the others 4."""
    spec = DemSpec(kind=KIND_COLMOD, pattern_mod=7, pattern_off=0)
    R = fill_host(spec, 64, 0, 0, 64, 64)
    gt = (0.0, 1.0, 0.0, 64.0, 0.0, -1.0)
    P = from_rings([[(np.array([10.5, 41.5, 41.5, 10.5]), np.array([5.5, 5.5, 29.5, 29.5]))]])
    want = np.array([96, 96, 96, 120, 120, 120, 96], np.uint64)
    for H in (oracle.o0(R, gt, P, oracle.make_bins(7)), oracle.o1(R, gt, P, oracle.make_bins(7))):
        assert (H[0] == want).all()
    # lo=2, width=2, nbins=3, clamp: residues {0,1}->bin0 (clamped), {2,3}->0, {4,5}->1, {6}->2
    per_res = np.array([4, 4, 4, 5, 5, 5, 4]) * 24
    want_c = np.array([per_res[0] + per_res[1] + per_res[2] + per_res[3], per_res[4] + per_res[5], per_res[6]])
    H = oracle.o0(R, gt, P, oracle.make_bins(3, lo=2, width=2))
    assert (H[0] == want_c.astype(np.uint64)).all()
    # drop: residues 0,1 dropped
    want_d = np.array([per_res[2] + per_res[3], per_res[4] + per_res[5], per_res[6]])
    H = oracle.o1(R, gt, P, oracle.make_bins(3, lo=2, width=2, oor_drop=True))
    assert (H[0] == want_d.astype(np.uint64)).all()
    # nbins=2 width=2 lo=0 clamp: bins {0,1}->0, {2,3}->1, {4,5,6}->1 (clamped high)
    H = oracle.o0(R, gt, P, oracle.make_bins(2, lo=0, width=2))
    assert (H[0] == np.array([per_res[0] + per_res[1], per_res[2:].sum()], np.uint64)).all()
    # nodata = 3: residue 3 never counted
    H = oracle.o1(R, gt, P, oracle.make_bins(7, nodata=3))
    w = want.copy()
    w[3] = 0
    assert (H[0] == w).all()


def _clip_ref(v, nbins, lo, width, nodata, drop):
    v = v.astype(np.int64).ravel()
    if nodata is not None:
        v = v[v != nodata]
    d = v - lo
    if drop:
        d = d[d >= 0]
        b = d // width
        b = b[b < nbins]
    else:
        b = np.where(d < 0, 0, d // width)
        b = np.minimum(b, nbins - 1)
    return np.bincount(b, minlength=nbins).astype(np.uint64)


@pytest.mark.parametrize("lo,width,nbins,drop", [(0, 1, 256, False), (0, 1, 256, True),
                                                  (-100, 3, 50, False), (20, 7, 9, True)])
def test_whole_raster_equals_bincount(lo, width, nbins, drop):
    """A polygon enclosing the whole raster: H == np.bincount of the mapped values."""
    R = fill_host(TINY.dem, 1024, 0, 0, 300, 200)  # non-square window
    gt = (0.0, 1.0, 0.0, 300.0, 0.0, -1.0)
    P = from_rings([[(np.array([-1.0, 201, 201, -1]), np.array([-1.0, -1, 301, 301]))]])
    bins = oracle.make_bins(nbins, lo=lo, width=width, nodata=-32768, oor_drop=drop)
    want = _clip_ref(R, nbins, lo, width, -32768, drop)
    assert (oracle.o0(R, gt, P, bins)[0] == want).all()
    assert (oracle.o1(R, gt, P, bins)[0] == want).all()
    for v in (-32768, -5, 0, 1, 19, 20, 26, 27, 83, 84, 10000):
        b = oracle.bin_of(v, bins)
        ref = _clip_ref(np.array([v]), nbins, lo, width, -32768, drop)
        assert (b < 0 and ref.sum() == 0) or (b >= 0 and ref[b] == 1)


@pytest.mark.parametrize("cfg", [TINY, TINY_LONLAT], ids=lambda c: c.name)
def test_tiny_tiling_partition_and_o0_eq_o1(cfg):
    """Jagged Voronoi tiling with an enclave: every centre is in exactly one polygon, so the
    per-polygon histograms sum to the global histogram; O0 == O0(prefilter) == O1 everywhere."""
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    bins = oracle.make_bins(cfg.nbins, nodata=cfg.nodata)
    h0 = oracle.o0(R, cfg.gt, P, bins)
    h0p = oracle.o0(R, cfg.gt, P, bins, prefilter=True)
    h1 = oracle.o1(R, cfg.gt, P, bins)
    assert (h0 == h1).all() and (h0 == h0p).all()
    assert (h0.sum(axis=0) == _clip_ref(R, cfg.nbins, 0, 1, cfg.nodata, False)).all()
    # membership on a sample: exactly one polygon per centre
    rng = np.random.default_rng(3)
    rr = rng.integers(0, cfg.rows, 3000)
    cc = rng.integers(0, cfg.cols, 3000)
    m = oracle.membership(rr, cc, cfg.gt, P)
    assert (m.sum(axis=1) == 1).all()
    # the enclave (last polygon) is a hole of its host: host + enclave = host's outer ring alone
    k_enc = P.n_poly - 1
    host = [k for k in range(P.n_poly - 1) if P.poly_ring_off[k + 1] - P.poly_ring_off[k] == 2]
    assert len(host) == 1
    outer = P.subset([host[0]])
    outer = from_rings([outer.rings(0)[:1]])
    ho = oracle.o1(R, cfg.gt, outer, bins)
    assert (ho[0] == h0[host[0]] + h0[k_enc]).all()


def test_degenerate_inputs():
    R = fill_host(TINY.dem, 1024, 0, 0, 64, 64)
    gt = (0.0, 1.0, 0.0, 64.0, 0.0, -1.0)
    sq = (np.array([5.0, 30, 30, 5]), np.array([5.0, 5, 30, 30]))
    sq_closed = (np.append(sq[0], 5.0), np.append(sq[1], 5.0))
    P = from_rings([
        [],                                              # zero rings
        [(np.array([]), np.array([]))],                  # empty ring
        [(np.array([3.0]), np.array([3.0]))],            # 1-vertex ring
        [(np.array([3.0, 40]), np.array([3.0, 50]))],    # 2-vertex ring
        [sq], [sq_closed],                               # implicit vs explicit closure
        [sq, (np.array([3.0, 40]), np.array([3.0, 50]))],  # + degenerate ring changes nothing
        [(sq[0] + 1000, sq[1])],                         # off the raster
        [(np.repeat(sq[0], 2), np.repeat(sq[1], 2))],    # duplicated consecutive vertices
    ])
    bins = oracle.make_bins(256, nodata=-32768)
    for H in (oracle.o0(R, gt, P, bins), oracle.o1(R, gt, P, bins)):
        assert H[0:4].sum() == 0 and H[7].sum() == 0
        assert (H[4] == H[5]).all() and (H[4] == H[6]).all() and (H[4] == H[8]).all()
        assert H[4].sum() > 0


def test_zonal_stats_from_histogram_match_cells():
    """oracle.zonal_stats (from the oracle histogram) == the same statistics computed straight
    from the cell values inside each polygon (oracle membership), with no clamping in play."""
    cfg = TINY
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, 256, 384)  # a window; polygons cover it partially
    gt = (0.0, 1.0, 0.0, 1024.0, 0.0, -1.0)
    lo, nb = -400, 1200  # every DEM value of the window has its own bin
    H = oracle.o1(R, gt, P, oracle.make_bins(nb, lo=lo, nodata=-32768))
    st = oracle.zonal_stats(H)
    rr, cc = np.meshgrid(np.arange(256), np.arange(384), indexing="ij")
    mem = oracle.membership(rr.ravel(), cc.ravel(), gt, P)
    vals = R.ravel().astype(np.int64)
    for k in range(P.n_poly):
        sel = (mem[:, k] == 1) & (vals != -32768)
        b = vals[sel] - lo
        assert st[k, 0] == b.size
        if b.size == 0:
            assert st[k, 1] == st[k, 2] == st[k, 3] == -1
            continue
        assert st[k, 1] == b.min() and st[k, 2] == b.max()
        assert st[k, 3] == np.sort(b)[(b.size + 1) // 2 - 1]
        assert st[k, 4] == b.sum()
        s2 = int((b * b).sum())
        assert st[k, 5] == np.int64(np.uint64(s2 & ((1 << 64) - 1)).view(np.int64)) and st[k, 6] == s2 >> 64
        assert st[k, 7] == np.unique(b).size


def test_representative_point_offsets():
    """SURVEY §8f-3 ('it is possible to use some other points (e.g., corners ...)').
    With gt = (0,1,0,20,0,-1) and the point (c + 0, r + 1), cell (r, c) is represented by the
    integer point (c, 19 - r).  Right triangle (0,0),(8,0),(0,8), half-open rule: the left leg
    (x = 0) is never crossed from x >= 0, the hypotenuse is crossed iff x < 8 - y, y in [0, 8):
    sum_{y=0..7} (8 - y) = 36 integer points (vs 28 cell centres).  Rectangle x in [2, 9],
    y in [3, 7]: x in {2..8} (7) x y in {3..6} (4) = 28 with corners too."""
    R = np.zeros((20, 24), np.int16)
    gt = (0.0, 1.0, 0.0, 20.0, 0.0, -1.0)
    P = from_rings([[(np.array([0.0, 8, 0]), np.array([0.0, 0, 8]))],
                    [(np.array([2.0, 9, 9, 2]), np.array([3.0, 3, 7, 7]))]])
    bins = oracle.make_bins(1)
    for fn in (oracle.o0, oracle.o1):
        assert [int(v) for v in fn(R, gt, P, bins, rep=(0.0, 1.0))[:, 0]] == [36, 28]
        assert [int(v) for v in fn(R, gt, P, bins)[:, 0]] == [28, 28]
    # centre == explicit (0.5, 0.5)
    assert (oracle.o1(R, gt, P, bins, rep=(0.5, 0.5)) == oracle.o1(R, gt, P, bins)).all()


def test_centre_operation_order_non_dyadic():
    """R7: the centre is gt0 + ((c + 0.5) * gt1), three binary64 ops in that order (the reading both
    sides implement).  Under a lon/lat geotransform (1 arc-second, not dyadic) other orders give
    other doubles, so this pins the oracle's order: numpy float64 scalars (IEEE, no FMA) evaluate
    the stated order, and the alternative orders must disagree on some cells (the check bites)."""
    from synth.configs import CONUS
    gt = CONUS.gt
    rng = np.random.default_rng(7)
    rr = rng.integers(0, CONUS.rows, 2000)
    cc = rng.integers(0, CONUS.cols, 2000)
    alt_x = alt_y = 0
    for r, c in zip(rr, cc):
        xc, yc = oracle.centre(gt, int(r), int(c))
        want_x = np.float64(gt[0]) + (np.float64(c) + np.float64(0.5)) * np.float64(gt[1])
        want_y = np.float64(gt[3]) + (np.float64(r) + np.float64(0.5)) * np.float64(gt[5])
        assert xc == want_x and yc == want_y
        alt_x += (np.float64(gt[0]) + np.float64(c) * np.float64(gt[1]) + np.float64(0.5) * np.float64(gt[1])) != xc
        alt_y += (np.float64(gt[3]) + np.float64(r) * np.float64(gt[5]) + np.float64(0.5) * np.float64(gt[5])) != yc
    assert alt_x > 0 and alt_y > 0
