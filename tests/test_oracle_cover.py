"""Pins of the oracle's "geometrically intersect" variant (reading R15, §III ¶1:
"the raster cells that geometrically intersect with P_k"): a cell counts in P_k when its CLOSED
rectangle meets the CLOSED polygon region.

The oracle (oracle/zh_oracle.c zho_cover_o0) decides it as "centre inside (ray crossing) OR some
edge meets the rectangle (separating-axis test in doubles)".  It is pinned here against
  - closed forms for axis-aligned rectangles on and off the grid lines;
  - an independent EXACT formulation in rational arithmetic (fractions.Fraction): two closed sets,
    a rectangle R and a polygon region P, meet iff a vertex of P lies in R, or a corner of R lies
    in P (boundary included), or an edge of P crosses a side of R — on dyadic inputs where every
    double operation of the oracle is exact, so the two must agree cell by cell;
  - invariants: cover contains the centre test; on an exact tiling every cell is covered and the
    cells covered twice are the ones an edge reaches.
A plausible slip (open instead of closed comparisons, a sign or operand swap in the orientation,
a missing corner, a wrong grid-line index) fails at least one of them.
"""
import random
from fractions import Fraction as F

import numpy as np
import pytest

import oracle
from synth.configs import TINY
from synth.polygons import from_rings

H_ = 12
GT = (0.0, 1.0, 0.0, float(H_), 0.0, -1.0)  # cell (r, c) = [c, c+1] x [H-r-1, H-r]


def _count(P, rows=H_, cols=H_, gt=GT):
    R = np.zeros((rows, cols), np.int16)
    return oracle.cover_o0(R, gt, P, oracle.make_bins(1))[:, 0].astype(int)


def _rect(x0, y0, x1, y1):
    return [(np.array([x0, x1, x1, x0]), np.array([y0, y0, y1, y1]))]


def test_rectangles_closed_form():
    # on grid lines: cells c with [c, c+1] meeting [a, b] are c in [a-1, b] (touching sides and
    # corners count), clipped to the raster
    cases = [(2, 3, 5, 7), (0, 0, 4, 2), (3, 3, 4, 4), (7, 1, 12, 12), (1, 5, 1.25, 6)]
    P = from_rings([_rect(*c) for c in cases])
    got = _count(P)
    for k, (a, c, b, d) in enumerate(cases):
        cols = [i for i in range(H_) if i + 1 >= a and i <= b]
        # row r spans y in [H-r-1, H-r]
        rows = [r for r in range(H_) if H_ - r >= c and H_ - r - 1 <= d]
        assert got[k] == len(cols) * len(rows), (k, got[k], len(cols), len(rows))
    # strictly inside cells (quarter offsets): exactly the cells the rectangle overlaps
    P2 = from_rings([_rect(2.25, 3.25, 5.75, 7.5), _rect(4.5, 4.5, 4.75, 4.75)])
    assert list(_count(P2)) == [4 * 5, 1]


def test_segment_touch_cases():
    # cell [1,2] x [1,2]
    c = (1.0, 2.0, 1.0, 2.0)
    assert oracle.seg_touches(0, 0, 1, 1, *c)            # ends at a corner
    assert oracle.seg_touches(0, 3, 3, 0, *c)            # passes through the corner (1,2)-(2,1) diagonal
    assert oracle.seg_touches(0, 1.5, 0.5, 1.5, 1.0, 2.0, 1.0, 2.0) is False
    assert oracle.seg_touches(2, 0, 2, 5, *c)            # along the right side
    assert oracle.seg_touches(1.5, 1.5, 1.5, 1.5, *c)    # a point inside
    assert not oracle.seg_touches(2.25, 0, 2.25, 5, *c)
    assert not oracle.seg_touches(0, 0, 0.75, 3, *c)


def test_segment_touch_diagonal_corner_exact():
    # the line x + y = 2.25 meets the square [1,2]^2 (it passes through (1.25, 1) and (1, 1.25))
    assert oracle.seg_touches(0, 2.25, 2.25, 0, 1.0, 2.0, 1.0, 2.0)
    # x + y = 1.75 stays below-left of the corner (1, 1)
    assert not oracle.seg_touches(0, 1.75, 1.75, 0, 1.0, 2.0, 1.0, 2.0)
    # x + y = 2 touches the corner only
    assert oracle.seg_touches(0, 2, 2, 0, 1.0, 2.0, 1.0, 2.0)


# ---- exact rational reference ------------------------------------------------------------------
def _orient(a, b, c):
    return (b[0] - a[0]) * (c[1] - a[1]) - (b[1] - a[1]) * (c[0] - a[0])


def _on_seg(a, b, p):
    return _orient(a, b, p) == 0 and min(a[0], b[0]) <= p[0] <= max(a[0], b[0]) and \
        min(a[1], b[1]) <= p[1] <= max(a[1], b[1])


def _seg_meet(a, b, c, d):
    o1, o2, o3, o4 = _orient(a, b, c), _orient(a, b, d), _orient(c, d, a), _orient(c, d, b)
    if ((o1 > 0 and o2 < 0) or (o1 < 0 and o2 > 0)) and ((o3 > 0 and o4 < 0) or (o3 < 0 and o4 > 0)):
        return True
    return _on_seg(a, b, c) or _on_seg(a, b, d) or _on_seg(c, d, a) or _on_seg(c, d, b)


def _in_closed_poly(rings, p):
    inside = False
    for ring in rings:
        n = len(ring)
        for i in range(n):
            a, b = ring[i], ring[(i + 1) % n]
            if _on_seg(a, b, p):
                return True
            if (a[1] > p[1]) != (b[1] > p[1]):
                xi = a[0] + (p[1] - a[1]) * (b[0] - a[0]) / (b[1] - a[1])
                if p[0] < xi:
                    inside = not inside
    return inside


def _exact_meets(rings, x0, x1, y0, y1):
    corners = [(x0, y0), (x1, y0), (x1, y1), (x0, y1)]
    sides = [(corners[i], corners[(i + 1) % 4]) for i in range(4)]
    for ring in rings:
        for v in ring:
            if x0 <= v[0] <= x1 and y0 <= v[1] <= y1:
                return True
    for cpt in corners:
        if _in_closed_poly(rings, cpt):
            return True
    for ring in rings:
        n = len(ring)
        for i in range(n):
            a, b = ring[i], ring[(i + 1) % n]
            for s, t in sides:
                if _seg_meet(a, b, s, t):
                    return True
    return False


def _simple(ring):
    n = len(ring)
    for i in range(n):
        a, b = ring[i], ring[(i + 1) % n]
        for j in range(i + 1, n):
            if j == i or (j + 1) % n == i or j == (i + 1) % n:
                continue
            if _seg_meet(a, b, ring[j], ring[(j + 1) % n]):
                return False
    return True


def _random_star(rng, cx, cy, n):
    while True:
        angs = sorted(rng.uniform(0, 2 * np.pi) for _ in range(n))
        pts = []
        for a in angs:
            r = rng.uniform(0.5, 4.5)
            # dyadic coordinates (quarters), some snapped to grid lines / corners
            q = 1 if rng.random() < 0.3 else 4
            x = round((cx + r * np.cos(a)) * q) / q
            y = round((cy + r * np.sin(a)) * q) / q
            pts.append((F(x), F(y)))
        if len(set(pts)) == len(pts) and _simple(pts):
            return pts


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_cover_equals_exact_rational_geometry(seed):
    rng = random.Random(seed)
    polys = []
    for _ in range(4):
        ring = _random_star(rng, rng.uniform(3, 9), rng.uniform(3, 9), rng.randint(3, 9))
        polys.append([ring])
    # a polygon with a hole (square with a square hole, on and off grid lines)
    outer = [(F(1), F(1)), (F(8), F(1)), (F(8), F(8)), (F(1), F(8))]
    hole = [(F(3), F(3)), (F(5.5), F(3)), (F(5.5), F(5.25)), (F(3), F(5.25))]
    polys.append([outer, hole])
    P = from_rings([[(np.array([float(p[0]) for p in ring]), np.array([float(p[1]) for p in ring]))
                     for ring in rings] for rings in polys])
    rr, cc = np.meshgrid(np.arange(H_), np.arange(H_), indexing="ij")
    got = oracle.cover_membership(rr.ravel(), cc.ravel(), GT, P)
    want = np.zeros_like(got)
    for q, (r, c) in enumerate(zip(rr.ravel(), cc.ravel())):
        x0, x1 = F(int(c)), F(int(c) + 1)
        y0, y1 = F(H_ - int(r) - 1), F(H_ - int(r))
        for k, rings in enumerate(polys):
            want[q, k] = _exact_meets(rings, x0, x1, y0, y1)
    assert np.array_equal(got, want), np.argwhere(got != want)[:10]
    # the histogram form agrees with the per-cell form, with and without the prefilter
    R = np.zeros((H_, H_), np.int16)
    for pf in (False, True):
        Hc = oracle.cover_o0(R, GT, P, oracle.make_bins(1), prefilter=pf)[:, 0]
        assert np.array_equal(Hc.astype(np.int64), want.sum(axis=0).astype(np.int64))


def test_cover_contains_centre_and_tiling_invariants():
    cfg = TINY
    P = cfg.polygons()
    rng = np.random.default_rng(5)
    rows = rng.integers(0, cfg.rows, 4000)
    cols = rng.integers(0, cfg.cols, 4000)
    cov = oracle.cover_membership(rows, cols, cfg.gt, P)
    cen = oracle.membership(rows, cols, cfg.gt, P)
    assert np.all(cov >= cen)                     # cover contains the centre test
    # the tiny tiling partitions the extent: every cell is covered at least once ...
    assert np.all(cov.sum(axis=1) >= 1)
    # ... and a cell covered more than once (or covered without its centre inside) is reached
    # by some polygon edge
    multi = np.nonzero((cov.sum(axis=1) > 1) | (cov != cen).any(axis=1))[0]
    assert multi.size > 0
    for q in multi[:200]:
        r, c = int(rows[q]), int(cols[q])
        X0 = cfg.gt[0] + c * cfg.gt[1]
        X1 = cfg.gt[0] + (c + 1) * cfg.gt[1]
        Y0 = cfg.gt[3] + r * cfg.gt[5]
        Y1 = cfg.gt[3] + (r + 1) * cfg.gt[5]
        hit = False
        for k in np.nonzero(cov[q])[0]:
            for rx, ry in P.rings(int(k)):
                n = len(rx)
                for i in range(n):
                    j = (i + 1) % n
                    if oracle.seg_touches(rx[i], ry[i], rx[j], ry[j], X0, X1, Y0, Y1):
                        hit = True
                        break
                if hit:
                    break
            if hit:
                break
        assert hit, (r, c)


def test_cover_histogram_prefilter_on_tiny():
    cfg = TINY
    P = cfg.polygons()
    from synth.dem import fill_host
    R = fill_host(cfg.dem, cfg.cols, 0, 0, 96, cfg.cols)
    b = oracle.make_bins(cfg.nbins, nodata=cfg.nodata)
    a = oracle.cover_o0(R, cfg.gt, P, b, prefilter=True)
    z = oracle.cover_o0(R, cfg.gt, P, b, prefilter=False)
    assert np.array_equal(a, z)
    cen = oracle.o1(R, cfg.gt, P, b)
    assert np.all(a >= cen) and a.sum() > cen.sum()
