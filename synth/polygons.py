"""Synthetic county-like polygon sets (INPUT GENERATION ONLY — no zonal-histogram arithmetic).

Jagged Voronoi tilings that partition their extent EXACTLY (SURVEY.md §8d "Polygon tiling
recipe"):

1. seeds in the extent plus their mirror images across the four sides, so each original
   seed's Voronoi cell is clipped to the extent;
2. boundary ridges (against a mirror) stay straight;
3. each interior ridge ab shared by seeds s1, s2 is replaced ONCE by a graph
   p(t) = a + t(b-a) + h(t) n, h from recursive midpoint displacement, clamped to
   [-lam E2 min(t,1-t), lam E1 min(t,1-t)] with E_i = height of s_i over ab / max(1, t_s, 1-t_s).
   The curve therefore stays inside triangles (s1,a,b) u (s2,a,b), which are interior-disjoint
   across ridges, so no two curves cross and none self-intersects;
4. both neighbours reference the identical vertex list (one reversed); every vertex is
   mapped to geo coordinates once, so shared borders are bit-identical;
5. enclaves: a jagged circle of radius 0.4 x (min distance seed -> own ring) is a separate
   polygon AND a hole ring of its host (multi-ring polygons, "not rare");
6. an optional land mask drops the cells whose seed lies in "ocean" (the paper's
   outside-only tiles, e.g. southern Florida, §IV.C).

Coordinates are produced in cell space (u = column coordinate, v = row coordinate) and
mapped with the raster geotransform x = gt0 + u*gt1, y = gt3 + v*gt5.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np


@dataclass
class Polygons:
    """Ring-offset polygon arrays, the layout the zh_polygons ABI struct takes (include/zh.h)."""
    poly_ring_off: np.ndarray  # int64 [P+1]
    ring_vert_off: np.ndarray  # int64 [R+1]
    x: np.ndarray              # float64 [V]
    y: np.ndarray              # float64 [V]
    meta: dict = field(default_factory=dict)

    @property
    def n_poly(self) -> int:
        return int(self.poly_ring_off.shape[0] - 1)

    @property
    def n_ring(self) -> int:
        return int(self.ring_vert_off.shape[0] - 1)

    @property
    def n_vert(self) -> int:
        return int(self.x.shape[0])

    def rings(self, k: int):
        """List of (x, y) arrays for the rings of polygon k."""
        out = []
        for r in range(int(self.poly_ring_off[k]), int(self.poly_ring_off[k + 1])):
            a, b = int(self.ring_vert_off[r]), int(self.ring_vert_off[r + 1])
            out.append((self.x[a:b], self.y[a:b]))
        return out

    def subset(self, ks) -> "Polygons":
        return from_rings([self.rings(int(k)) for k in ks])


def from_rings(polys) -> Polygons:
    """Build ring-offset arrays from [[(xs, ys), ...ring...], ...polygon...]."""
    pro = [0]
    rvo = [0]
    xs, ys = [], []
    for rings in polys:
        for rx, ry in rings:
            rx = np.asarray(rx, dtype=np.float64)
            ry = np.asarray(ry, dtype=np.float64)
            xs.append(rx)
            ys.append(ry)
            rvo.append(rvo[-1] + rx.shape[0])
        pro.append(len(rvo) - 1)
    x = np.concatenate(xs) if xs else np.zeros(0)
    y = np.concatenate(ys) if ys else np.zeros(0)
    return Polygons(np.asarray(pro, np.int64), np.asarray(rvo, np.int64), x, y)


def _jag_ridges(A, B, Sp, Sq, level, rng, amp_frac, lam, decay):
    """Midpoint-displacement graphs over ridges A->B; returns interior points [n, K-1, 2]."""
    K = 1 << level
    d = B - A
    L = np.hypot(d[:, 0], d[:, 1])
    ok = L > 1e-9
    Ls = np.where(ok, L, 1.0)
    nrm = np.stack([-d[:, 1] / Ls, d[:, 0] / Ls], axis=1)
    hp = np.einsum("ij,ij->i", Sp - A, nrm)
    hq = np.einsum("ij,ij->i", Sq - A, nrm)
    tp = np.einsum("ij,ij->i", Sp - A, d) / (Ls * Ls)
    tq = np.einsum("ij,ij->i", Sq - A, d) / (Ls * Ls)
    mp = np.maximum(1.0, np.maximum(tp, 1.0 - tp))
    mq = np.maximum(1.0, np.maximum(tq, 1.0 - tq))
    # the side with positive height gets the upper bound
    Epos = np.where(hp > 0, np.abs(hp) / mp, np.abs(hq) / mq)
    Eneg = np.where(hp > 0, np.abs(hq) / mq, np.abs(hp) / mp)
    t = np.arange(K + 1, dtype=np.float64) / K
    tri = np.minimum(t, 1.0 - t)[None, :]
    upper = lam * Epos[:, None] * tri
    lower = -lam * Eneg[:, None] * tri
    h = np.zeros((A.shape[0], K + 1))
    amp = amp_frac * L
    for lev in range(level):
        step = K >> lev
        half = step // 2
        idx = np.arange(half, K, step)
        h[:, idx] = 0.5 * (h[:, idx - half] + h[:, idx + half]) + \
            amp[:, None] * rng.uniform(-1.0, 1.0, size=(A.shape[0], idx.shape[0]))
        h[:, idx] = np.minimum(np.maximum(h[:, idx], lower[:, idx]), upper[:, idx])
        amp = amp * decay
    h[~ok] = 0.0
    ti = t[1:-1][None, :, None]
    pts = A[:, None, :] + ti * d[:, None, :] + h[:, 1:-1, None] * nrm[:, None, :]
    return pts, ok


def _jagged_circle(c, R, level, rng, wobble=0.15):
    M = 1 << level
    th = 2 * np.pi * np.arange(M) / M
    rad = np.ones(M)
    for f in (2, 3, 5, 8, 13):
        rad += (wobble / 5.0) * np.sin(f * th + rng.uniform(0, 2 * np.pi))
    rad += (wobble / 5.0) * rng.uniform(-1, 1, size=M)
    return c[0] + R * rad * np.cos(th), c[1] + R * rad * np.sin(th)


def _seg_dist(p, ax, ay, bx, by):
    dx, dy = bx - ax, by - ay
    ll = dx * dx + dy * dy
    t = np.where(ll > 0, ((p[0] - ax) * dx + (p[1] - ay) * dy) / np.where(ll > 0, ll, 1), 0.0)
    t = np.clip(t, 0, 1)
    qx, qy = ax + t * dx, ay + t * dy
    return np.hypot(p[0] - qx, p[1] - qy)


def voronoi_tiling(width: float, height: float, gt, n_seeds: int, level: int, seed: int,
                   n_holes: int = 0, mask=None, amp_frac: float = 0.18, lam: float = 0.8,
                   decay: float = 0.55, hole_level: int | None = None, east_bias: float = 0.0) -> Polygons:
    """Jagged Voronoi tiling of [0,width]x[0,height] (cell space), mapped through gt.

    mask(a, b) -> bool array over normalised seed positions keeps a subset of the cells.
    Polygons are ordered: kept Voronoi cells (seed order), then enclaves.
    """
    from scipy.spatial import Voronoi

    rng = np.random.default_rng(seed)
    W, H = float(width), float(height)
    u = rng.uniform(0, W, n_seeds)
    if east_bias > 0:
        nb = int(n_seeds * east_bias)
        u[:nb] = W * (0.5 + 0.5 * rng.uniform(0, 1, nb))
    v = rng.uniform(0, H, n_seeds)
    S = np.stack([u, v], axis=1)
    pts = np.concatenate([S, np.stack([-u, v], 1), np.stack([2 * W - u, v], 1),
                          np.stack([u, -v], 1), np.stack([u, 2 * H - v], 1)])
    vor = Voronoi(pts)
    VV = vor.vertices
    rp = vor.ridge_points
    rv = np.asarray(vor.ridge_vertices)
    n = n_seeds
    interior = (rp[:, 0] < n) & (rp[:, 1] < n) & (rv[:, 0] >= 0) & (rv[:, 1] >= 0)
    # canonical direction min vertex -> max vertex
    va = np.minimum(rv[:, 0], rv[:, 1])
    vb = np.maximum(rv[:, 0], rv[:, 1])
    ridge_of = {}
    for j in np.nonzero((rp[:, 0] < n) | (rp[:, 1] < n))[0]:
        ridge_of[(int(va[j]), int(vb[j]))] = int(j)
    jag_idx = np.nonzero(interior)[0]
    pts_j, ok_j = _jag_ridges(VV[va[jag_idx]], VV[vb[jag_idx]], pts[rp[jag_idx, 0]], pts[rp[jag_idx, 1]],
                              level, rng, amp_frac, lam, decay)
    jag_pos = {int(j): i for i, j in enumerate(jag_idx)}

    keep = np.ones(n, dtype=bool)
    if mask is not None:
        keep = np.asarray(mask(S[:, 0] / W, S[:, 1] / H), dtype=bool)
    rings_u = []  # per kept polygon: list of (u, v) rings in cell space
    kept_ids = []
    for i in range(n):
        if not keep[i]:
            continue
        reg = vor.regions[vor.point_region[i]]
        reg = np.asarray(reg)
        assert reg.size >= 3 and (reg >= 0).all()
        ang = np.arctan2(VV[reg, 1] - S[i, 1], VV[reg, 0] - S[i, 0])
        reg = reg[np.argsort(ang)]
        us, vs = [], []
        m = reg.shape[0]
        for e in range(m):
            a, b = int(reg[e]), int(reg[(e + 1) % m])
            us.append(VV[a:a + 1, 0])
            vs.append(VV[a:a + 1, 1])
            j = ridge_of.get((min(a, b), max(a, b)))
            if j is not None and j in jag_pos and ok_j[jag_pos[j]]:
                p = pts_j[jag_pos[j]]
                if a > b:
                    p = p[::-1]
                us.append(p[:, 0])
                vs.append(p[:, 1])
        rings_u.append([(np.concatenate(us), np.concatenate(vs))])
        kept_ids.append(i)

    # enclaves (holes + separate polygons)
    hl = hole_level if hole_level is not None else max(4, level - 1)
    enclaves = []
    if n_holes > 0 and kept_ids:
        hosts = rng.choice(len(kept_ids), size=min(n_holes, len(kept_ids)), replace=False)
        for h in hosts:
            ru, rvv = rings_u[h][0]
            c = S[kept_ids[h]]
            rmin = _seg_dist(c, ru, rvv, np.roll(ru, -1), np.roll(rvv, -1)).min()
            cu, cv = _jagged_circle(c, 0.4 * rmin, hl, rng)
            rings_u[h].append((cu, cv))
            enclaves.append([(cu, cv)])
    rings_u.extend(enclaves)

    gt0, gt1, _, gt3, _, gt5 = [float(g) for g in gt]
    polys = []
    for rings in rings_u:
        polys.append([(gt0 + ru * gt1, gt3 + rvv * gt5) for ru, rvv in rings])
    P = from_rings(polys)
    P.meta = {"n_seeds": n_seeds, "level": level, "seed": seed, "n_holes": len(enclaves),
              "kept": len(kept_ids)}
    return P


def conus_mask(a, b):
    """CONUS-like land mask over normalised coordinates (a east, b south)."""
    body = ((a - 0.50) / 0.49) ** 2 + ((b - 0.42) / 0.44) ** 2 <= 1.0
    florida = (a > 0.80) & (a < 0.88) & (b > 0.70) & (b < 0.97)
    gulf = ((a - 0.66) / 0.10) ** 2 + ((b - 0.93) / 0.12) ** 2 <= 1.0
    lakes = ((a - 0.72) / 0.05) ** 2 + ((b - 0.18) / 0.06) ** 2 <= 1.0
    return (body | florida) & ~gulf & ~lakes
