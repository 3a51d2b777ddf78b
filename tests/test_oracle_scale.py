"""O0 == O1 at the full-size configs (SURVEY.md §8c "Self-consistency" pin): the literal definition
(O0, with its exact bounding-box prefilter, itself pinned to the prefilter-free loop in
tests/test_oracle_pins.py) and the row-hoisted O1 — the only checker fast enough for whole
full-size matrices — must agree on the jagged lon/lat polygons of the state and CONUS configs
(Fig. 5's predicate, evaluated literally vs hoisted per row).

Per-cell comparison through CODED windows: the oracle sees a window whose cells carry distinct
bin codes (every other cell nodata), so out[k][code] is exactly "cell `code` is inside polygon k"
for both oracles.  Cells: >= 10^5 random cells (100 per row of 125 random runs of 8 rows, all polygons);
all cells of >= 50 whole 256 x 256 tiles (half uniform, half drawn from tiles that hold a polygon
vertex, i.e. boundary tiles), against the polygons whose bounding box comes within 4 cells of the
tile (the others contain none of its centres: the prefilter argument O0's pin covers)."""
import numpy as np
import pytest

import oracle
from synth.configs import CONUS, STATE

NODATA = -32768


@pytest.fixture(scope="module", params=["state", "conus"])
def cfgP(request):
    cfg = {"state": STATE, "conus": CONUS}[request.param]
    return cfg, cfg.polygons()


def _compare(win, row0, col0, cfg, P, nbins):
    bins = oracle.make_bins(nbins, nodata=NODATA)
    a = oracle.o0(win, cfg.gt, P, bins, row0=row0, col0=col0, prefilter=True)
    b = oracle.o1(win, cfg.gt, P, bins, row0=row0, col0=col0)
    assert np.array_equal(a, b), (row0, col0, int((a != b).sum()))
    return int(a.sum())


def test_o0_equals_o1_random_cells(cfgP):
    cfg, P = cfgP
    rng = np.random.default_rng(569)
    per_row, group = 100, 8
    starts = np.sort(rng.choice(cfg.rows // group, size=125, replace=False)) * group
    rows = (starts[:, None] + np.arange(group)[None, :]).ravel()
    inside = 0
    for g in range(0, rows.size, group):
        rr = rows[g:g + group]
        # one window of 8 consecutive random rows, 100 random cells coded in each
        r0, r1 = int(rr[0]), int(rr[-1]) + 1
        win = np.full((r1 - r0, cfg.cols), NODATA, dtype=np.int16)
        code = 0
        for r in rr:
            cols = rng.choice(cfg.cols, size=per_row, replace=False)
            win[r - r0, cols] = np.arange(code, code + per_row, dtype=np.int16)
            code += per_row
        inside += _compare(win, r0, 0, cfg, P, code)
    # the configs' polygons cover most of the extent: most sampled centres are inside one
    assert inside > 0.4 * rows.size * per_row


def _tiles(cfg, P, n, rng):
    T = 256
    TR, TC = cfg.rows // T, cfg.cols // T
    picks = set()
    while len(picks) < n // 2:
        picks.add((int(rng.integers(TR)), int(rng.integers(TC))))
    vr = ((P.y - cfg.gt[3]) / cfg.gt[5]).astype(np.int64) // T
    vc = ((P.x - cfg.gt[0]) / cfg.gt[1]).astype(np.int64) // T
    ok = (vr >= 0) & (vr < TR) & (vc >= 0) & (vc < TC)
    cand = np.unique(vr[ok] * TC + vc[ok])
    for t in rng.choice(cand, size=n - len(picks), replace=False):
        picks.add((int(t) // TC, int(t) % TC))
    return sorted(picks), T


def test_o0_equals_o1_whole_tiles(cfgP):
    cfg, P = cfgP
    rng = np.random.default_rng(570)
    tiles, T = _tiles(cfg, P, 50, rng)
    # per-polygon bounding boxes in cell coordinates
    nv = np.diff(P.ring_vert_off)
    first = P.ring_vert_off[P.poly_ring_off[:-1]]
    last = P.ring_vert_off[P.poly_ring_off[1:]]
    u = (P.x - cfg.gt[0]) / cfg.gt[1]
    v = (P.y - cfg.gt[3]) / cfg.gt[5]
    bb = np.array([[u[a:b].min(), u[a:b].max(), v[a:b].min(), v[a:b].max()] if b > a else [1, 0, 1, 0]
                   for a, b in zip(first, last)])
    assert nv.sum() == P.n_vert
    boundary_tiles = 0
    code_rows = 32768 // T  # rows per window with distinct codes 0..32767
    for tr, tc in tiles:
        r0, c0 = tr * T, tc * T
        near = np.nonzero((bb[:, 1] >= c0 - 4) & (bb[:, 0] <= c0 + T + 4) &
                          (bb[:, 3] >= r0 - 4) & (bb[:, 2] <= r0 + T + 4))[0]
        Ps = P.subset(near)
        owners = set()
        for h in range(0, T, code_rows):
            win = (np.arange(code_rows * T, dtype=np.int32).reshape(code_rows, T)).astype(np.int16)
            a = oracle.o0(win, cfg.gt, Ps, oracle.make_bins(32768), row0=r0 + h, col0=c0, prefilter=True)
            b = oracle.o1(win, cfg.gt, Ps, oracle.make_bins(32768), row0=r0 + h, col0=c0)
            assert np.array_equal(a, b), (tr, tc, h)
            owners |= set(np.nonzero(a.any(axis=1))[0].tolist())
        boundary_tiles += len(owners) > 1
    assert boundary_tiles >= 10  # the comparison reached tiles where polygons meet
