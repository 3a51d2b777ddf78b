"""GPU parity: libzh (through the C ABI) vs the CPU oracle, element by element, bit-exact.

Inputs come from synth/ (seeded; the device raster is generated on the GPU and checked equal to
the host raster the oracle reads).  The oracle never sees anything computed by libzh.
"""
import numpy as np
import pytest

import oracle
from synth.configs import TINY, TINY_LONLAT
from synth.dem import KIND_LINMOD, DemSpec, fill_device, fill_host
from synth.polygons import from_rings

pytestmark = pytest.mark.gpu


def _zh():
    from paper_conf_ipps_zhangw14_b200 import zh
    return zh


def device_raster(spec, rows, cols, row0=0, nrows=None, pitch=None, gcols=None):
    import torch
    nrows = rows - row0 if nrows is None else nrows
    pitch = pitch or ((cols + 7) // 8 * 8)
    t = torch.full((nrows, pitch), 12345, dtype=torch.int16, device="cuda")
    fill_device(spec, gcols or cols, t.data_ptr(), row0, 0, nrows, cols, pitch,
                torch.cuda.current_stream().cuda_stream)
    return t


def gpu_hist(t, gt, P, nbins, tile, cols, rows=None, row0=0, **kw):
    """Run both libzh paths — the four steps (zh_tile_hist, zh_aggregate, zh_pip_update) and the
    fused one (zh_fused_update) — check they agree bit for bit, and return the result."""
    zh = _zh()
    res = []
    for fused in (False, True):
        with zh.ZonalHistogram(t, gt, P, nbins, tile=tile, cols=cols, rows=rows, row0=row0, fused=fused,
                               **kw) as z:
            res.append(z.run())
    assert (res[0] == res[1]).all(), "fused path differs from the four-step path"
    return res[1]


@pytest.fixture(scope="module")
def tiny():
    cfg = TINY
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    bins = oracle.make_bins(cfg.nbins, nodata=cfg.nodata)
    H = oracle.o0(R, cfg.gt, P, bins)
    return cfg, P, R, H


def test_device_generator_matches_host(tiny, cuda_device):
    cfg, P, R, _ = tiny
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    assert (t.cpu().numpy()[:, :cfg.cols] == R).all()


@pytest.mark.parametrize("out_u64", [True, False])
def test_tiny_bit_exact(tiny, cuda_device, out_u64):
    cfg, P, R, H = tiny
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    G = gpu_hist(t, cfg.gt, P, cfg.nbins, cfg.tile, cfg.cols, nodata=cfg.nodata, out_u64=out_u64)
    assert (G.astype(np.uint64) == H).all()


@pytest.mark.parametrize("tile", [1, 5, 8, 13, 64, 100, 128, 256, 360, 1000, 1024, 2048])
def test_tiny_tile_size_invariance(tiny, cuda_device, tile):
    cfg, P, R, H = tiny
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    G = gpu_hist(t, cfg.gt, P, cfg.nbins, tile, cfg.cols, nodata=cfg.nodata)
    assert (G == H).all()


def test_force_all_intersect_identical(tiny, cuda_device):
    cfg, P, R, H = tiny
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    for tile in (64, 128):
        G = gpu_hist(t, cfg.gt, P, cfg.nbins, tile, cfg.cols, nodata=cfg.nodata, force_isect=True)
        assert (G == H).all()


def test_step1_tile_histograms_vs_bincount(tiny, cuda_device):
    cfg, P, R, H = tiny
    zh = _zh()
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    T = 100  # ragged edge tiles, unaligned columns
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=T, cols=cfg.cols, nodata=cfg.nodata) as z:
        z.zh_tile_hist()
        th = z.tile_hist_host()
    TC = (cfg.cols + T - 1) // T
    for tid in range(th.shape[0]):
        tr, tc = divmod(tid, TC)
        blk = R[tr * T:(tr + 1) * T, tc * T:(tc + 1) * T].astype(np.int64).ravel()
        blk = blk[blk != cfg.nodata]
        ref = np.bincount(np.clip(blk, 0, cfg.nbins - 1), minlength=cfg.nbins)
        assert (th[tid] == ref).all(), tid


def test_step2_classification_is_sound(tiny, cuda_device):
    """Inside pairs: every cell centre of the tile is inside (oracle); outside (unlisted) MBB
    tiles: no centre inside; intersect pairs are whatever is left."""
    cfg, P, R, H = tiny
    zh = _zh()
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    T = 64
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=T, cols=cfg.cols, nodata=cfg.nodata) as z:
        ni, nx = z.zh_pair_tiles()
        ins, isx = z.pairs_host()
    assert ni > 0 and nx > 0
    TC = (cfg.cols + T - 1) // T
    rr, cc = np.meshgrid(np.arange(cfg.rows), np.arange(cfg.cols), indexing="ij")
    mem = oracle.membership(rr.ravel(), cc.ravel(), cfg.gt, P).reshape(cfg.rows, cfg.cols, P.n_poly)
    listed = set()
    for tile, k in ins:
        tr, tc = divmod(int(tile), TC)
        assert mem[tr * T:(tr + 1) * T, tc * T:(tc + 1) * T, k].all()
        listed.add((int(tile), int(k)))
    for tile, k in isx:
        listed.add((int(tile), int(k)))
    for tid in range(TC * TC):
        tr, tc = divmod(tid, TC)
        blk = mem[tr * T:(tr + 1) * T, tc * T:(tc + 1) * T]
        for k in np.nonzero(blk.reshape(-1, P.n_poly).any(axis=0))[0]:
            assert (tid, int(k)) in listed
    # lists sorted by (polygon, tile)
    for L in (ins, isx):
        key = L[:, 1].astype(np.int64) * (1 << 32) + L[:, 0]
        assert (np.diff(key) > 0).all()


def test_tiny_lonlat_bit_exact(cuda_device):
    cfg = TINY_LONLAT
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    for tile in (32, 128, 200):
        assert (gpu_hist(t, cfg.gt, P, cfg.nbins, tile, cfg.cols, nodata=cfg.nodata) == H).all()


@pytest.mark.parametrize("flip", ["x", "y", "xy"])
def test_flipped_geotransforms(tiny, cuda_device, flip):
    cfg, P, R, _ = tiny
    gt = list(cfg.gt)
    if "x" in flip:
        gt[0], gt[1] = float(cfg.cols), -1.0
    if "y" in flip:
        gt[3], gt[5] = 0.0, 1.0
    H = oracle.o1(R, gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    for tile in (64, 100):
        assert (gpu_hist(t, gt, P, cfg.nbins, tile, cfg.cols, nodata=cfg.nodata) == H).all()


@pytest.mark.parametrize("lo,width,nbins,drop,nodata", [(0, 1, 256, True, -32768), (-100, 3, 77, False, None),
                                                         (20, 7, 9, True, -32768), (-20, 1, 300, False, 150),
                                                         # nodata below lo with values below nodata
                                                         # (tiny: -157..401): clamp counts them in
                                                         # bin 0, drop drops them
                                                         (0, 1, 256, False, -100), (0, 1, 256, True, -100),
                                                         (-50, 1, 5000, False, -120), (-150, 1, 600, False, -151),
                                                         # k_mixed_cells layouts: flat without nodata
                                                         # (kForm 0), power-of-two B (7,000 bins)
                                                         (0, 1, 4000, False, None), (0, 1, 7000, False, -32768)])
def test_bin_mappings(tiny, cuda_device, lo, width, nbins, drop, nodata):
    cfg, P, R, _ = tiny
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(nbins, lo=lo, width=width, nodata=nodata, oor_drop=drop))
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    G = gpu_hist(t, cfg.gt, P, nbins, 128, cfg.cols, lo=lo, width=width, nodata=nodata, oor_drop=drop)
    assert (G == H).all()


def test_ragged_raster_and_pitch(cuda_device):
    """1000 x 1003 raster (cols not a multiple of 8), pitch 1016, tiles 96 and 128 (ragged)."""
    rows, cols = 1000, 1003
    gt = (0.0, 1.0, 0.0, float(rows), 0.0, -1.0)
    spec = DemSpec(seed=21, base=-150, macro_amp=900, fine_amp=200)
    from synth.polygons import voronoi_tiling
    P = voronoi_tiling(cols, rows, gt, 12, 5, 22, n_holes=2)
    R = fill_host(spec, cols, 0, 0, rows, cols)
    H = oracle.o1(R, gt, P, oracle.make_bins(256, nodata=-32768))
    t = device_raster(spec, rows, cols, pitch=1016)
    for tile in (96, 128, 1003):
        assert (gpu_hist(t, gt, P, 256, tile, cols, nodata=-32768) == H).all()


def test_hand_worked_cases_on_gpu(cuda_device):
    import os
    import torch
    gold = os.path.join(os.path.dirname(__file__), "golden", "hand_counts.txt")
    names, polys, want = [], [], []
    for line in open(gold):
        if line.startswith("#") or not line.strip():
            continue
        n, rings, c, _ = [f.strip() for f in line.split("|")]
        rr = []
        for part in rings.split("/"):
            pts = [tuple(map(float, p.split(","))) for p in part.split()]
            rr.append((np.array([p[0] for p in pts]), np.array([p[1] for p in pts])))
        names.append(n)
        polys.append(rr)
        want.append(int(c))
    P = from_rings(polys)
    t = torch.zeros((20, 24), dtype=torch.int16, device="cuda")
    for tile in (1, 3, 4, 8, 24):
        G = gpu_hist(t, (0.0, 1.0, 0.0, 20.0, 0.0, -1.0), P, 1, tile, 24)
        assert [int(g) for g in G[:, 0]] == want, (tile, names)


def test_degenerate_polygons(cuda_device):
    cfg = TINY
    R = fill_host(cfg.dem, cfg.cols, 0, 0, 64, 64)
    gt = (0.0, 1.0, 0.0, 64.0, 0.0, -1.0)
    sq = (np.array([5.0, 30, 30, 5]), np.array([5.0, 5, 30, 30]))
    P = from_rings([[], [(np.array([]), np.array([]))], [(np.array([3.0]), np.array([3.0]))],
                    [(np.array([3.0, 40]), np.array([3.0, 50]))], [sq],
                    [(np.append(sq[0], 5.0), np.append(sq[1], 5.0))], [(sq[0] + 1000, sq[1])],
                    [(np.repeat(sq[0], 2), np.repeat(sq[1], 2))], [(sq[0] - 1000, sq[1] + 1e6)]])
    H = oracle.o0(R, gt, P, oracle.make_bins(256, nodata=-32768))
    t = device_raster(cfg.dem, 64, 64, gcols=cfg.cols)
    for tile in (8, 16, 64):
        assert (gpu_hist(t, gt, P, 256, tile, 64, nodata=-32768) == H).all()
    # no polygons at all
    E = from_rings([])
    assert gpu_hist(t, gt, E, 256, 16, 64).shape == (0, 256)


def test_tile_row_shards_sum_to_whole(tiny, cuda_device):
    """Shards of whole tile rows (the multi-GPU decomposition) sum to the single-shard result."""
    cfg, P, R, H = tiny
    T = 128
    for nsh in (2, 3, 8):
        tiles_rows = (cfg.rows + T - 1) // T
        per = -(-tiles_rows // nsh)
        acc = np.zeros_like(H)
        for g in range(nsh):
            r0 = min(cfg.rows, g * per * T)
            r1 = min(cfg.rows, (g + 1) * per * T)
            t = device_raster(cfg.dem, cfg.rows, cfg.cols, row0=r0, nrows=r1 - r0)
            acc += gpu_hist(t, cfg.gt, P, cfg.nbins, T, cfg.cols, rows=cfg.rows, row0=r0, nodata=cfg.nodata)
        assert (acc == H).all()


def test_host_raster_path(tiny, cuda_device):
    import torch
    cfg, P, R, H = tiny
    pinned = torch.from_numpy(R.copy()).pin_memory()
    G = gpu_hist(pinned, cfg.gt, P, cfg.nbins, cfg.tile, cfg.cols, nodata=cfg.nodata)
    assert (G == H).all()


@pytest.mark.parametrize("tile", [100, 128])
def test_host_raster_needed_tiles_only(tiny, cuda_device, tile):
    """zh_run of the fused path on a HOST raster uploads only the tiles some pair needs (2-D copies of
    tile runs, rounded out to 16-byte vectors; tiles not multiples of 8 wide; pitch > cols), and the
    device copy outside them is never read: poisoned cached blocks and a poisoned pitch tail change
    nothing."""
    import torch
    zh = _zh()
    cfg, P, R, H = tiny
    keep = [0, 5, 11, 15]  # a few polygons (15 = the enclave): most tiles have no pair
    Ps = P.subset(keep)
    pitch = cfg.cols + 24
    host = np.full((cfg.rows, pitch), -7777, dtype=np.int16)
    host[:, :cfg.cols] = R
    pinned = torch.from_numpy(host).pin_memory()
    # leave a poisoned block of the right size in libzh's cache: the context reuses it for its copy
    with zh.ZonalHistogram(torch.full_like(pinned, 31000), cfg.gt, Ps, cfg.nbins, tile=tile, cols=cfg.cols,
                           nodata=cfg.nodata, fused=False) as z:
        z.run()
    assert zh.LIB.zh_cache_bytes() > 0
    for fused in (True, False):
        with zh.ZonalHistogram(pinned, cfg.gt, Ps, cfg.nbins, tile=tile, cols=cfg.cols, nodata=cfg.nodata,
                               fused=fused) as z:
            G = z.run()
            st = z.stats()
        assert (G == H[keep]).all()
        full = cfg.rows * pitch * 2
        if fused:
            assert 0 < st["h2d_bytes"] < full // 2, st["h2d_bytes"]
        else:
            assert st["h2d_bytes"] == full


def test_cache_trim(cuda_device):
    zh = _zh()
    zh.LIB.zh_trim_cache(1)
    assert zh.LIB.zh_cache_bytes() == 0


def test_overlapping_polygons_and_linear_pattern(cuda_device):
    """Overlapping polygons count a cell in each; v = (r*cols + c) mod 4093 exercises all bins."""
    rows, cols = 512, 768
    gt = (10.0, 0.5, 0.0, 300.0, 0.0, -0.25)
    spec = DemSpec(kind=KIND_LINMOD, pattern_mod=4093, pattern_off=-7)
    R = fill_host(spec, cols, 0, 0, rows, cols)
    rng = np.random.default_rng(5)
    polys = []
    for _ in range(40):
        cx, cy = rng.uniform(10, 394), rng.uniform(172, 300)
        th = np.sort(rng.uniform(0, 2 * np.pi, 30))
        rad = rng.uniform(5, 60, 30)
        polys.append([(cx + rad * np.cos(th), cy + rad * np.sin(th))])
    P = from_rings(polys)
    H = oracle.o1(R, gt, P, oracle.make_bins(4096, lo=-7))
    t = device_raster(spec, rows, cols)
    for tile in (32, 64, 256):
        assert (gpu_hist(t, gt, P, 4096, tile, cols, lo=-7) == H).all()


@pytest.mark.parametrize("out_u64", [True, False])
def test_zonal_stats_match_oracle(tiny, cuda_device, out_u64):
    """zh_zonal_stats (exact integers from the device histogram) == the oracle's
    statistics of the oracle histogram; clamped default bins and an unclamped mapping."""
    cfg, P, R, H = tiny
    zh = _zh()
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    for lo, nb in ((0, cfg.nbins), (-400, 1200)):
        Hb = H if lo == 0 else oracle.o1(R, cfg.gt, P, oracle.make_bins(nb, lo=lo, nodata=cfg.nodata))
        want = oracle.zonal_stats(Hb)
        for fused in (False, True):
            with zh.ZonalHistogram(t, cfg.gt, P, nb, lo=lo, tile=cfg.tile, cols=cfg.cols, nodata=cfg.nodata,
                                   out_u64=out_u64, fused=fused) as z:
                z.run()
                got = z.zh_zonal_stats()
                derived = z.zonal_stats()
            assert (got == want).all()
            nz = want[:, 0] > 0
            assert (derived["min"][nz] == lo + want[nz, 1]).all()
            assert (derived["count"] == want[:, 0]).all()


@pytest.mark.parametrize("rep", [(0.0, 0.0), (0.0, 1.0), (1.0, 1.0), (0.25, 0.75)])
def test_representative_points(tiny, cuda_device, rep):
    """cell corners / arbitrary points of the cell instead of the centre."""
    cfg, P, R, _ = tiny
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata), rep=rep)
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    for tile in (64, 128):
        assert (gpu_hist(t, cfg.gt, P, cfg.nbins, tile, cfg.cols, nodata=cfg.nodata, rep=rep) == H).all()
    lon = TINY_LONLAT
    P2 = lon.polygons()
    R2 = fill_host(lon.dem, lon.cols, 0, 0, lon.rows, lon.cols)
    H2 = oracle.o1(R2, lon.gt, P2, oracle.make_bins(lon.nbins, nodata=lon.nodata), rep=rep)
    t2 = device_raster(lon.dem, lon.rows, lon.cols)
    assert (gpu_hist(t2, lon.gt, P2, lon.nbins, 128, lon.cols, nodata=lon.nodata, rep=rep) == H2).all()


@pytest.mark.parametrize("nbins,lo,width", [(20000, -10000, 1), (49152, -32768, 1), (3000, -400, 2)])
def test_large_and_generic_histograms(tiny, cuda_device, nbins, lo, width):
    """Histograms beyond the packed 16x2 path (nbins > 16000, width > 1): the generic per-cell
    path and the shared-memory budget logic (49,152 bins = 192 KB per CTA)."""
    cfg, P, R, _ = tiny
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(nbins, lo=lo, width=width, nodata=cfg.nodata))
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    G = gpu_hist(t, cfg.gt, P, nbins, 128, cfg.cols, lo=lo, width=width, nodata=cfg.nodata)
    assert (G == H).all()


def test_lonlat_vertices_exactly_on_centres(cuda_device):
    """Non-dyadic equality cases: a 1-arc-second lon/lat geotransform with polygon
    vertices placed EXACTLY on computed cell centres — x = gt0 + (c + 0.5) gt1, y = gt3 + (r + 0.5) gt5,
    the same binary64 expressions both sides evaluate — so centre rows meet vertices (ya == yc: the
    half-open straddle rule at its boundary, k_mbb_edges' exact row intervals), vertical edges sit on
    centre columns (xi == xc: not a crossing) and shared borders pass through centres.  GPU ==
    literal O0 (no prefilter) at several tile sizes, both paths."""
    ARC = 1.0 / 3600.0
    rows, cols = 600, 704
    gt = (-100.0, ARC, 0.0, 40.0, 0.0, -ARC)
    xc = lambda c: gt[0] + (c + 0.5) * gt[1]
    yc = lambda r: gt[3] + (r + 0.5) * gt[5]
    rng = np.random.default_rng(31)
    polys = []
    for _ in range(14):  # star-shaped, vertices on centres
        cr, cc = rng.integers(60, rows - 60), rng.integers(60, cols - 60)
        n = int(rng.integers(5, 40))
        th = np.sort(rng.uniform(0, 2 * np.pi, n))
        rad = rng.uniform(8, 55, n)
        r = np.clip(np.rint(cr + rad * np.sin(th)), 0, rows - 1).astype(int)
        c = np.clip(np.rint(cc + rad * np.cos(th)), 0, cols - 1).astype(int)
        polys.append([(np.array([xc(v) for v in c]), np.array([yc(v) for v in r]))])
    for _ in range(6):  # axis-aligned boxes with corners on centres, one with a hole on centres
        r0, c0 = rng.integers(0, rows - 80), rng.integers(0, cols - 80)
        h, w = rng.integers(5, 79, 2)
        box = (np.array([xc(c0), xc(c0 + w), xc(c0 + w), xc(c0)]), np.array([yc(r0), yc(r0), yc(r0 + h), yc(r0 + h)]))
        polys.append([box])
    r0, c0 = 200, 300
    outer = (np.array([xc(c0), xc(c0 + 90), xc(c0 + 90), xc(c0)]), np.array([yc(r0), yc(r0), yc(r0 + 70), yc(r0 + 70)]))
    hole = (np.array([xc(c0 + 10), xc(c0 + 30), xc(c0 + 30), xc(c0 + 10)]),
            np.array([yc(r0 + 10), yc(r0 + 10), yc(r0 + 50), yc(r0 + 50)]))
    polys.append([outer, hole])
    P = from_rings(polys)
    spec = TINY.dem
    R = fill_host(spec, cols, 0, 0, rows, cols)
    H = oracle.o0(R, gt, P, oracle.make_bins(256, nodata=-32768))
    assert H.sum() > 0
    t = device_raster(spec, rows, cols)
    for tile in (16, 64, 100, 128, 704):
        assert (gpu_hist(t, gt, P, 256, tile, cols, nodata=-32768) == H).all(), tile


@pytest.mark.parametrize("teeth", [700, 1600, 3500])
@pytest.mark.parametrize("flip_x", [False, True])
def test_comb_polygon_many_crossings(cuda_device, teeth, flip_x):
    """A comb whose every tooth row is crossed by 2 x teeth edges: 1,400 crossings per row fit the
    band kernel's shared flip list several rows at a time, 3,200 one row at a time, and 7,000
    overflow it (the exact per-(pair, row) slow path of k_parity.cu).  Mirrored x (gt1 < 0) takes
    the suffix form of the crossings.  GPU == literal O0."""
    rows, cols = 48, 1024
    gt = [0.0, 1.0, 0.0, float(rows), 0.0, -1.0]
    if flip_x:
        gt[0], gt[1] = float(cols), -1.0
    xs, ys = [3.25], [4.5]
    step = (cols - 8.0) / teeth
    for i in range(teeth):
        x0 = 4.0 + i * step
        xs += [x0 + 0.1 * step, x0 + 0.3 * step, x0 + 0.6 * step, x0 + 0.9 * step]
        ys += [4.5, 40.25, 40.25, 4.5]
    xs += [cols - 3.5, cols - 3.5, 3.25]
    ys += [4.5, 1.75, 1.75]
    P = from_rings([[(np.array(xs), np.array(ys))], [(np.array([1.0, 900.0, 900.0, 1.0]),
                                                       np.array([20.0, 20.0, 30.0, 30.0]))]])
    spec = TINY.dem
    R = fill_host(spec, cols, 0, 0, rows, cols)
    H = oracle.o0(R, gt, P, oracle.make_bins(256, nodata=-32768), prefilter=True)
    assert H[0].sum() > 0
    t = device_raster(spec, rows, cols)
    for tile in (16, 48, 256):
        assert (gpu_hist(t, gt, P, 256, tile, cols, nodata=-32768) == H).all(), tile


@pytest.mark.parametrize("fused", [True, False])
def test_step_graph_replays(tiny, cuda_device, fused):
    """zh_step_graph: first call direct (learns the sizes), second captures, later calls replay the
    CUDA graph — every result equals the oracle; timing events work inside the graph; a new output
    buffer drops the graph and the next replay writes the new buffer."""
    import torch
    zh = _zh()
    cfg, P, R, H = tiny
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=cfg.tile, cols=cfg.cols, nodata=cfg.nodata,
                           fused=fused) as z:
        z.set_timing(True)
        for i in range(4):
            z.zh_step_graph()
            got = z.output_device().cpu().numpy().view(np.uint64)
            assert (got == H).all(), i
            ms = z.step_ms()
            assert ms["step2_pair_tiles"] > 0
        out2 = torch.zeros((P.n_poly, cfg.nbins), dtype=torch.int64, device="cuda")
        z.set_output(out2)
        for i in range(3):
            z.zh_step_graph()
            assert (out2.cpu().numpy().view(np.uint64) == H).all(), i
        st = z.stats()  # a syncing call: also checks the device count guard
        assert st["n_isect"] > 0


def test_known_sizes_guard_fires(tiny, cuda_device, monkeypatch):
    """The host-sync-free steps trust the list sizes learnt by a context's first zh_pair_tiles; the
    device check must report a step whose counts differ (ZH_TEST_BAD_SIZES makes the context
    remember a wrong candidate count): the next syncing call fails with ZH_ERR_STATE."""
    zh = _zh()
    cfg, P, R, H = tiny
    t = device_raster(cfg.dem, cfg.rows, cfg.cols)
    monkeypatch.setenv("ZH_TEST_BAD_SIZES", "1")
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=cfg.tile, cols=cfg.cols, nodata=cfg.nodata) as z:
        z.zh_pair_tiles()      # learns the sizes (and, under the hook, a wrong candidate count)
        z.zh_fused_update()
        z.zh_pair_tiles()      # host-sync-free: the device check compares
        z.zh_fused_update()
        with pytest.raises(zh.ZhError) as ei:
            z.stats()
        assert ei.value.status == zh.ZH_ERR_STATE
    monkeypatch.delenv("ZH_TEST_BAD_SIZES")
    with zh.ZonalHistogram(t, cfg.gt, P, cfg.nbins, tile=cfg.tile, cols=cfg.cols, nodata=cfg.nodata) as z:
        for _ in range(3):
            z.zh_pair_tiles()
            z.zh_fused_update()
        z.stats()  # no mismatch: no error
        assert (z.output_device().cpu().numpy().view(np.uint64) == H).all()


@pytest.mark.parametrize("seed", range(12))
def test_random_configurations_fuzz(cuda_device, seed):
    """Seeded random configurations against the literal O0: raster size and pitch, geotransform
    (dyadic or lon/lat, either orientation), tile size, bin mapping (lo, width, nbins, clamp / drop,
    nodata in or below the range), output width, and random polygons (stars, boxes on centres,
    holes, overlaps, degenerate rings) — both libzh paths and the CUDA-graph step."""
    import torch
    zh = _zh()
    rng = np.random.default_rng(1000 + seed)
    rows, cols = int(rng.integers(40, 300)), int(rng.integers(40, 300))
    pitch = (cols + 7) // 8 * 8 + 8 * int(rng.integers(0, 3))
    if rng.random() < 0.5:
        cs = 1.0 / 3600.0
        gt = [-100.0, cs, 0.0, 40.0, 0.0, -cs]
    else:
        cs = float(rng.choice([0.5, 1.0, 2.0]))
        gt = [0.0, cs, 0.0, rows * cs, 0.0, -cs]
    if rng.random() < 0.3:  # mirrored x
        gt[0], gt[1] = gt[0] + cols * gt[1], -gt[1]
    if rng.random() < 0.3:  # mirrored y
        gt[3], gt[5] = gt[3] + rows * gt[5], -gt[5]
    tile = int(rng.choice([1, 3, 8, 16, 17, 32, 64, 100, 128, 256]))
    spec = DemSpec(seed=int(rng.integers(1, 1000)), base=-150, macro_amp=900, fine_amp=200,
                   void_thresh=int(rng.choice([12500, 30000])))
    lo = int(rng.integers(-200, 100))
    width = int(rng.choice([1, 1, 2, 7]))
    nbins = int(rng.integers(1, 600))
    drop = bool(rng.random() < 0.3)
    nodata = [None, -32768, int(rng.integers(-200, 300))][int(rng.integers(0, 3))]
    out_u64 = bool(rng.random() < 0.7)
    X = lambda c: gt[0] + c * gt[1]
    Y = lambda r: gt[3] + r * gt[5]
    polys = []
    for _ in range(int(rng.integers(1, 9))):
        kind = rng.random()
        if kind < 0.6:  # jagged star
            cr, cc = rng.uniform(0, rows), rng.uniform(0, cols)
            n = int(rng.integers(3, 60))
            th = np.sort(rng.uniform(0, 2 * np.pi, n))
            rad = rng.uniform(2, max(rows, cols) / 2, n)
            rr, ccs = cr + rad * np.sin(th), cc + rad * np.cos(th)
            if rng.random() < 0.3:  # some vertices exactly on centres
                rr, ccs = np.floor(rr) + 0.5, np.floor(ccs) + 0.5
            ring = (X(ccs), Y(rr))
            rings = [ring]
            if rng.random() < 0.3:  # a hole
                rings.append((X(cc + 0.3 * (ccs - cc)), Y(cr + 0.3 * (rr - cr))))
            polys.append(rings)
        elif kind < 0.85:  # box with corners on grid lines or centres
            r0, c0 = rng.integers(-5, rows), rng.integers(-5, cols)
            h, w = rng.integers(1, rows), rng.integers(1, cols)
            off = float(rng.choice([0.0, 0.5]))
            xs = X(np.array([c0, c0 + w, c0 + w, c0]) + off)
            ys = Y(np.array([r0, r0, r0 + h, r0 + h]) + off)
            polys.append([(xs, ys)])
        else:  # degenerate
            polys.append([(X(np.array([1.0, 5.0])), Y(np.array([1.0, 5.0])))])
    P = from_rings(polys)
    R = fill_host(spec, cols, 0, 0, rows, cols)
    H = oracle.o0(R, gt, P, oracle.make_bins(nbins, lo=lo, width=width, nodata=nodata, oor_drop=drop))
    t = device_raster(spec, rows, cols, pitch=pitch)
    kw = dict(lo=lo, width=width, nodata=nodata, oor_drop=drop, out_u64=out_u64)
    G = gpu_hist(t, gt, P, nbins, tile, cols, **kw)
    assert (G.astype(np.uint64) == H).all(), (seed, tile, lo, width, nbins, drop, nodata)
    with zh.ZonalHistogram(t, gt, P, nbins, tile=tile, cols=cols, **kw) as z:
        for _ in range(3):
            z.zh_step_graph()
        got = z.output_device().cpu().numpy()
    got = got.view(np.uint64) if out_u64 else got.view(np.uint32)
    assert (got.astype(np.uint64) == H).all(), seed


def test_large_polygon_set_validated_on_device(cuda_device):
    """>= 2^20 vertices: zh_create scans them on the device behind their H2D (ZH_DEVICE_SCAN) — a
    NaN or infinite vertex is rejected with its index, coordinates too large for the cell size are
    UNSUPPORTED, and a clean set of that size equals the oracle."""
    zh = _zh()
    n = (1 << 20) + 7
    th = np.linspace(0.0, 2.0 * np.pi, n, endpoint=False)
    x, y = 32.0 + 20.5 * np.cos(th), 32.0 + 20.5 * np.sin(th)
    gt = (0.0, 1.0, 0.0, 64.0, 0.0, -1.0)
    spec = DemSpec(seed=3)
    t = device_raster(spec, 64, 64)
    bins = oracle.make_bins(256, nodata=-32768)
    P = from_rings([[(x, y)]])
    G = gpu_hist(t, gt, P, 256, 16, 64, nodata=-32768)
    R = fill_host(spec, 64, 0, 0, 64, 64)
    assert (G == oracle.o1(R, gt, P, bins)).all()
    for bad, code in ((np.nan, zh.ZH_ERR_INVALID_ARG), (np.inf, zh.ZH_ERR_INVALID_ARG)):
        xb = x.copy()
        xb[777777] = bad
        with pytest.raises(zh.ZhError) as ei:
            zh.ZonalHistogram(t, gt, from_rings([[(xb, y)]]), 256, tile=16, cols=64, nodata=-32768)
        assert ei.value.status == code and "777777" in str(ei.value)
    # cell size 1 against |coordinate| ~ 2^31: the rounding of the coordinates is no longer far
    # below a cell (zh_create's 2^-30 condition)
    with pytest.raises(zh.ZhError) as ei:
        zh.ZonalHistogram(t, gt, from_rings([[(x + 2.0 ** 31, y)]]), 256, tile=16, cols=64, nodata=-32768)
    assert ei.value.status == zh.ZH_ERR_UNSUPPORTED
