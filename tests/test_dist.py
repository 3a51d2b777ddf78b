"""Multi-GPU host logic on CPU: tile-row sharding and the histogram reduction (gloo, world 2).

The per-rank compute here is the oracle on the rank's strip (the GPU shard path is covered by
tests/test_gpu_parity.py::test_tile_row_shards_sum_to_whole); what is tested is that the strips
partition the raster into whole tile rows and that the all-reduce of the partial histograms
(int64 view of uint64 counts) reproduces the single-process result bit for bit.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_zhangw14_b200.dist import reduce_histograms, shard_rows


@pytest.mark.parametrize("rows,tile,world", [(1024, 128, 2), (1000, 96, 3), (93600, 256, 8), (5, 7, 4),
                                             (0, 16, 2), (256, 256, 8)])
def test_shard_rows_partition_whole_tile_rows(rows, tile, world):
    spans = [shard_rows(rows, tile, world, r) for r in range(world)]
    assert spans[0][0] == 0 and spans[-1][1] == rows
    for (a0, a1), (b0, b1) in zip(spans, spans[1:]):
        assert a1 == b0
    for r0, r1 in spans:
        assert r0 <= r1 and r0 % tile == 0 or r0 == rows


def test_shard_rows_rejects_bad_args():
    with pytest.raises(ValueError):
        shard_rows(10, 0, 2, 0)
    with pytest.raises(ValueError):
        shard_rows(10, 4, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from synth.configs import TINY as cfg
        from synth.dem import fill_host
        P = cfg.polygons()
        r0, r1 = shard_rows(cfg.rows, cfg.tile, world, rank)
        R = fill_host(cfg.dem, cfg.cols, r0, 0, r1 - r0, cfg.cols, nthreads=2)
        H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata), row0=r0, nthreads=2)
        t = torch.from_numpy(H.view(np.int64).copy())
        t0 = t.clone()
        reduce_histograms(t)                  # all-reduce: every rank holds the sum
        reduce_histograms(t0, to_rank0=True)  # reduce: rank 0 holds the sum (what bench.py uses)
        q.put((rank, (t.numpy().view(np.uint64).copy(), t0.numpy().view(np.uint64).copy())))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_reduce_equals_single_process():
    import oracle
    from synth.configs import TINY as cfg
    from synth.dem import fill_host
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    for r in range(world):
        assert (res[r][0] == H).all()
    assert (res[0][1] == H).all()


def test_sparse_plan_host_logic():
    from paper_conf_ipps_zhangw14_b200.dist import sparse_plan
    t = np.array([[1, 1, 0, 0, 1],
                  [0, 1, 1, 0, 0],
                  [0, 1, 0, 0, 1]], bool)
    shared, owned = sparse_plan(t)
    assert shared.tolist() == [1, 4]
    assert [o.tolist() for o in owned] == [[0], [2], []]
    # every touched polygon is either shared or owned by exactly one rank; untouched ones by none
    cover = np.zeros(5, int)
    cover[shared] += 1
    for o in owned:
        cover[o] += 1
    assert cover.tolist() == [1, 1, 1, 0, 1]


def _sparse_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ipps_zhangw14_b200.dist import SparseReducer
        from synth.configs import TINY as cfg
        from synth.dem import fill_host
        P = cfg.polygons()
        r0, r1 = shard_rows(cfg.rows, cfg.tile, world, rank)
        R = fill_host(cfg.dem, cfg.cols, r0, 0, r1 - r0, cfg.cols, nthreads=2)
        H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata), row0=r0, nthreads=2)
        # touched = the rows that can be non-zero, plus a few spurious ones (any superset is valid)
        extra = np.random.default_rng(rank).integers(0, P.n_poly, 2)
        touched = np.union1d(np.nonzero(H.any(axis=1))[0], extra)
        red = SparseReducer(touched, P.n_poly)
        t = torch.from_numpy(H.view(np.int64).copy())
        t0 = t.clone()
        red.reduce(t)                   # all-reduce form
        red.reduce(t0, to_rank0=True)   # reduce form
        red.reduce(torch.from_numpy(H.view(np.int64).copy()), to_rank0=True)  # reusable plan
        q.put((rank, (t.numpy().view(np.uint64).copy(), t0.numpy().view(np.uint64).copy(),
                      len(red.shared), red.rows_moved())))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_sparse_reduce_equals_single_process(world):
    import oracle
    from synth.configs import TINY as cfg
    from synth.dem import fill_host
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sparse_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    P = cfg.polygons()
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    for r in range(world):
        assert (res[r][0] == H).all()
    assert (res[0][1] == H).all()
    n_shared = res[0][2]
    assert 0 < n_shared < P.n_poly  # some polygons span the strip borders, not all
    assert res[0][3] < world * P.n_poly  # fewer rows on the fabric than the dense reduce


@pytest.mark.parametrize("world", [2, 3, 8])
def test_strip_polygons_cover_every_nonzero_row(world):
    """dist.strip_polygons: a rank that pairs only the polygons whose bounding box meets its strip
    loses nothing — on every strip of the tiny and lon/lat configs the oracle's histograms of the
    other polygons are all zero, and the strips' results summed equal the whole raster's."""
    import oracle
    from paper_conf_ipps_zhangw14_b200.dist import strip_polygons
    from synth.configs import TINY, TINY_LONLAT
    from synth.dem import fill_host
    for cfg in (TINY, TINY_LONLAT):
        P = cfg.polygons()
        bins = oracle.make_bins(cfg.nbins, nodata=cfg.nodata)
        R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
        whole = oracle.o1(R, cfg.gt, P, bins)
        acc = np.zeros_like(whole)
        for r in range(world):
            r0, r1 = shard_rows(cfg.rows, 64, world, r)
            ids = strip_polygons(P, cfg.gt, r0, r1)
            H = oracle.o1(R[r0:r1], cfg.gt, P, bins, row0=r0)
            others = np.setdiff1d(np.arange(P.n_poly), ids)
            assert not H[others].any()
            if r1 > r0:
                Hs = oracle.o1(R[r0:r1], cfg.gt, P.subset(ids), bins, row0=r0)
                assert (Hs == H[ids]).all()
            acc += H
        assert (acc == whole).all()
        assert len(strip_polygons(P, cfg.gt, 0, cfg.rows)) == P.n_poly
        assert len(strip_polygons(P, cfg.gt, 5, 5)) == 0
