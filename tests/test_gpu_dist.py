"""The multi-GPU path on one GPU: world_size 2 processes (torch.distributed, gloo over the same
cuda:0 — there is one GPU in this environment), each holding a tile-row strip of the tiny and
state rasters in HBM, running libzh on its strip (both paths), and all-reducing the int64 view of
the uint64 histograms.  The reduced result must equal the oracle bit for bit — also through the
sparse reduce (dist.SparseReducer, on host copies: gloo has no CUDA point-to-point), whose plan
comes from the touched polygons of libzh's step-2 pairs (every non-zero row must be touched)."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cfg_name, q):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangw14_b200 import zh
    from paper_conf_ipps_zhangw14_b200.dist import SparseReducer, reduce_histograms, shard_rows, touched_polygons
    from synth.configs import CONFIGS
    from synth.dem import fill_device
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cfg = CONFIGS[cfg_name]
        P = cfg.polygons()
        r0, r1 = shard_rows(cfg.rows, cfg.tile, world, rank)
        pitch = (cfg.cols + 7) // 8 * 8
        t = torch.empty((max(r1 - r0, 1), pitch), dtype=torch.int16, device="cuda")
        fill_device(cfg.dem, cfg.cols, t.data_ptr(), r0, 0, r1 - r0, cfg.cols, pitch,
                    torch.cuda.current_stream().cuda_stream)
        res = []
        for fused in (False, True):
            out = torch.zeros((P.n_poly, cfg.nbins), dtype=torch.int64, device="cuda")
            with zh.ZonalHistogram(t[:r1 - r0], cfg.gt, P, cfg.nbins, tile=cfg.tile, rows=cfg.rows, cols=cfg.cols,
                                   row0=r0, nodata=cfg.nodata, fused=fused) as z:
                z.set_output(out)
                z.zh_run(None)
                touched = touched_polygons(z)
            part = out.cpu()
            nz = np.nonzero(part.numpy().any(axis=1))[0]
            assert np.isin(nz, touched).all()
            reduce_histograms(out, to_rank0=fused)  # four-step: all-reduce; fused: reduce to rank 0 (bench.py)
            res.append(out.cpu().numpy().view(np.uint64).copy())
        part_dev = part.cuda()
        SparseReducer(touched, P.n_poly).reduce(part, to_rank0=True)
        res.append(part.numpy().view(np.uint64).copy())
        # the same on the device tensor (what bench.py does; gloo stages the point-to-point rows)
        SparseReducer(touched, P.n_poly, device=part_dev.device).reduce(part_dev, to_rank0=True)
        res.append(part_dev.cpu().numpy().view(np.uint64).copy())
        q.put((rank, res[0], res[1], res[2], res[3]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("cfg_name", ["tiny", "state"])
def test_two_ranks_reduce_to_oracle(cuda_device, cfg_name):
    import torch.multiprocessing as mp

    import oracle
    from synth.configs import CONFIGS
    from synth.dem import fill_host
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg_name, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    cfg = CONFIGS[cfg_name]
    P = cfg.polygons()
    bins = oracle.make_bins(cfg.nbins, nodata=cfg.nodata)
    if cfg_name == "tiny":
        R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
        want = oracle.o1(R, cfg.gt, P, bins)
        rows = range(P.n_poly)
    else:  # state: sampled polygons, each from its own raster window
        rows = [0, P.n_poly // 2, P.n_poly - 1]
        want = np.zeros((P.n_poly, cfg.nbins), np.uint64)
        for k in rows:
            r0, r1, c0, c1 = oracle.polygon_window(P, k, cfg.gt, cfg.rows, cfg.cols)
            win = fill_host(cfg.dem, cfg.cols, r0, c0, r1 - r0, c1 - c0)
            want[k] = oracle.o1(win, cfg.gt, P.subset([k]), bins, row0=r0, col0=c0)[0]
    for rank, four, fused, sparse, sparse_dev in got:
        for k in rows:
            assert (four[k] == want[k]).all(), (rank, k)
            if rank == 0:
                assert (fused[k] == want[k]).all(), (rank, k)
                assert (sparse[k] == want[k]).all(), (rank, k)
        if rank == 0:
            assert (sparse == fused).all()
            assert (sparse_dev == fused).all()


def test_plan_rows_balanced_shards(cuda_device):
    """zh_plan_rows gives contiguous whole-tile-row shards; the shards of the tiny
    config sum to the oracle's whole-raster histograms; on CONUS the estimated costs are balanced."""
    import torch

    from paper_conf_ipps_zhangw14_b200 import zh
    from paper_conf_ipps_zhangw14_b200.dist import plan_shards
    from synth.configs import CONUS, TINY
    from synth.dem import fill_device
    cfg = TINY
    P = cfg.polygons()
    pitch = cfg.cols
    full = torch.empty((cfg.rows, pitch), dtype=torch.int16, device="cuda")
    fill_device(cfg.dem, cfg.cols, full.data_ptr(), 0, 0, cfg.rows, cfg.cols, pitch,
                torch.cuda.current_stream().cuda_stream)
    with zh.ZonalHistogram(full, cfg.gt, P, cfg.nbins, tile=64, nodata=cfg.nodata) as z:
        want = z.run()
    import oracle
    from synth.dem import fill_host
    R = fill_host(cfg.dem, cfg.cols, 0, 0, cfg.rows, cfg.cols)
    H = oracle.o1(R, cfg.gt, P, oracle.make_bins(cfg.nbins, nodata=cfg.nodata))
    assert (want == H).all()
    for n in (2, 3, 5):
        b = plan_shards(cfg.rows, cfg.cols, cfg.gt, P, 64, n)
        assert b[0] == 0 and b[-1] == cfg.rows and all(x <= y for x, y in zip(b, b[1:]))
        assert all(x % 64 == 0 for x in b[:-1])
        acc = np.zeros_like(want)
        for s in range(n):
            if b[s + 1] == b[s]:
                continue
            with zh.ZonalHistogram(full[b[s]:b[s + 1]], cfg.gt, P, cfg.nbins, tile=64, rows=cfg.rows, row0=b[s],
                                   nodata=cfg.nodata) as z:
                acc += z.run()
        assert (acc == H).all()  # the balanced shards sum to the oracle, not only to libzh
    C = CONUS
    PC = C.polygons()
    bounds, cost = zh.plan_rows(C.rows, C.cols, C.gt, PC, 8, tile=C.tile)
    assert bounds[0] == 0 and bounds[-1] == C.rows
    assert cost.max() / cost.mean() < 1.15, cost


def _nccl_worker(rank, world, port, cfg_name, q):
    """One GPU per rank, NCCL: each rank pairs only its strip's polygons (dist.strip_polygons) on a
    work-balanced strip, then the partial histograms are combined by the dense NCCL reduce and by
    the sparse reducer (NCCL reduce of the shared rows + batched point-to-point of the owned rows)."""
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangw14_b200 import zh
    from paper_conf_ipps_zhangw14_b200.dist import (SparseReducer, plan_shards, reduce_histograms, strip_polygons,
                                                    touched_polygons)
    from synth.configs import CONFIGS
    from synth.dem import fill_device
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    try:
        cfg = CONFIGS[cfg_name]
        P = cfg.polygons()
        b = plan_shards(cfg.rows, cfg.cols, cfg.gt, P, cfg.tile, world)
        r0, r1 = b[rank], b[rank + 1]
        ids = strip_polygons(P, cfg.gt, r0, r1)
        pitch = (cfg.cols + 7) // 8 * 8
        t = torch.empty((max(r1 - r0, 1), pitch), dtype=torch.int16, device="cuda")
        fill_device(cfg.dem, cfg.cols, t.data_ptr(), r0, 0, r1 - r0, cfg.cols, pitch,
                    torch.cuda.current_stream().cuda_stream)
        out = torch.zeros((P.n_poly, cfg.nbins), dtype=torch.int64, device="cuda")
        sub = torch.zeros((max(len(ids), 1), cfg.nbins), dtype=torch.int64, device="cuda")
        idx = torch.as_tensor(ids, device="cuda")
        with zh.ZonalHistogram(t[:r1 - r0], cfg.gt, P.subset(ids), cfg.nbins, tile=cfg.tile, rows=cfg.rows,
                               cols=cfg.cols, row0=r0, nodata=cfg.nodata) as z:
            z.set_output(sub[:len(ids)])
            z.zh_run(None)
            touched = ids[touched_polygons(z)]
        out.index_copy_(0, idx, sub[:len(ids)])
        dense = out.clone()
        reduce_histograms(dense, to_rank0=True)
        SparseReducer(touched, P.n_poly, device=out.device).reduce(out, to_rank0=True)
        q.put((rank, dense.cpu().numpy().view(np.uint64).copy(), out.cpu().numpy().view(np.uint64).copy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("cfg_name", ["tiny", "state"])
def test_nccl_two_gpus_equal_oracle(cuda_device, cfg_name):
    """PAPER.md:24 §IV.C's master combine on >= 2 B200s over NCCL (skipped on a one-GPU box): dense
    reduce and sparse reduce (shared rows reduced, owned rows point-to-point) of strips that pair
    only their own polygons == the oracle over the whole raster."""
    import torch
    import torch.multiprocessing as mp

    import oracle
    from synth.configs import CONFIGS
    from synth.dem import fill_host
    if torch.cuda.device_count() < 2:
        pytest.skip("needs >= 2 GPUs (NCCL over NVLink)")
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_nccl_worker, args=(r, world, port, cfg_name, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = dict((r, (d, s)) for r, d, s in (q.get(timeout=900) for _ in range(world)))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    cfg = CONFIGS[cfg_name]
    P = cfg.polygons()
    bins = oracle.make_bins(cfg.nbins, nodata=cfg.nodata)
    want = np.zeros((P.n_poly, cfg.nbins), np.uint64)
    for r0 in range(0, cfg.rows, 4096):
        n = min(4096, cfg.rows - r0)
        oracle.o1(fill_host(cfg.dem, cfg.cols, r0, 0, n, cfg.cols), cfg.gt, P, bins, row0=r0, out=want)
    dense, sparse = got[0]
    assert (dense == want).all()
    assert (sparse == want).all()
