"""Multi-GPU decomposition: tile-row shards + one reduction of the per-polygon histograms.

The paper splits its rasters into 36 sub-rasters over 1-16 MPI nodes and lets a master sum the
per-polygon histograms (§IV.A, §IV.C; wall time = max over nodes).
Here one process per GPU holds a strip of WHOLE tile rows (so no tile straddles two ranks and
steps 1-4 run unchanged per rank), polygons are replicated, and the [n_poly, nbins] partial
histograms are combined with one NCCL all-reduce (or reduce to rank 0) through torch.distributed
over NVLink/NVSwitch.  Integer sums are exact and associative, so the result is bit-identical
for any number of GPUs (tests/test_dist.py).
"""
from __future__ import annotations


def shard_rows(rows: int, tile: int, world: int, rank: int) -> tuple[int, int]:
    """Rows [r0, r1) of rank `rank`: ceil(tile_rows / world) whole tile rows per rank, the last
    ranks possibly short or empty.  r0 is always a multiple of `tile`."""
    if rows < 0 or tile < 1 or world < 1 or not (0 <= rank < world):
        raise ValueError("bad shard arguments")
    tile_rows = -(-rows // tile)
    per = -(-tile_rows // world)
    r0 = min(rows, rank * per * tile)
    r1 = min(rows, (rank + 1) * per * tile)
    return r0, r1


def plan_shards(rows: int, cols: int, gt, polygons, tile: int, world: int, balanced: bool = True):
    """Row bounds (world + 1) of the decomposition: equal whole-tile-row strips, or — balanced —
    strips of about equal estimated work from step 2's pairs over the whole raster (zh_plan_rows,
    SURVEY.md §8f-2; §IV.C notes that equal partitions leave nodes near the coast
    with little step-4 work).  Every rank computes the same plan (deterministic)."""
    if not balanced or world == 1:
        return [shard_rows(rows, tile, world, r)[0] for r in range(world)] + [rows]
    from . import zh
    bounds, _ = zh.plan_rows(rows, cols, gt, polygons, world, tile=tile)
    return [int(b) for b in bounds]


def reduce_histograms(out, group=None, to_rank0: bool = False):
    """Sum the per-rank partial histograms in place.  `out` is the int64 (uint64 bits) or int32
    view of libzh's output; two's-complement sums are bit-identical to unsigned ones."""
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return out
    if to_rank0:
        dist.reduce(out, dst=0, op=dist.ReduceOp.SUM, group=group)
    else:
        dist.all_reduce(out, op=dist.ReduceOp.SUM, group=group)
    return out
