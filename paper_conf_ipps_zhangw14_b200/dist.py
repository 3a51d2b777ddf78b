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


def strip_polygons(polygons, gt, r0: int, r1: int, margin: int = 2):
    """Ids of the polygons whose vertex bounding box comes within `margin` rows of the strip's rows
    [r0, r1): every other polygon has no cell centre in the strip (a centre inside a polygon lies
    inside its bounding box), so its partial histogram on this strip is zero and the rank need not
    pair it at all (step 2 over the strip's polygons only).  Host-side geometry,
    computed once per decomposition."""
    import numpy as np
    P = polygons
    if r1 <= r0 or P.n_poly == 0:
        return np.zeros(0, dtype=np.int64)
    first = P.ring_vert_off[P.poly_ring_off[:-1]]
    last = P.ring_vert_off[P.poly_ring_off[1:]]
    v = (np.asarray(P.y, dtype=np.float64) - gt[3]) / gt[5]  # fractional row coordinate
    nonempty = np.nonzero(last > first)[0]
    if nonempty.size == 0:
        return np.zeros(0, dtype=np.int64)
    lo = np.minimum.reduceat(v, first[nonempty])
    hi = np.maximum.reduceat(v, first[nonempty])
    # reduceat over the first vertex of each non-empty polygon: the segments run to the next
    # non-empty polygon's first vertex, which is exactly this polygon's vertex range
    keep = (hi >= r0 - margin) & (lo <= r1 + margin)
    return nonempty[keep].astype(np.int64)


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


def sparse_plan(touched):
    """Who sends what ('a sparse reduce of only the polygons that span shards').

    touched[r, k] — rank r's partial histogram of polygon k may be non-zero (every k with a step-2
    pair in r's strip; any superset is correct).  Returns (shared, owned): `shared` = polygons
    touched by >= 2 ranks (summed with a collective over their rows only); owned[r] = polygons
    touched by rank r alone (their rows are already final on r and are only moved, not summed).
    Polygons touched by no rank stay zero everywhere.  Pure host logic, same on every rank."""
    import numpy as np
    t = np.asarray(touched, dtype=bool)
    n = t.sum(axis=0)
    shared = np.nonzero(n >= 2)[0].astype(np.int64)
    owned = [np.nonzero((n == 1) & t[r])[0].astype(np.int64) for r in range(t.shape[0])]
    return shared, owned


def touched_polygons(z) -> "np.ndarray":
    """Polygons with a step-2 pair (inside or intersecting) in the strip of context `z` (after
    zh_pair_tiles): the only rows of its partial histogram that can be non-zero."""
    import numpy as np
    ins, isx = z.pairs_host()
    return np.unique(np.concatenate([ins[:, 1], isx[:, 1]])).astype(np.int64)


class SparseReducer:
    """Sum per-rank partial histograms moving only rows that can be non-zero.

    The plan is geometry only (built once per decomposition from each rank's touched polygons and
    one all-gather of P-byte masks).  Per call: the rows of polygons that span strips are packed
    and reduced (to rank 0) or all-reduced; the rows of single-strip polygons are final on their
    rank and are sent to rank 0 (point-to-point), or all-gathered for the all-reduce form.  With
    tile-row strips only the polygons crossing a strip border are summed, and every other row
    crosses the fabric at most once (the dense NCCL reduce moves all n_poly rows through every
    link).  Integer sums: bit-identical to `reduce_histograms` (tests/test_dist.py)."""

    def __init__(self, touched, n_poly: int, group=None, device=None):
        import numpy as np
        import torch
        import torch.distributed as dist
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        mask = torch.zeros(n_poly, dtype=torch.uint8)
        mask[torch.as_tensor(np.asarray(touched, dtype=np.int64))] = 1
        if device is not None and dist.get_backend(group) != "gloo":
            mask = mask.to(device)
        masks = [torch.empty_like(mask) for _ in range(self.world)]
        dist.all_gather(masks, mask, group=group)
        self.shared, self.owned = sparse_plan(torch.stack(masks).cpu().numpy())
        dev = torch.device(device) if device is not None else mask.device
        self._shared = torch.as_tensor(self.shared, device=dev)
        self._owned = [torch.as_tensor(o, device=dev) for o in self.owned]
        self.max_owned = max(len(o) for o in self.owned)

    def rows_moved(self) -> int:
        """Rows each call puts on the fabric (reduce form): shared rows once per rank + owned rows
        of ranks != 0."""
        return len(self.shared) * self.world + sum(len(o) for o in self.owned[1:])

    def reduce(self, out, to_rank0: bool = False):
        import torch
        import torch.distributed as dist
        if self.world == 1:
            return out
        g = self.group
        if len(self.shared):
            buf = out.index_select(0, self._shared)
            if to_rank0:
                dist.reduce(buf, dst=dist.get_global_rank(g, 0) if g is not None else 0, group=g)
            else:
                dist.all_reduce(buf, group=g)
            if not to_rank0 or self.rank == 0:
                out.index_copy_(0, self._shared, buf)
        # gloo has no CUDA point-to-point / all-gather-into-tensor: stage those rows through host
        # memory (the shared-GPU test mode); NCCL moves them device to device
        dev = torch.device("cpu") if out.is_cuda and dist.get_backend(g) == "gloo" else out.device
        if to_rank0:
            ops, bufs = [], []
            glob = (lambda r: dist.get_global_rank(g, r)) if g is not None else (lambda r: r)
            if self.rank == 0:
                for r in range(1, self.world):
                    if len(self.owned[r]):
                        b = torch.empty((len(self.owned[r]), out.shape[1]), dtype=out.dtype, device=dev)
                        bufs.append((r, b))
                        ops.append(dist.P2POp(dist.irecv, b, glob(r), g))
            elif len(self.owned[self.rank]):
                b = out.index_select(0, self._owned[self.rank]).to(dev)
                bufs.append((self.rank, b))
                ops.append(dist.P2POp(dist.isend, b, glob(0), g))
            if ops:
                for w in dist.batch_isend_irecv(ops):
                    w.wait()
            if self.rank == 0:
                for r, b in bufs:
                    out.index_copy_(0, self._owned[r], b.to(out.device))
        elif self.max_owned:
            mine = self._owned[self.rank]
            send = torch.zeros((self.max_owned, out.shape[1]), dtype=out.dtype, device=dev)
            if len(mine):
                send[:len(mine)] = out.index_select(0, mine).to(dev)
            recv = torch.empty((self.world * self.max_owned, out.shape[1]), dtype=out.dtype, device=dev)
            dist.all_gather_into_tensor(recv, send, group=g)
            for r in range(self.world):
                if r != self.rank and len(self.owned[r]):
                    rows = recv[r * self.max_owned:r * self.max_owned + len(self.owned[r])]
                    out.index_copy_(0, self._owned[r], rows.to(out.device))
        return out
