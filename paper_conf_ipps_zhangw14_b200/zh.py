"""Thin ctypes binding of libzh (include/zh.h) — argument marshalling only.

Every step of the zonal-histogramming path runs in libzh's sm_100a kernels; this module only
converts torch tensors / numpy arrays into the C structs and pointers.  There is no CPU
fallback: if libzh.so is missing or fails to load, importing the binding raises.

Function names follow the C ABI (zh_create, zh_tile_hist, zh_pair_tiles, zh_aggregate,
zh_pip_update, zh_run, ...); `ZonalHistogram` bundles them for convenience.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

# ZH_LIBZH: load another build of libzh (A/B experiments); default is the in-tree build.
_LIB_PATH = os.environ.get("ZH_LIBZH", _build.LIB)

ZH_DIST_L1, ZH_DIST_EMD, ZH_DIST_CHI2 = 0, 1, 2
_DIST_KINDS = {"l1": ZH_DIST_L1, "emd": ZH_DIST_EMD, "chi2": ZH_DIST_CHI2}
SUMMARY_FIELDS = ("count", "min", "max", "median", "mean", "std")

ZH_OK, ZH_ERR_INVALID_ARG, ZH_ERR_UNSUPPORTED, ZH_ERR_OOM, ZH_ERR_CUDA, ZH_ERR_OVERFLOW, ZH_ERR_STATE = range(7)
_STATUS = {0: "ZH_OK", 1: "ZH_ERR_INVALID_ARG", 2: "ZH_ERR_UNSUPPORTED", 3: "ZH_ERR_OOM", 4: "ZH_ERR_CUDA",
           5: "ZH_ERR_OVERFLOW", 6: "ZH_ERR_STATE"}


class ZhError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class zh_raster(ctypes.Structure):
    _fields_ = [("data", ctypes.c_void_p), ("rows", ctypes.c_int64), ("cols", ctypes.c_int64),
                ("pitch", ctypes.c_int64), ("row0", ctypes.c_int64), ("nrows", ctypes.c_int64),
                ("gt", ctypes.c_double * 6), ("on_host", ctypes.c_int32), ("reserved", ctypes.c_int32)]


class zh_polygons(ctypes.Structure):
    _fields_ = [("n_poly", ctypes.c_int64), ("n_ring", ctypes.c_int64), ("n_vert", ctypes.c_int64),
                ("poly_ring_off", ctypes.c_void_p), ("ring_vert_off", ctypes.c_void_p),
                ("x", ctypes.c_void_p), ("y", ctypes.c_void_p)]


class zh_bins(ctypes.Structure):
    _fields_ = [("lo", ctypes.c_int32), ("width", ctypes.c_int32), ("nbins", ctypes.c_int32),
                ("use_nodata", ctypes.c_int32), ("nodata", ctypes.c_int32), ("oor_drop", ctypes.c_int32)]


class zh_options(ctypes.Structure):
    _fields_ = [("tile", ctypes.c_int32), ("out_u64", ctypes.c_int32), ("force_isect", ctypes.c_int32),
                ("fused", ctypes.c_int32), ("stream", ctypes.c_void_p), ("rep_custom", ctypes.c_int32),
                ("cover", ctypes.c_int32), ("rep_x", ctypes.c_double), ("rep_y", ctypes.c_double)]


class zh_stats(ctypes.Structure):
    _fields_ = [("n_tiles", ctypes.c_int64), ("n_candidates", ctypes.c_int64), ("n_inside", ctypes.c_int64),
                ("n_isect", ctypes.c_int64), ("n_band_entries", ctypes.c_int64), ("n_edges", ctypes.c_int64),
                ("device_bytes", ctypes.c_int64), ("n_pure_tiles", ctypes.c_int64), ("n_pip_pairs", ctypes.c_int64),
                ("n_pure_cells", ctypes.c_int64), ("n_pip_cells", ctypes.c_int64), ("h2d_bytes", ctypes.c_int64),
                ("n_mixed_groups", ctypes.c_int64), ("n_group_cells", ctypes.c_int64),
                ("n_mixed_cells", ctypes.c_int64)]


EXPORTS = ["zh_create", "zh_upload_raster", "zh_tile_hist", "zh_pair_tiles", "zh_aggregate", "zh_pip_update",
           "zh_fused_update", "zh_zonal_stats", "zh_zonal_summary", "zh_hist_distance", "zh_plan_rows",
           "zh_run", "zh_step_graph", "zh_output_device", "zh_set_output", "zh_copy_tile_hist", "zh_copy_pairs", "zh_get_stats",
           "zh_set_timing", "zh_get_step_ms", "zh_launch_count", "zh_last_error", "zh_abi_version", "zh_destroy",
           "zh_trim_cache", "zh_cache_bytes"]


def _load():
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"libzh.so not built at {_LIB_PATH}: run `python -c 'import __graft_entry__ as g; "
                          f"g.build()'` (nvcc, sm_100a).  There is no CPU fallback.")
    lib = ctypes.CDLL(_LIB_PATH)
    vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
    st = ctypes.c_int
    sig = {
        "zh_create": (st, [ctypes.POINTER(vp), ctypes.POINTER(zh_raster), ctypes.POINTER(zh_polygons),
                           ctypes.POINTER(zh_bins), ctypes.POINTER(zh_options)]),
        "zh_upload_raster": (st, [vp]),
        "zh_tile_hist": (st, [vp]),
        "zh_pair_tiles": (st, [vp, ctypes.POINTER(i64), ctypes.POINTER(i64)]),
        "zh_aggregate": (st, [vp]),
        "zh_pip_update": (st, [vp]),
        "zh_fused_update": (st, [vp]),
        "zh_zonal_stats": (st, [vp, vp, vp]),
        "zh_zonal_summary": (st, [vp, vp, vp]),
        "zh_hist_distance": (st, [vp, i32, vp, vp, i64, vp]),
        "zh_plan_rows": (st, [ctypes.POINTER(zh_raster), ctypes.POINTER(zh_polygons), ctypes.POINTER(zh_options), i32,
                              vp, vp]),
        "zh_run": (st, [vp, vp]),
        "zh_step_graph": (st, [vp]),
        "zh_output_device": (st, [vp, ctypes.POINTER(vp), ctypes.POINTER(i64)]),
        "zh_set_output": (st, [vp, vp]),
        "zh_copy_tile_hist": (st, [vp, vp, i64]),
        "zh_copy_pairs": (st, [vp, vp, vp]),
        "zh_get_stats": (st, [vp, ctypes.POINTER(zh_stats)]),
        "zh_set_timing": (st, [vp, i32]),
        "zh_get_step_ms": (st, [vp, ctypes.POINTER(ctypes.c_float), i32]),
        "zh_launch_count": (i64, [vp]),
        "zh_last_error": (ctypes.c_char_p, []),
        "zh_abi_version": (i32, []),
        "zh_destroy": (None, [vp]),
        "zh_trim_cache": (None, [i32]),
        "zh_cache_bytes": (i64, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


LIB = _load()


def _check(status: int) -> None:
    if status != ZH_OK:
        raise ZhError(status, LIB.zh_last_error().decode(errors="replace"))


def _stream_handle(stream) -> int:
    if stream is None:
        try:
            import torch
            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream
        except Exception:  # pragma: no cover
            pass
        return 0
    if hasattr(stream, "cuda_stream"):
        return stream.cuda_stream
    return int(stream)


def plan_rows(rows: int, cols: int, gt, polygons, n_shards: int, tile: int = 256, stream=None, rep=None):
    """zh_plan_rows: row bounds (n_shards + 1) of a work-balanced tile-row decomposition and the
    estimated cost per shard."""
    r = zh_raster()
    r.data = None
    r.rows, r.cols, r.pitch, r.row0, r.nrows = rows, cols, (cols + 7) // 8 * 8, 0, rows
    r.gt = (ctypes.c_double * 6)(*[float(g) for g in gt])
    r.on_host = 0
    pro = np.ascontiguousarray(polygons.poly_ring_off, dtype=np.int64)
    rvo = np.ascontiguousarray(polygons.ring_vert_off, dtype=np.int64)
    x = np.ascontiguousarray(polygons.x, dtype=np.float64)
    y = np.ascontiguousarray(polygons.y, dtype=np.float64)
    p = zh_polygons(pro.shape[0] - 1, rvo.shape[0] - 1, x.shape[0], pro.ctypes.data, rvo.ctypes.data,
                    x.ctypes.data, y.ctypes.data)
    o = zh_options(tile, 1, 0, 0, _stream_handle(stream), 0 if rep is None else 1, 0,
                   0.5 if rep is None else float(rep[0]), 0.5 if rep is None else float(rep[1]))
    bounds = np.zeros(n_shards + 1, dtype=np.int64)
    cost = np.zeros(n_shards, dtype=np.float64)
    _check(LIB.zh_plan_rows(ctypes.byref(r), ctypes.byref(p), ctypes.byref(o), n_shards, bounds.ctypes.data,
                            cost.ctypes.data))
    return bounds, cost


class _CAI:
    """__cuda_array_interface__ view of a borrowed device pointer (no copy)."""

    def __init__(self, ptr: int, shape, typestr: str, owner):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr, "data": (ptr, False),
                                         "version": 3, "strides": None}
        self._owner = owner


class ZonalHistogram:
    """One libzh context: a raster shard, a polygon set, a bin mapping and a tile size.

    raster: a CUDA int16 torch tensor [nrows, >=cols] (device, borrowed — keep it alive), or a
    host numpy/torch int16 array (on_host; pinned memory recommended).  Its first row is global
    row `row0` of a raster with `rows` rows (default: a single shard holding the whole raster).
    polygons: any object with poly_ring_off, ring_vert_off, x, y arrays (synth.polygons.Polygons).
    rep: None for cell centres, or (ox, oy) in [0, 1]^2 — the representative point (c+ox, r+oy).
    cover: count a cell in P_k when its closed rectangle meets the closed polygon (the literal
    "geometrically intersect" of PAPER.md:12; R15) instead of testing its centre.
    """

    def __init__(self, raster, gt, polygons, nbins: int, lo: int = 0, width: int = 1, nodata=None,
                 oor_drop: bool = False, tile: int = 256, out_u64: bool = True, force_isect: bool = False,
                 row0: int = 0, rows: int | None = None, cols: int | None = None, stream=None,
                 fused: bool = True, rep=None, cover: bool = False):
        self._keep = []
        on_host, ptr, nrows, ncols_buf, pitch = self._raster_ptr(raster)
        ncols = cols if cols is not None else ncols_buf
        r = zh_raster()
        r.data = ptr
        r.rows = rows if rows is not None else row0 + nrows
        r.cols = ncols
        r.pitch = pitch
        r.row0 = row0
        r.nrows = nrows
        r.gt = (ctypes.c_double * 6)(*[float(g) for g in gt])
        r.on_host = int(on_host)
        pro = np.ascontiguousarray(polygons.poly_ring_off, dtype=np.int64)
        rvo = np.ascontiguousarray(polygons.ring_vert_off, dtype=np.int64)
        x = np.ascontiguousarray(polygons.x, dtype=np.float64)
        y = np.ascontiguousarray(polygons.y, dtype=np.float64)
        p = zh_polygons(pro.shape[0] - 1, rvo.shape[0] - 1, x.shape[0], pro.ctypes.data, rvo.ctypes.data,
                        x.ctypes.data, y.ctypes.data)
        b = zh_bins(lo, width, nbins, 0 if nodata is None else 1, 0 if nodata is None else int(nodata), int(oor_drop))
        self.stream = _stream_handle(stream)
        o = zh_options(tile, int(out_u64), int(force_isect), int(fused), self.stream,
                       0 if rep is None else 1, int(cover), 0.5 if rep is None else float(rep[0]),
                       0.5 if rep is None else float(rep[1]))
        h = ctypes.c_void_p()
        _check(LIB.zh_create(ctypes.byref(h), ctypes.byref(r), ctypes.byref(p), ctypes.byref(b), ctypes.byref(o)))
        self.h = h
        self.n_poly = int(pro.shape[0] - 1)
        self.nbins = int(nbins)
        self.out_u64 = bool(out_u64)
        self.tile = int(tile)
        self._keep.append(raster)

    @staticmethod
    def _raster_ptr(raster):
        try:
            import torch
        except Exception:  # pragma: no cover
            torch = None
        if torch is not None and isinstance(raster, torch.Tensor):
            if raster.dtype != torch.int16 or raster.dim() != 2 or raster.stride(1) != 1:
                raise ValueError("raster must be a 2-D int16 tensor with unit column stride")
            return (not raster.is_cuda, raster.data_ptr(), raster.shape[0], raster.shape[1], raster.stride(0))
        a = np.asarray(raster)
        if a.dtype != np.int16 or a.ndim != 2 or a.strides[1] != 2:
            raise ValueError("raster must be a 2-D int16 array with unit column stride")
        return (True, a.ctypes.data, a.shape[0], a.shape[1], a.strides[0] // 2)

    # ---- the C ABI, one method per call
    def zh_upload_raster(self):
        _check(LIB.zh_upload_raster(self.h))

    def zh_tile_hist(self):
        _check(LIB.zh_tile_hist(self.h))

    def zh_pair_tiles(self):
        a, b = ctypes.c_int64(), ctypes.c_int64()
        _check(LIB.zh_pair_tiles(self.h, ctypes.byref(a), ctypes.byref(b)))
        return a.value, b.value

    def zh_aggregate(self):
        _check(LIB.zh_aggregate(self.h))

    def zh_pip_update(self):
        _check(LIB.zh_pip_update(self.h))

    def zh_fused_update(self):
        _check(LIB.zh_fused_update(self.h))

    def zh_run(self, host_out: np.ndarray | None = None) -> np.ndarray | None:
        if host_out is not None:
            dt = np.uint64 if self.out_u64 else np.uint32
            assert host_out.dtype == dt and host_out.size == self.n_poly * self.nbins and host_out.flags.c_contiguous
            _check(LIB.zh_run(self.h, host_out.ctypes.data))
            return host_out
        _check(LIB.zh_run(self.h, None))
        return None

    def zh_step_graph(self):
        _check(LIB.zh_step_graph(self.h))

    def run(self) -> np.ndarray:
        out = np.empty((self.n_poly, self.nbins), dtype=np.uint64 if self.out_u64 else np.uint32)
        return self.zh_run(out)

    def zh_zonal_stats(self) -> np.ndarray:
        """Raw exact statistics [n_poly, 8] int64 (see zh.h: count, min/max/median bin, sum b,
        sum b^2 low/high words, non-zero bins)."""
        out = np.zeros((self.n_poly, 8), dtype=np.int64)
        _check(LIB.zh_zonal_stats(self.h, out.ctypes.data if self.n_poly else None, None))
        return out

    def zh_zonal_summary(self) -> np.ndarray:
        """[n_poly, 6] float64: count, min, max, median, mean, std in value units, computed by libzh
        from the exact integer statistics (zh.h states the rounding of each field)."""
        out = np.zeros((self.n_poly, len(SUMMARY_FIELDS)), dtype=np.float64)
        _check(LIB.zh_zonal_summary(self.h, out.ctypes.data if self.n_poly else None, None))
        return out

    def zonal_stats(self) -> dict:
        """zh_zonal_summary as a dict of columns (value units of this context's bin mapping)."""
        out = self.zh_zonal_summary()
        return {f: out[:, i] for i, f in enumerate(SUMMARY_FIELDS)}

    def zh_hist_distance(self, kind: str = "l1", a=None, b=None) -> np.ndarray:
        """Distances between normalised polygon histograms (zh.h: l1, emd, chi2).  a, b: polygon id
        sequences (pairwise, same length) -> [n]; both None -> the all-pairs [n_poly, n_poly] matrix."""
        k = _DIST_KINDS[kind]
        if a is None and b is None:
            out = np.empty((self.n_poly, self.n_poly), dtype=np.float64)
            _check(LIB.zh_hist_distance(self.h, k, None, None, 0, out.ctypes.data))
            return out
        ia = np.ascontiguousarray(a, dtype=np.int32)
        ib = np.ascontiguousarray(b, dtype=np.int32)
        if ia.shape != ib.shape or ia.ndim != 1:
            raise ValueError("a and b must be 1-D sequences of the same length")
        out = np.empty(ia.shape[0], dtype=np.float64)
        _check(LIB.zh_hist_distance(self.h, k, ia.ctypes.data, ib.ctypes.data, ia.shape[0], out.ctypes.data))
        return out

    def output_device(self):
        """The output as a torch CUDA tensor view (int64 for u64, int32 for u32 — same bits)."""
        import torch
        p, n = ctypes.c_void_p(), ctypes.c_int64()
        _check(LIB.zh_output_device(self.h, ctypes.byref(p), ctypes.byref(n)))
        typestr = "<i8" if self.out_u64 else "<i4"
        return torch.as_tensor(_CAI(p.value or 0, (self.n_poly, self.nbins), typestr, self), device="cuda")

    def set_output(self, tensor) -> None:
        """Use a caller-owned CUDA tensor ([n_poly, nbins] int64/int32) as the output buffer."""
        if tensor is None:
            _check(LIB.zh_set_output(self.h, None))
            return
        assert tensor.is_cuda and tensor.is_contiguous() and tensor.numel() == self.n_poly * self.nbins
        assert tensor.element_size() == (8 if self.out_u64 else 4)
        self._keep.append(tensor)
        _check(LIB.zh_set_output(self.h, tensor.data_ptr()))

    def tile_hist_host(self) -> np.ndarray:
        st = self.stats()
        out = np.empty((st["n_tiles"], self.nbins), dtype=np.uint32)
        _check(LIB.zh_copy_tile_hist(self.h, out.ctypes.data, out.size))
        return out

    def pairs_host(self):
        st = self.stats()
        ins = np.empty((st["n_inside"], 2), dtype=np.int32)
        isx = np.empty((st["n_isect"], 2), dtype=np.int32)
        _check(LIB.zh_copy_pairs(self.h, ins.ctypes.data, isx.ctypes.data))
        return ins, isx

    def stats(self) -> dict:
        s = zh_stats()
        _check(LIB.zh_get_stats(self.h, ctypes.byref(s)))
        return {f: int(getattr(s, f)) for f, _ in zh_stats._fields_}

    def set_timing(self, enable: bool = True) -> None:
        _check(LIB.zh_set_timing(self.h, int(enable)))

    STEP_NAMES = ("step1_tile_hist", "step2_pair_tiles", "step3_aggregate", "step4_pip_update", "fused_update",
                  "fused_pure_kernel", "fused_pip_kernel", "fused_parity_kernel")

    def step_ms(self) -> dict:
        """Device ms of the last call of each step (-1: not called since timing was enabled)."""
        ms = (ctypes.c_float * len(self.STEP_NAMES))()
        _check(LIB.zh_get_step_ms(self.h, ms, len(self.STEP_NAMES)))
        return dict(zip(self.STEP_NAMES, list(ms)))

    def launch_count(self) -> int:
        return int(LIB.zh_launch_count(self.h))

    def close(self) -> None:
        if getattr(self, "h", None):
            LIB.zh_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
