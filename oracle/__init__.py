"""CPU oracle for zonal histogramming — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
may import this package.  The product path (paper_conf_ipps_zhangw14_b200 + libzh.so)
never imports it and shares no code with it.

The arithmetic lives in oracle/zh_oracle.c (plain C, gcc -O2 -ffp-contract=off, OpenMP
over rows); see its header for the definition it computes (§III ¶1, cell
centres PAPER.md:18 §III.D, Franklin's ray-crossing test PAPER.md:20 Fig. 5) and every
reading taken where the paper is silent (also DESIGN.md §3).

Parity status: pinned (tests/test_oracle_pins.py) — hand-worked counts, Fig. 5 crossing
counts, closed-form histograms, np.bincount, the tiling partition invariant, O0 == O1.  The cover
variant (reading R15) is pinned in tests/test_oracle_cover.py — closed forms and an exact
rational-arithmetic reference on dyadic polygons.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "zh_oracle.c")


class Bins(ctypes.Structure):
    """Bin mapping (reading R3/R4): bin = (v - lo) // width, clamp or drop, nodata skipped."""
    _fields_ = [("lo", ctypes.c_int32), ("width", ctypes.c_int32), ("nbins", ctypes.c_int32),
                ("use_nodata", ctypes.c_int32), ("nodata", ctypes.c_int32), ("oor_drop", ctypes.c_int32)]


def make_bins(nbins: int, lo: int = 0, width: int = 1, nodata: int | None = None, oor_drop: bool = False) -> Bins:
    return Bins(lo, width, nbins, 0 if nodata is None else 1, 0 if nodata is None else nodata, int(oor_drop))


def build(force: bool = False) -> str:
    """Compile the oracle (no FMA contraction: -ffp-contract=off, reading R7)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC",
                               "-shared", _SRC, "-o", _SO, "-lm"])
    return _SO


_lib = None
_I64P = ctypes.POINTER(ctypes.c_int64)


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        vp, i64, dbl = ctypes.c_void_p, ctypes.c_int64, ctypes.c_double
        lib.zho_bin.restype = ctypes.c_int
        lib.zho_bin.argtypes = [ctypes.c_int32, ctypes.POINTER(Bins)]
        lib.zho_centre.restype = None
        lib.zho_centre.argtypes = [vp, i64, i64, ctypes.POINTER(dbl), ctypes.POINTER(dbl)]
        lib.zho_crossings.restype = i64
        lib.zho_crossings.argtypes = [dbl, dbl, i64, vp, vp, vp, vp]
        lib.zho_o0.restype = None
        lib.zho_o0.argtypes = [vp, i64, i64, i64, i64, i64, vp, i64, vp, vp, vp, vp, ctypes.POINTER(Bins), vp,
                               ctypes.c_int, ctypes.c_int]
        lib.zho_o1.restype = None
        lib.zho_o1.argtypes = [vp, i64, i64, i64, i64, i64, vp, i64, vp, vp, vp, vp, ctypes.POINTER(Bins), vp,
                               ctypes.c_int]
        lib.zho_seg_touches.restype = ctypes.c_int
        lib.zho_seg_touches.argtypes = [dbl] * 8
        lib.zho_cover_o0.restype = None
        lib.zho_cover_o0.argtypes = [vp, i64, i64, i64, i64, i64, vp, i64, vp, vp, vp, vp, ctypes.POINTER(Bins), vp,
                                     ctypes.c_int, ctypes.c_int]
        lib.zho_cover_membership.restype = None
        lib.zho_cover_membership.argtypes = [vp, vp, i64, vp, i64, vp, vp, vp, vp, vp, ctypes.c_int]
        lib.zho_membership.restype = None
        lib.zho_membership.argtypes = [vp, vp, i64, vp, i64, vp, vp, vp, vp, vp, ctypes.c_int]
        _lib = lib
    return _lib


def _c64(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def _gt8(gt, rep=None):
    """gt (6 GDAL coefficients) + the representative point offsets (default: the cell centre)."""
    g = [float(v) for v in gt][:6]
    r = (0.5, 0.5) if rep is None else (float(rep[0]), float(rep[1]))
    return np.array(g + list(r), dtype=np.float64)


def _poly_args(P):
    pro = _c64(P.poly_ring_off, np.int64)
    rvo = _c64(P.ring_vert_off, np.int64)
    x = _c64(P.x, np.float64)
    y = _c64(P.y, np.float64)
    return (pro, rvo, x, y)


def _nthreads(n):
    return int(n or os.cpu_count() or 1)


def bin_of(v: int, bins: Bins) -> int:
    return int(_L().zho_bin(int(v), ctypes.byref(bins)))


def centre(gt, r: int, c: int, rep=None):
    g = _gt8(gt, rep)
    xc, yc = ctypes.c_double(), ctypes.c_double()
    _L().zho_centre(g.ctypes.data, r, c, ctypes.byref(xc), ctypes.byref(yc))
    return xc.value, yc.value


def crossings(P, k: int, xc: float, yc: float) -> int:
    pro, rvo, x, y = _poly_args(P)
    return int(_L().zho_crossings(float(xc), float(yc), int(k), pro.ctypes.data, rvo.ctypes.data,
                                  x.ctypes.data, y.ctypes.data))


def _hist(fn, win, row0, col0, gt, P, bins, nthreads, extra, rep=None, out=None):
    win = np.asarray(win)
    assert win.dtype == np.int16 and win.ndim == 2 and win.strides[1] == 2
    nrows, ncols = win.shape
    pitch = win.strides[0] // 2
    g = _gt8(gt, rep)
    pro, rvo, x, y = _poly_args(P)
    if out is None:
        out = np.zeros((P.n_poly, bins.nbins), dtype=np.uint64)
    assert out.dtype == np.uint64 and out.shape == (P.n_poly, bins.nbins) and out.flags.c_contiguous
    fn(win.ctypes.data, int(row0), int(col0), nrows, ncols, pitch, g.ctypes.data, P.n_poly,
       pro.ctypes.data, rvo.ctypes.data, x.ctypes.data, y.ctypes.data, ctypes.byref(bins), out.ctypes.data,
       *extra, _nthreads(nthreads))
    return out


def o0(win, gt, P, bins: Bins, row0: int = 0, col0: int = 0, prefilter: bool = False, nthreads=None, rep=None):
    """O0: the definition (every cell x polygon x edge).  Returns uint64 [n_poly, nbins].
    rep: representative point offsets in the cell (default (0.5, 0.5), the centre)."""
    return _hist(_L().zho_o0, win, row0, col0, gt, P, bins, nthreads, (int(prefilter),), rep)


def o1(win, gt, P, bins: Bins, row0: int = 0, col0: int = 0, nthreads=None, rep=None, out=None):
    """O1: row-hoisted intercepts, identical comparisons to O0.  Returns uint64 [n_poly, nbins]
    (accumulated into `out` when given: rows are independent, so bands of a raster can be fed
    one after another)."""
    return _hist(_L().zho_o1, win, row0, col0, gt, P, bins, nthreads, (), rep, out)


def seg_touches(x0, y0, x1, y1, X0, X1, Y0, Y1) -> bool:
    """R15: does the segment (x0,y0)-(x1,y1) meet the closed rectangle between the grid lines?"""
    return bool(_L().zho_seg_touches(*(float(v) for v in (x0, y0, x1, y1, X0, X1, Y0, Y1))))


def cover_o0(win, gt, P, bins: Bins, row0: int = 0, col0: int = 0, prefilter: bool = True, nthreads=None):
    """The "geometrically intersect" variant (reading R15): a cell counts in P_k when
    its closed rectangle meets the closed polygon.  Returns uint64 [n_poly, nbins]."""
    return _hist(_L().zho_cover_o0, win, row0, col0, gt, P, bins, nthreads, (int(prefilter),))


def cover_membership(rows, cols, gt, P, nthreads=None) -> np.ndarray:
    """covered[q, k] in {0,1} for the cells (rows[q], cols[q]) (reading R15)."""
    rows = _c64(rows, np.int64)
    cols = _c64(cols, np.int64)
    g = _gt8(gt)
    pro, rvo, x, y = _poly_args(P)
    out = np.zeros((rows.shape[0], P.n_poly), dtype=np.uint8)
    _L().zho_cover_membership(rows.ctypes.data, cols.ctypes.data, rows.shape[0], g.ctypes.data, P.n_poly,
                              pro.ctypes.data, rvo.ctypes.data, x.ctypes.data, y.ctypes.data, out.ctypes.data,
                              _nthreads(nthreads))
    return out


def membership(rows, cols, gt, P, nthreads=None, rep=None) -> np.ndarray:
    """inside[q, k] in {0,1} for the cells (rows[q], cols[q])."""
    rows = _c64(rows, np.int64)
    cols = _c64(cols, np.int64)
    g = _gt8(gt, rep)
    pro, rvo, x, y = _poly_args(P)
    out = np.zeros((rows.shape[0], P.n_poly), dtype=np.uint8)
    _L().zho_membership(rows.ctypes.data, cols.ctypes.data, rows.shape[0], g.ctypes.data, P.n_poly,
                        pro.ctypes.data, rvo.ctypes.data, x.ctypes.data, y.ctypes.data, out.ctypes.data,
                        _nthreads(nthreads))
    return out


def polygon_window(P, k: int, gt, rows: int, cols: int, margin: int = 2):
    """Row/col window [r0,r1) x [c0,c1) of the raster that can hold centres of polygon k.
    (Only chooses how much raster the caller generates; the oracle itself tests every cell given.)"""
    a, b = int(P.ring_vert_off[P.poly_ring_off[k]]), int(P.ring_vert_off[P.poly_ring_off[k + 1]])
    if a == b:
        return 0, 0, 0, 0
    xs, ys = P.x[a:b], P.y[a:b]
    cc = (np.array([xs.min(), xs.max()]) - gt[0]) / gt[1]
    rr = (np.array([ys.min(), ys.max()]) - gt[3]) / gt[5]
    c0 = max(0, int(np.floor(cc.min())) - margin)
    c1 = min(cols, int(np.ceil(cc.max())) + margin)
    r0 = max(0, int(np.floor(rr.min())) - margin)
    r1 = min(rows, int(np.ceil(rr.max())) + margin)
    return r0, max(r0, r1), c0, max(c0, c1)


def zonal_stats(H) -> np.ndarray:
    """Zonal statistics of each histogram row, the plain definition in exact Python integers
    (min/max/average/count/std of PAPER.md:10 §I ¶1), in units of bin indices:
    [count, min_bin, max_bin, lower-median bin, sum b, sum b^2 low word, sum b^2 high word,
    non-zero bins]; bins are -1 for an empty row."""
    H = np.asarray(H)
    out = np.zeros((H.shape[0], 8), dtype=np.int64)
    for k in range(H.shape[0]):
        row = [int(v) for v in H[k]]
        n = sum(row)
        nzb = [b for b, v in enumerate(row) if v]
        s1 = sum(b * v for b, v in enumerate(row))
        s2 = sum(b * b * v for b, v in enumerate(row))
        med = -1
        if n:
            target, run = (n + 1) // 2, 0
            for b, v in enumerate(row):
                run += v
                if run >= target:
                    med = b
                    break
        lo64 = s2 & ((1 << 64) - 1)
        out[k] = [n, nzb[0] if nzb else -1, nzb[-1] if nzb else -1, med, s1,
                  lo64 - (1 << 64) if lo64 >= (1 << 63) else lo64, s2 >> 64, len(nzb)]
    return out
