"""Synthetic SRTM-like DEM rasters (INPUT GENERATION ONLY — no zonal-histogram arithmetic).

Both sides of the parity tests draw their raster from here: the host evaluation
(`fill_host`, gcc build of csrc/dem_host.c) feeds the CPU oracle, the device evaluation
(`fill_device`, nvcc build of csrc/dem_dev.cu) fills the HBM raster libzh reads.  They
evaluate the same integer function of (seed, row, col) from csrc/dem_core.h, so they
agree bit for bit (tests/test_synth.py, tests/test_gpu_parity.py).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_HOST_SO = os.path.join(_HERE, "libsynth_host.so")
_DEV_SO = os.path.join(_HERE, "libsynth_cuda.so")

NODATA = -32768

KIND_DEM, KIND_COLMOD, KIND_ROWMOD, KIND_LINMOD = 0, 1, 2, 3


class _Params(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint32), ("base", ctypes.c_int32), ("macro_amp", ctypes.c_int32),
                ("fine_amp", ctypes.c_int32), ("void_thresh", ctypes.c_int32),
                ("lo_clip", ctypes.c_int32), ("hi_clip", ctypes.c_int32)]


@dataclass(frozen=True)
class DemSpec:
    """A raster recipe: kind 0 = fractal DEM, 1..3 = closed-form patterns (value = idx mod m + off)."""
    seed: int = 1
    base: int = 500
    macro_amp: int = 1400
    fine_amp: int = 300
    void_thresh: int = 11800  # > 16383 disables voids
    lo_clip: int = -400
    hi_clip: int = 8000
    kind: int = KIND_DEM
    pattern_mod: int = 256
    pattern_off: int = 0

    def _c(self) -> _Params:
        return _Params(self.seed & 0xFFFFFFFF, self.base, self.macro_amp, self.fine_amp,
                       self.void_thresh, self.lo_clip, self.hi_clip)


_host = None
_dev = None


def build(force: bool = False) -> None:
    """Compile both generator libraries in-tree (gcc for the host, nvcc for sm_100a)."""
    import subprocess
    src = os.path.join(_HERE, "csrc")
    if force or not os.path.exists(_HOST_SO):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared",
                               os.path.join(src, "dem_host.c"), "-o", _HOST_SO])
    if force or not os.path.exists(_DEV_SO):
        subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
                               "-Xcompiler", "-fPIC", "-shared", os.path.join(src, "dem_dev.cu"),
                               "-o", _DEV_SO])


def _host_lib():
    global _host
    if _host is None:
        if not os.path.exists(_HOST_SO):
            build()
        _host = ctypes.CDLL(_HOST_SO)
        _host.zhs_fill_host.restype = None
        _host.zhs_fill_host.argtypes = [ctypes.POINTER(_Params), ctypes.c_int, ctypes.c_int32, ctypes.c_int32,
                                        ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                                        ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int]
    return _host


def _dev_lib():
    global _dev
    if _dev is None:
        if not os.path.exists(_DEV_SO):
            build()
        _dev = ctypes.CDLL(_DEV_SO)
        _dev.zhs_fill_device.restype = ctypes.c_int
        _dev.zhs_fill_device.argtypes = [ctypes.POINTER(_Params), ctypes.c_int, ctypes.c_int32, ctypes.c_int32,
                                         ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                                         ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p]
    return _dev


def fill_host(spec: DemSpec, gcols: int, row0: int, col0: int, nrows: int, ncols: int,
              out: np.ndarray | None = None, nthreads: int | None = None) -> np.ndarray:
    """Window [row0,row0+nrows) x [col0,col0+ncols) of the global raster (gcols columns) as int16."""
    if out is None:
        out = np.empty((nrows, ncols), dtype=np.int16)
    assert out.dtype == np.int16 and out.ndim == 2 and out.shape[0] >= nrows and out.shape[1] >= ncols
    assert out.strides[1] == 2
    pitch = out.strides[0] // 2
    p = spec._c()
    _host_lib().zhs_fill_host(ctypes.byref(p), spec.kind, spec.pattern_mod, spec.pattern_off, gcols,
                              out.ctypes.data, row0, col0, nrows, ncols, pitch,
                              nthreads or os.cpu_count() or 1)
    return out


def fill_device(spec: DemSpec, gcols: int, dptr: int, row0: int, col0: int, nrows: int, ncols: int,
                pitch: int, stream: int = 0) -> None:
    """Fill a device buffer (raw pointer) with the same window the host fill would produce."""
    p = spec._c()
    rc = _dev_lib().zhs_fill_device(ctypes.byref(p), spec.kind, spec.pattern_mod, spec.pattern_off, gcols,
                                    ctypes.c_void_p(dptr), row0, col0, nrows, ncols, pitch,
                                    ctypes.c_void_p(stream))
    if rc != 0:
        raise RuntimeError(f"zhs_fill_device failed: cuda error {rc}")
