"""CPU-side checks of the boundary: libzh builds for sm_100a, loads, exports every symbol zh.h
declares, and rejects malformed input without touching a GPU (validation happens before any
CUDA call)."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "zh.h")).read()
    return sorted(set(re.findall(r"^\s*(?:zh_status|void|const char\*|int32_t|int64_t)\s+(zh_\w+)\s*\(", src, re.M)))


def test_header_declares_the_north_star_calls():
    names = _declared()
    for n in ["zh_create", "zh_tile_hist", "zh_pair_tiles", "zh_aggregate", "zh_pip_update", "zh_run",
              "zh_output_device", "zh_last_error", "zh_destroy"]:
        assert n in names


def test_library_exports_every_declared_symbol():
    from paper_conf_ipps_zhangw14_b200 import _build
    lib = _build.build()
    out = subprocess.run(["nm", "-D", "--defined-only", lib], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (zh_\w+)", out))
    missing = [n for n in _declared() if n not in exported]
    assert not missing, missing
    from paper_conf_ipps_zhangw14_b200 import zh
    assert set(zh.EXPORTS) == set(_declared())
    assert zh.LIB.zh_abi_version() == 8


def test_library_is_sm100a_sass():
    from paper_conf_ipps_zhangw14_b200 import _build
    lib = _build.build()
    out = subprocess.run(["cuobjdump", "--list-elf", lib], capture_output=True, text=True, check=True).stdout
    assert "sm_100a" in out


def _sass_functions(lib):
    out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True, check=True).stdout
    funcs, cur = {}, None
    for line in out.splitlines():
        m = re.match(r"\s+Function : (\S+)", line)
        if m:
            cur = m.group(1)
            funcs[cur] = []
        elif cur is not None:
            funcs[cur].append(line)
    return funcs


def test_pip_predicate_has_no_contracted_fma():
    """The intercept / centre expressions are written with __dadd_rn/__dsub_rn/__dmul_rn/__ddiv_rn
    (R7), which nvcc never contracts.  Weak SASS check on every kernel evaluating the predicate:
    DMUL and DADD are present, and DFMA appears only as part of division sequences (each IEEE
    double division is an MUFU.RCP64H followed by a handful of DFMAs).  k_mbb_edges' row searches
    start from reciprocal first guesses ((y - gt3) * igt5 - oy, free to contract: first_false
    re-decides every row with the exact row_centre expression); its divisions are the MBB's
    tile rectangle (a one-cell margin, no decision of the predicate)."""
    from paper_conf_ipps_zhangw14_b200 import _build
    funcs = _sass_functions(_build.build())
    names = [n for n in funcs if any(k in n for k in ("k_pipILi", "k_parity", "k_classify", "k_mbb_edges"))]
    assert any("k_parity" in n for n in names) and any("k_mbb_edges" in n for n in names)
    for n in names:
        sass = "\n".join(funcs[n])
        assert "DMUL" in sass and "DADD" in sass, n
        n_rcp = sass.count("MUFU.RCP64H")
        if "k_mbb_edges" in n:
            # four divisions of the tile rectangle (a conservative margin, not the predicate) and
            # the reciprocal first guesses of the row searches; the row decisions are DADD/DMUL
            assert n_rcp <= 8 and sass.count("DFMA") <= 10 * n_rcp + 4, n
            continue
        assert n_rcp >= 1, n
        assert sass.count("DFMA") <= 10 * n_rcp, n


def test_cover_segment_test_is_not_contracted():
    """R15's segment-vs-cell test (k_touch) is written with __dsub_rn/__dmul_rn: its orientation
    products must appear as DMUL, never fused into a DFMA with the following subtraction."""
    from paper_conf_ipps_zhangw14_b200 import _build
    funcs = _sass_functions(_build.build())
    names = [n for n in funcs if "k_touch" in n]
    assert names
    sass = "\n".join(funcs[names[0]])
    assert sass.count("DMUL") >= 8  # two products per corner, four corners


def _mk(lib_zh, **over):
    zh = lib_zh
    r = zh.zh_raster()
    buf = np.zeros((16, 16), np.int16)
    r.data = buf.ctypes.data
    r.rows, r.cols, r.pitch, r.row0, r.nrows = 16, 16, 16, 0, 16
    r.gt = (ctypes.c_double * 6)(0, 1, 0, 16, 0, -1)
    r.on_host = 1
    pro = np.array([0, 1], np.int64)
    rvo = np.array([0, 3], np.int64)
    x = np.array([0.0, 8, 0])
    y = np.array([0.0, 0, 8])
    p = zh.zh_polygons(1, 1, 3, pro.ctypes.data, rvo.ctypes.data, x.ctypes.data, y.ctypes.data)
    b = zh.zh_bins(0, 1, 16, 0, 0, 0)
    o = zh.zh_options(4, 1, 0, 0, None)
    for k, v in over.items():
        obj, field = k.split("__")
        target = {"r": r, "p": p, "b": b, "o": o}[obj]
        setattr(target, field, v)
    return r, p, b, o, (buf, pro, rvo, x, y)


@pytest.mark.parametrize("over,status", [
    ({"o__tile": 0}, 1), ({"b__nbins": 0}, 1), ({"b__width": 0}, 1), ({"r__pitch": 8}, 1),
    ({"r__row0": 3, "r__nrows": 8}, 1), ({"r__nrows": 20}, 1), ({"b__nbins": 1 << 20}, 1),
    # nodata must be an int16 value (a wider one would alias a real value in the packed bin path)
    ({"b__use_nodata": 1, "b__nodata": 65535}, 1), ({"b__use_nodata": 1, "b__nodata": -32769}, 1),
    # uint32 shared histograms: T^2 < 2^31
    ({"o__tile": 46341}, 2),
])
def test_create_rejects_malformed_input(over, status):
    from paper_conf_ipps_zhangw14_b200 import zh
    r, p, b, o, keep = _mk(zh, **over)
    h = ctypes.c_void_p()
    st = zh.LIB.zh_create(ctypes.byref(h), ctypes.byref(r), ctypes.byref(p), ctypes.byref(b), ctypes.byref(o))
    assert st == status
    assert h.value is None
    assert zh.LIB.zh_last_error()


def test_create_rejects_rotation_nan_and_bad_offsets():
    from paper_conf_ipps_zhangw14_b200 import zh
    r, p, b, o, keep = _mk(zh)
    r.gt = (ctypes.c_double * 6)(0, 1, 0.1, 16, 0, -1)
    h = ctypes.c_void_p()
    assert zh.LIB.zh_create(ctypes.byref(h), ctypes.byref(r), ctypes.byref(p), ctypes.byref(b), ctypes.byref(o)) == 2
    r, p, b, o, keep = _mk(zh)
    keep[3][1] = np.nan
    assert zh.LIB.zh_create(ctypes.byref(h), ctypes.byref(r), ctypes.byref(p), ctypes.byref(b), ctypes.byref(o)) == 1
    r, p, b, o, keep = _mk(zh)
    keep[2][1] = 5  # ring_vert_off end != n_vert
    assert zh.LIB.zh_create(ctypes.byref(h), ctypes.byref(r), ctypes.byref(p), ctypes.byref(b), ctypes.byref(o)) == 1
    # uint32 output with a polygon whose MBB could exceed 2^32 cells
    r, p, b, o, keep = _mk(zh)
    r.rows, r.cols, r.nrows = 100000, 100000, 100000
    keep[3][:] = [0, 1e6, 0]
    keep[4][:] = [0, 0, -1e6]
    r.pitch = 100000
    o.out_u64 = 0
    assert zh.LIB.zh_create(ctypes.byref(h), ctypes.byref(r), ctypes.byref(p), ctypes.byref(b), ctypes.byref(o)) == 5


def test_null_context_calls_fail_cleanly():
    from paper_conf_ipps_zhangw14_b200 import zh
    for f in ["zh_tile_hist", "zh_aggregate", "zh_pip_update", "zh_upload_raster"]:
        assert getattr(zh.LIB, f)(None) == 1
    assert zh.LIB.zh_run(None, None) == 1
    zh.LIB.zh_destroy(None)
