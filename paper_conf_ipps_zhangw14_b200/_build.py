"""In-tree build of libzh.so (nvcc, sm_100a).  No torch extension machinery: plain -shared.

Each source compiles to its own object in parallel (the kernels call no device code across
files: shared device functions live in the headers), then one nvcc link makes the library.
"""
from __future__ import annotations

import os
import subprocess
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OBJ = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libzh.so")
SOURCES = ["zh_api.cu", "k_tile_hist.cu", "k_pairs.cu", "k_aggregate.cu", "k_pip.cu", "k_fused.cu", "k_stats.cu",
           "k_touch.cu", "k_features.cu"]
HEADERS = ["zh_internal.cuh", "zh_ctx.h", "zh_tilehist.cuh", "zh_parity.cuh", "zh_pip.cuh"]

NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
              "-Xcompiler", "-fPIC", "-Xptxas", "-O3"]


def _deps():
    return [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(ROOT, "include", "zh.h"), __file__]


def _obj(src: str) -> str:
    return os.path.join(OBJ, src.replace(".cu", ".o"))


def _stale_obj(src: str, extra_flags) -> bool:
    o = _obj(src)
    if not os.path.exists(o):
        return True
    t = os.path.getmtime(o)
    flag_file = o + ".flags"
    if not os.path.exists(flag_file) or open(flag_file).read() != " ".join(extra_flags):
        return True
    return any(os.path.getmtime(d) > t for d in _deps() + [os.path.join(CSRC, src)])


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, s) for s in SOURCES] + _deps()
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, extra_flags=(), out: str | None = None) -> str:
    """Compile (changed objects only unless force) and link libzh.so.  extra_flags (e.g.
    ["-DZH_X=1"]) and out (another library path) serve A/B builds."""
    extra_flags = list(extra_flags)
    out = out or LIB
    if not force and not extra_flags and out == LIB and not _stale():
        return LIB
    nvcc = os.environ.get("NVCC", "nvcc")
    os.makedirs(OBJ, exist_ok=True)
    obj_dir_flags = extra_flags
    todo = [s for s in SOURCES if force or _stale_obj(s, obj_dir_flags)]

    def compile_one(src):
        cmd = [nvcc, *NVCC_FLAGS, *extra_flags, "-c", os.path.join(CSRC, src), "-o", _obj(src) + ".tmp"]
        if verbose:
            print(" ".join(cmd))
        subprocess.check_call(cmd)
        os.replace(_obj(src) + ".tmp", _obj(src))
        with open(_obj(src) + ".flags", "w") as f:
            f.write(" ".join(obj_dir_flags))

    with ThreadPoolExecutor(max_workers=min(len(todo), os.cpu_count() or 1) or 1) as ex:
        list(ex.map(compile_one, todo))
    cmd = [nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", *[_obj(s) for s in SOURCES],
           "-o", out + ".tmp"]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(out + ".tmp", out)
    return out


if __name__ == "__main__":
    build(force=True, verbose=True)
