#!/usr/bin/env python
"""bench.py — zonal histogramming throughput on B200 (raster cells/s, end-to-end), driver contract.

A "step" is one pass of the whole hot path: zh_pair_tiles (step 2, incl.
zeroing the output) then zh_fused_update (steps 1 + 3 + 4 fused tile by tile, SURVEY.md §8f-1;
`--path four_step` runs zh_tile_hist, zh_aggregate, zh_pip_update instead — both are timed) over
the CONUS-scale synthetic raster (93,600 x 216,000 int16 = 20.2 G cells, 40.4 GB resident in HBM)
and ~3,100 jagged county polygons; with N > 1 GPUs each rank holds a strip of whole tile rows
and the step ends with an NCCL all-reduce of the [n_poly, 5000] uint64 histograms.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config conus] [--impl ours|reference]

value = raster cells of the whole job / device time per step (max over ranks; CUDA events).
e2e   = the same metric through the public C ABI from HOST buffers: per step zh_create (polygon
        H2D) + zh_run on a pinned host raster (raster H2D, the four steps, result D2H).
roofline = the dominant kernel's algorithmic bytes / its CUDA-event time vs measured HBM peak.
cpu_baseline = the CPU oracle (oracle/, O1 row-hoisted, all host cores) on a bounded row band.
--impl reference = that oracle as the reference arm (this tier has no reference implementation).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CLOCK_Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
           "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
           "clocks_event_reasons.sw_power_cap")


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.lines: list[str] = []
        self.proc = None
        self.t = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={CLOCK_Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
            if self.t is not None:
                self.t.join(timeout=2)

    def summary(self) -> dict:
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for n, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


# BASELINE.json's metric (raster cells/s), measured over one device step; the end-to-end seconds
# are the e2e / e2e_resident objects of the same line
METRIC = ("raster cells/s (zonal histogram of the whole raster; device step = pairing + fused steps 1/3/4 "
          "with raster and polygons resident in HBM; e2e objects: host-side end to end)")


def host_info() -> dict:
    """The host the CPU oracle runs on (record nproc, the CPU model and host DRAM)."""
    model, mem = None, None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
        for line in open("/proc/meminfo"):
            if line.startswith("MemTotal"):
                mem = round(int(line.split()[1]) / 2 ** 20, 1)
                break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model, "host_mem_gib": mem}


def measured_peaks() -> dict:
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return {"hbm_gbs": float(d["hbm_gbs"]), "source": "measured (MEASURED_PEAKS.json)"}
    return {"hbm_gbs": 6650.0, "source": "fallback (B200_PROFILING.md)"}


def read_ceiling():
    """Read-only ceiling of the tile access pattern (no histogram: 16-byte loads of 256 x 256 tiles,
    runs of 8 tiles per CTA, XOR only) measured on a B200 by tools/microbench/tile_read_bw.cu and
    committed as profiles/r02/microbench_tile_read_bw.txt; the copy peak of MEASURED_PEAKS.json counts
    read + write bytes, which a kernel that only reads can exceed."""
    p = os.path.join(ROOT, "profiles", "r02", "microbench_tile_read_bw.txt")
    if not os.path.exists(p):
        return None
    best = None
    for line in open(p):
        if "run 8" in line and "GB/s" in line:
            v = float(line.split("=")[-1].split()[0])
            best = v if best is None else max(best, v)
    return (best, "tools/microbench/tile_read_bw.cu, runs of 8 tiles (profiles/r02/microbench_tile_read_bw.txt)") \
        if best else None


def traffic_from_profile(kernel_key: str, config: str, tile: int, path: str):
    """dram read+write bytes per launch of the dominant kernel from the committed ncu --set full
    capture of THIS configuration (profiles/ncu_traffic.json: {"<config>/T<tile>/<path>": {kernel:
    bytes}}), or None when no capture of this configuration exists (another config's bytes would
    say nothing about this launch)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    try:
        d = json.load(open(p))
        return d.get(f"{config}/T{tile}/{path}", {}).get(kernel_key)
    except Exception:
        return None


# ------------------------------------------------------------------------------------------------
# CPU oracle leg (cpu_baseline and --impl reference)
# ------------------------------------------------------------------------------------------------
def oracle_band(cfg, P, row_start: int, nrows: int, host_rows=None, threads=None):
    """Time the oracle (O1, all host cores) on rows [row_start, row_start+nrows) x all columns."""
    import numpy as np

    import oracle
    from synth.dem import fill_host
    threads = threads or os.cpu_count() or 1
    if host_rows is None:
        host_rows = fill_host(cfg.dem, cfg.cols, row_start, 0, nrows, cfg.cols, nthreads=threads)
    bins = oracle.make_bins(cfg.nbins, lo=cfg.lo, width=cfg.width, nodata=cfg.nodata, oor_drop=cfg.oor_drop)
    t0 = time.perf_counter()
    H = oracle.o1(host_rows, cfg.gt, P, bins, row0=row_start, nthreads=threads)
    dt = time.perf_counter() - t0
    return dt, int(np.asarray(H).sum()), threads


def calibrated_band(cfg, P, budget_s: float, row_mid: int | None = None, host=None, raster_dev=None):
    """Pick a band of rows centred on row_mid whose oracle time is ~budget_s: probe bands of
    doubling height until one takes >= budget_s / 8, then scale linearly."""
    row_mid = cfg.rows // 2 if row_mid is None else row_mid
    n = 64
    while True:
        n = min(n, cfg.rows)
        start = max(0, min(cfg.rows - n, row_mid - n // 2))
        if host is not None:
            band = host[start:start + n, :cfg.cols]
        elif raster_dev is not None:
            band = raster_dev[start:start + n, :cfg.cols].cpu().numpy()
        else:
            band = None
        dt, _, _ = oracle_band(cfg, P, start, n, host_rows=band)
        if dt >= budget_s / 8 or n >= cfg.rows:
            break
        n *= 2
    n = int(max(1, min(cfg.rows, n * budget_s / max(dt, 1e-6))))
    start = max(0, min(cfg.rows - n, row_mid - n // 2))
    return start, n


def run_reference(args, cfg):
    """Reference arm: the CPU oracle as it stands, on our config/metric, bounded sample per step."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    P = cfg.polygons()
    budget = max(2.0, min(10.0, 150.0 / max(1, args.steps + args.warmup)))
    start, n = calibrated_band(cfg, P, budget)
    from synth.dem import fill_host
    host = fill_host(cfg.dem, cfg.cols, start, 0, n, cfg.cols)
    for _ in range(args.warmup):
        oracle_band(cfg, P, start, n, host_rows=host)
    times = []
    threads = os.cpu_count() or 1
    for _ in range(args.steps):
        dt, _, threads = oracle_band(cfg, P, start, n, host_rows=host)
        times.append(dt)
    ms = 1000.0 * sum(times) / len(times)
    cells = n * cfg.cols
    value = cells / (ms / 1000.0)
    sample = (f"rows [{start},{start + n}) x all {cfg.cols} cols of {cfg.name} ({cells} cells, "
              f"{P.n_poly} polygons), oracle O1 (row-hoisted Franklin test), {threads} threads")
    line = {"impl": "reference", "metric": METRIC, "value": value,
            "unit": "cells/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "i16",
            "data": "synthetic", "config": cfg.describe(),
            "cpu_baseline": {"value": value, "unit": "cells/s", "cores": threads, "kind": "oracle", "sample": sample,
                             "host": host_info()},
            "e2e": {"value": value, "unit": "cells/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------------------------------
# our arm
# ------------------------------------------------------------------------------------------------
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="conus")
    ap.add_argument("--tile", type=int, default=None)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--verbose", action="store_true")
    ap.add_argument("--path", default="fused", choices=["fused", "four_step"],
                    help="fused: step 2 + zh_fused_update (steps 1+3+4 fused, SURVEY §8f-1); four_step: 2,1,3,4")
    ap.add_argument("--no-other", action="store_true", help="skip timing the other path")
    ap.add_argument("--no-graph", action="store_true",
                    help="issue the step's calls one by one instead of replaying them from a CUDA graph (zh_step_graph)")
    ap.add_argument("--cover", action="store_true",
                    help="count cells whose closed rectangle meets the polygon (R15, PAPER.md:12) instead of "
                         "testing the cell centre (not the headline configuration)")
    ap.add_argument("--equal-shards", action="store_true",
                    help="N > 1: equal tile-row strips instead of the work-balanced plan (zh_plan_rows)")
    ap.add_argument("--dense-reduce", action="store_true",
                    help="N > 1: NCCL reduce of all n_poly rows instead of the sparse reduce (dist.SparseReducer)")
    args = ap.parse_args()

    from synth.configs import CONFIGS
    cfg = CONFIGS[args.config]
    if args.tile:
        from dataclasses import replace
        cfg = replace(cfg, tile=args.tile)
    if args.impl == "reference":
        return run_reference(args, cfg)

    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangw14_b200 import zh
    from paper_conf_ipps_zhangw14_b200.dist import (SparseReducer, plan_shards, reduce_histograms, strip_polygons,
                                                    touched_polygons)
    from synth.dem import fill_device

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # ZH_BENCH_SHARED_GPU=1: every rank on cuda:0 with gloo — exercises the multi-rank code path on a
    # one-GPU box (numbers are not a scaling measurement then).  Default: one GPU per rank, NCCL.
    shared = os.environ.get("ZH_BENCH_SHARED_GPU", "0") == "1"
    if shared:
        local = 0
    torch.cuda.set_device(local)
    if world > 1 and not shared:
        # communicator set-up lines in the log (which NCCL transport / NVLS the ranks got)
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    def log(*a):
        if args.verbose and rank == 0:
            print(*a, file=sys.stderr, flush=True)

    t_setup = time.perf_counter()
    P = cfg.polygons()
    log(f"polygons: {P.n_poly} polys {P.n_vert} vertices ({time.perf_counter() - t_setup:.1f}s)")
    T = cfg.tile
    bounds = plan_shards(cfg.rows, cfg.cols, cfg.gt, P, T, world, balanced=not args.equal_shards)
    r0, r1 = bounds[rank], bounds[rank + 1]
    nrows = r1 - r0
    pitch = (cfg.cols + 7) // 8 * 8
    stream = torch.cuda.current_stream()
    raster = torch.empty((max(nrows, 1), pitch), dtype=torch.int16, device="cuda")
    fill_device(cfg.dem, cfg.cols, raster.data_ptr(), r0, 0, nrows, cfg.cols, pitch, stream.cuda_stream)
    torch.cuda.synchronize()
    log(f"raster shard rows [{r0},{r1}) generated ({time.perf_counter() - t_setup:.1f}s)")
    raster_v = raster[:nrows]
    out = torch.zeros((P.n_poly, cfg.nbins), dtype=torch.int64, device="cuda")
    # N > 1: each rank pairs only the polygons whose bounding box meets its strip (the others have
    # no cell centre there); its rows land in the global [n_poly, nbins] buffer by one index copy
    if world > 1:
        ids = strip_polygons(P, cfg.gt, r0, r1)
        Pr = P.subset(ids)
        out_r = torch.zeros((max(len(ids), 1), cfg.nbins), dtype=torch.int64, device="cuda")[:len(ids)]
        idx = torch.as_tensor(ids, device="cuda")
        log(f"rank {rank}: rows [{r0},{r1}), {len(ids)} of {P.n_poly} polygons")
    else:
        ids, Pr, out_r, idx = None, P, out, None

    def to_global():
        if idx is not None and len(ids):
            out.index_copy_(0, idx, out_r)

    z = zh.ZonalHistogram(raster_v, cfg.gt, Pr, cfg.nbins, lo=cfg.lo, width=cfg.width, nodata=cfg.nodata,
                          oor_drop=cfg.oor_drop, tile=T, rows=cfg.rows, cols=cfg.cols, row0=r0, stream=stream,
                          fused=(args.path == "fused"), cover=args.cover)
    z.set_output(out_r)

    # N > 1: sparse reduce (only polygons spanning strips are summed; the plan is geometry only),
    # unless --dense-reduce (the shared-GPU gloo mode stages its point-to-point rows through the host)
    reducer = None
    if world > 1 and not args.dense_reduce:
        z.zh_pair_tiles()
        reducer = SparseReducer(ids[touched_polygons(z)], P.n_poly, device=out.device)
        log(f"sparse reduce: {len(reducer.shared)} shared polygons, {reducer.rows_moved()} rows moved "
            f"(dense: {world * P.n_poly})")

    def reduce_out():
        to_global()
        if reducer is not None:
            reducer.reduce(out, to_rank0=True)
        else:
            reduce_histograms(out, to_rank0=True)  # only rank 0 reads the result (half the traffic of an all-reduce)

    path = args.path
    z.set_timing(True)
    lib_ms = []  # per timed step: the library's own event timings (steps, fused inner kernels)

    def one_step(record=False, mode=None):
        mode = mode or path
        if mode == path and not args.no_graph:
            z.zh_step_graph()  # the step replayed from a CUDA graph (captured during the warm-up)
        else:
            z.zh_pair_tiles()
            if mode == "fused":
                z.zh_fused_update()
            else:
                z.zh_tile_hist()
                z.zh_aggregate()
                z.zh_pip_update()
        if record:
            lib_ms.append(z.step_ms())  # syncs after the step's last kernel
        if world > 1:
            if record:
                r0e, r1e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                r0e.record(stream)
                reduce_out()
                r1e.record(stream)
                red_ev.append((r0e, r1e))
            else:
                reduce_out()

    red_ev = []  # per timed step: events around the histogram reduction (N > 1)
    clk = ClockSampler(local).__enter__()
    time.sleep(0.5)  # nvidia-smi needs a moment before its first sample
    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()
    st = z.stats()
    log(f"stats {st}")

    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches0 = z.launch_count()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        one_step(record=True)
    e1.record(stream)
    torch.cuda.synchronize()
    clk.__exit__(None, None, None)
    if world > 1:
        dist.barrier()
    launches = z.launch_count() - launches0
    ms_local = e0.elapsed_time(e1) / args.steps
    ms_t = torch.tensor([ms_local], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms = float(ms_t.item())
    value = cfg.cells / (ms / 1000.0)
    st = z.stats()

    def avg(rows, key):
        v = [r[key] for r in rows if r[key] >= 0]
        return sum(v) / len(v) if v else None

    peaks = measured_peaks()
    cells_local = nrows * cfg.cols
    B_pad = (cfg.nbins + 3) // 4 * 4
    # algorithmic bytes per launch
    kern = {}
    if path == "fused":
        kern["k_fused_pure"] = (avg(lib_ms, "fused_pure_kernel"), 2.0 * st["n_pure_cells"])
        # mixed tiles: the HBM bytes k_mixed_cells must read are every mixed tile's cells once
        # (n_mixed_cells; a tile's later groups of <= 2 pairs re-read it from L2 — n_group_cells
        # counts those too and is reported beside); the per-pair k_pip_cells (when the grouped form
        # does not apply) reads a tile once per pair
        grouped = st["n_mixed_groups"] > 0
        cell_k = "k_mixed_cells" if grouped else "k_pip_cells"
        kern[cell_k] = (avg(lib_ms, "fused_pip_kernel"), 2.0 * (st["n_mixed_cells"] if grouped else st["n_pip_cells"]))
        steps_detail = {"step2_pair_tiles": {"ms": avg(lib_ms, "step2_pair_tiles")},
                        "fused_update(steps1+3+4)": {"ms": avg(lib_ms, "fused_update")}}
    else:
        kern["k_tile_hist"] = (avg(lib_ms, "step1_tile_hist"), 2.0 * cells_local + 4.0 * B_pad * st["n_tiles"])
        kern["k_aggregate"] = (avg(lib_ms, "step3_aggregate"), 4.0 * cfg.nbins * st["n_inside"])
        kern["k_pip_cells+k_parity (pair-cell bytes, not HBM bytes)"] = (avg(lib_ms, "step4_pip_update"),
                                                                         2.0 * st["n_isect"] * T * T)
        steps_detail = {"step2_pair_tiles": {"ms": avg(lib_ms, "step2_pair_tiles")}}
    for name, (t, b) in kern.items():
        steps_detail[name] = {"ms": t, "alg_bytes": b, "alg_GBps": b / (t / 1000.0) / 1e9 if t else None}
    if path == "fused" and st["n_mixed_groups"] > 0:
        t = steps_detail["k_mixed_cells"]["ms"]
        steps_detail["k_mixed_cells"]["group_read_bytes"] = 2.0 * st["n_group_cells"]  # incl. L2 re-reads
        steps_detail["k_mixed_cells"]["group_read_GBps"] = 2.0 * st["n_group_cells"] / (t / 1000.0) / 1e9 if t else None
    if path == "fused":
        # the parity bitmaps of the mixed pairs (FP64 crossing work; after k_fused_pure, exact grid)
        steps_detail["k_parity"] = {"ms": avg(lib_ms, "fused_parity_kernel")}
    if red_ev:
        steps_detail["reduce_histograms"] = {
            "ms": sum(a.elapsed_time(b) for a, b in red_ev) / len(red_ev),
            "kind": "sparse" if reducer is not None else "dense",
            "rows_moved": reducer.rows_moved() if reducer is not None else world * P.n_poly}
    dom = max(kern, key=lambda k: kern[k][0] or 0.0)
    dom_ms, dom_b = kern[dom]
    achieved = dom_b / (dom_ms / 1000.0) / 1e9
    roofline = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": achieved / peaks["hbm_gbs"],
                # the ncu capture is of the N = 1 launch; a shard's launch is a different one
                "traffic": traffic_from_profile(dom, cfg.name, T, path) if world == 1 else None,
                "peak_source": peaks["source"], "alg_bytes_per_launch": dom_b,
                "share_of_step": dom_ms / ms if ms > 0 else None}
    rc = read_ceiling()
    if rc is not None:  # the copy peak counts read + write bytes; these kernels only read
        roofline["read_ceiling"] = {"value": rc[0], "unit": "GB/s", "frac": achieved / rc[0], "source": rc[1]}
    log(f"timed ({path}): {ms:.3f} ms/step, {steps_detail}")

    # the other path, timed the same way (every SURVEY §8a row measured); not the headline
    other = None
    if not args.no_other:
        other_mode = "four_step" if path == "fused" else "fused"
        lib_ms.clear()
        for _ in range(2):
            one_step(mode=other_mode)
        torch.cuda.synchronize()
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        for _ in range(args.steps):
            one_step(record=True, mode=other_mode)
        f1.record(stream)
        torch.cuda.synchronize()
        st2 = z.stats()
        other = {"path": other_mode, "ms_per_step": f0.elapsed_time(f1) / args.steps}
        if other_mode == "four_step":
            tb = 2.0 * cells_local + 4.0 * B_pad * st2["n_tiles"]
            for key, b in (("step1_tile_hist", tb), ("step2_pair_tiles", None),
                           ("step3_aggregate", 4.0 * cfg.nbins * st2["n_inside"]),
                           ("step4_pip_update", 2.0 * st2["n_isect"] * T * T)):
                t = avg(lib_ms, key)
                other[key] = {"ms": t}
                if b and key != "step4_pip_update":
                    other[key]["alg_GBps"] = b / (t / 1000.0) / 1e9 if t else None
                    other[key]["frac_of_hbm_peak"] = other[key]["alg_GBps"] / peaks["hbm_gbs"] if t else None
                elif b:
                    # 2 B x every cell of every intersecting pair: pairs sharing a tile re-read it
                    # (from L2), and vectors with no inside cell are not read at all — a rate of
                    # pair-cells, not of HBM bytes (ncu: profiles/ for the DRAM bytes)
                    other[key]["pair_cell_GBps"] = b / (t / 1000.0) / 1e9 if t else None
        else:
            other["fused_update"] = {"ms": avg(lib_ms, "fused_update")}
        log(f"other path: {other}")

    # ---- end to end through the C ABI from host buffers
    e2e = None
    e2e_res = None
    host = None
    if not args.no_e2e:
        e2e_res = run_e2e_resident(args, cfg, P, Pr, raster_v, out, out_r, r0, world, rank, stream, log, reduce_out)
        e2e, host = run_e2e(args, cfg, P, Pr, z, raster_v, out, out_r, r0, nrows, pitch, world, rank, stream, log,
                            reduce_out)
    z.close()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        start, n = calibrated_band(cfg, P, args.cpu_seconds, host=host, raster_dev=raster_v)
        if host is not None:
            band = host[start:start + n, :cfg.cols]
        else:
            band = raster_v[start:start + n, :cfg.cols].cpu().numpy()
        dt, cnt, threads = oracle_band(cfg, P, start, n, host_rows=band)
        cpu = {"value": n * cfg.cols / dt, "unit": "cells/s", "cores": threads, "kind": "oracle", "host": host_info(),
               "sample": f"rows [{start},{start + n}) x all {cfg.cols} cols of {cfg.name} ({n * cfg.cols} cells, "
                         f"{P.n_poly} polygons), oracle O1 on {threads} host threads, {dt:.1f} s"}

    if rank == 0:
        clocks = clk.summary()
        line = {"metric": METRIC, "value": value, "unit": "cells/s",
                "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "i16",
                "data": "synthetic (fractal int16 DEM + jagged Voronoi counties, seeded)",
                "config": dict(cfg.describe(), n_poly=P.n_poly, n_vert=P.n_vert,
                               parallelism=f"tile-row shards x{world}" + (" (shared GPU, gloo)" if shared else "")
                               + ("" if world == 1 else (" equal" if args.equal_shards else " work-balanced"))
                               + ("" if world == 1 else (" sparse-reduce" if reducer is not None else " dense-reduce")),
                               l2="inputs larger than L2 (40 GB raster)", counts="uint64", pip="float64 no-FMA",
                               semantics="closed rectangle meets polygon (R15)" if args.cover else "centre inside"),
                "e2e": e2e, "e2e_resident": e2e_res, "gpu_launches": launches, "roofline": roofline, "cpu_baseline": cpu,
                "clocks": clocks, "path": path, "steps_detail": steps_detail, "other_path": other,
                "pairs": {k: st[k] for k in ("n_tiles", "n_candidates", "n_inside", "n_isect", "n_band_entries",
                                             "n_edges", "n_pure_tiles", "n_pip_pairs", "n_pure_cells", "n_pip_cells")},
                "setup_s": time.perf_counter() - t_setup}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def _pin_polygons(P):
    """Page-lock the polygon vertex arrays (zh_create's H2D then runs at PCIe speed)."""
    import numpy as np
    import torch
    cudart = torch.cuda.cudart()
    pinned = []
    for a in (P.x, P.y):
        if a.flags.c_contiguous and a.dtype == np.float64 and a.nbytes:
            rv = cudart.cudaHostRegister(a.ctypes.data, a.nbytes, 0)
            if (int(rv) if not isinstance(rv, tuple) else int(rv[0])) == 0:
                pinned.append(a)
    return pinned


def _unpin(arrs):
    import torch
    for a in arrs:
        torch.cuda.cudart().cudaHostUnregister(a.ctypes.data)


def run_e2e_resident(args, cfg, P, Pr, raster_v, out, out_r, r0, world, rank, stream, log, reduce_out):
    """SURVEY.md §8d's end-to-end time (the paper's, §IV.A: data resident in GPU memory,
    disk I/O excluded): from "raster in HBM, polygons on the host" to "P x B matrix on the host" —
    zh_create (polygon H2D), zh_run (step 2 + fused steps 1/3/4), the reduce (N > 1), the result
    D2H and zh_destroy, every step."""
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangw14_b200 import zh
    poly_pinned = _pin_polygons(Pr)
    res_pin = torch.empty((P.n_poly, cfg.nbins), dtype=torch.int64, pin_memory=True)
    res = res_pin.numpy().view(np.uint64)
    times = []
    for it in range(max(args.e2e_steps, 5) + 1):  # first iteration is a warm-up
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        z2 = zh.ZonalHistogram(raster_v, cfg.gt, Pr, cfg.nbins, lo=cfg.lo, width=cfg.width, nodata=cfg.nodata,
                               oor_drop=cfg.oor_drop, tile=cfg.tile, rows=cfg.rows, cols=cfg.cols, row0=r0,
                               stream=stream, fused=(args.path == "fused"), cover=args.cover)
        if world > 1:
            z2.set_output(out_r)
            z2.zh_run(None)
            reduce_out()
            if rank == 0:
                res_pin.copy_(out, non_blocking=True)
            torch.cuda.synchronize()
        else:
            z2.zh_run(res)
        dt = time.perf_counter() - t0
        z2.close()
        t = torch.tensor([dt], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        if it > 0:
            times.append(float(t.item()))
    _unpin(poly_pinned)
    sec = sum(times) / len(times)
    h2d = Pr.x.nbytes + Pr.y.nbytes + Pr.poly_ring_off.nbytes // 2 + Pr.ring_vert_off.nbytes // 2
    if world > 1:
        h2d_t = torch.tensor([h2d], dtype=torch.int64, device="cuda")
        dist.all_reduce(h2d_t)
        h2d = int(h2d_t.item())
    log(f"e2e (resident raster) {sec:.4f} s/step")
    return {"value": cfg.cells / sec, "unit": "cells/s", "seconds_per_step": sec, "h2d_bytes_per_step": h2d,
            "d2h_bytes_per_step": P.n_poly * cfg.nbins * 8, "steps": len(times),
            "includes": "raster resident in HBM (SURVEY.md 8d / PAPER.md:22): zh_create (polygon H2D from pinned "
                        "host arrays) + zh_run (step 2 + fused update) + reduce (N > 1) + result D2H + zh_destroy"}


def run_e2e(args, cfg, P, Pr, z, raster_v, out, out_r, r0, nrows, pitch, world, rank, stream, log, reduce_out):
    """E2E through the public API: host raster (pinned) + host polygons -> host histogram."""
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangw14_b200 import zh

    # pinned host copy of this rank's strip (identical to the device one; D2H is not timed)
    host = np.empty((max(nrows, 1), pitch), dtype=np.int16)
    cudart = torch.cuda.cudart()
    nbytes = host.nbytes
    reg = cudart.cudaHostRegister(host.ctypes.data, nbytes, 0)
    pinned = int(reg) == 0 if not isinstance(reg, tuple) else int(reg[0]) == 0
    torch.from_numpy(host)[:nrows].copy_(raster_v)
    # the polygon vertex arrays are pinned too (zh_create's H2D of 154 MB then runs at PCIe speed
    # instead of through pageable staging)
    poly_pinned = _pin_polygons(Pr)
    torch.cuda.synchronize()
    z.close()  # free the resident context's tile histograms before the e2e context allocates its own
    res_pin = torch.empty((P.n_poly, cfg.nbins), dtype=torch.int64, pin_memory=True)
    res = res_pin.numpy().view(np.uint64)  # pinned: the result's D2H runs at full PCIe speed
    host_v = host[:nrows]
    times = []
    for it in range(args.e2e_steps + 1):  # first iteration is a warm-up
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        z2 = zh.ZonalHistogram(host_v, cfg.gt, Pr, cfg.nbins, lo=cfg.lo, width=cfg.width, nodata=cfg.nodata,
                               oor_drop=cfg.oor_drop, tile=cfg.tile, rows=cfg.rows, cols=cfg.cols, row0=r0,
                               stream=stream, fused=(args.path == "fused"), cover=args.cover)
        if world > 1:
            z2.set_output(out_r)
            z2.zh_run(None)
            reduce_out()
            if rank == 0:
                res_pin.copy_(out, non_blocking=True)
            torch.cuda.synchronize()
        else:
            z2.zh_run(res)
        dt = time.perf_counter() - t0
        raster_h2d = z2.stats()["h2d_bytes"]
        z2.close()
        t = torch.tensor([dt], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        if it > 0:
            times.append(float(t.item()))
    if pinned:
        cudart.cudaHostUnregister(host.ctypes.data)
    _unpin(poly_pinned)
    host = host[:nrows, :cfg.cols]
    sec = sum(times) / len(times)
    poly_bytes = Pr.x.nbytes + Pr.y.nbytes + Pr.poly_ring_off.nbytes // 2 + Pr.ring_vert_off.nbytes // 2
    h2d = raster_h2d + poly_bytes  # the fused zh_run uploads only the tiles some pair needs
    if world > 1:
        h2d_total = torch.tensor([h2d], dtype=torch.int64, device="cuda")
        dist.all_reduce(h2d_total)
        h2d = int(h2d_total.item())
    d2h = P.n_poly * cfg.nbins * 8
    log(f"e2e {sec:.3f} s/step (pinned={pinned})")
    return {"value": cfg.cells / sec, "unit": "cells/s", "seconds_per_step": sec, "h2d_bytes_per_step": h2d,
            "d2h_bytes_per_step": d2h, "host_raster_pinned": bool(pinned), "host_vertices_pinned": len(poly_pinned) == 2, "steps": len(times),
            "raster_h2d_bytes": raster_h2d, "raster_bytes": nrows * pitch * 2,
            "includes": f"zh_create (polygon H2D, allocation from libzh's block cache) + zh_run ({args.path}: step 2, "
                        f"raster H2D of the tiles some pair needs, steps) + result D2H + zh_destroy"}, host


if __name__ == "__main__":
    sys.exit(main())
