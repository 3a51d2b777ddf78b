// zh_api.cu — the C ABI of libzh (include/zh.h): validation, context lifetime, step orchestration.
#include <float.h>

#ifndef ZH_DEVICE_SCAN
#define ZH_DEVICE_SCAN 1  // zh_create: the vertex scan of large inputs on the device
#endif
#include <math.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <map>
#include <mutex>
#include <new>
#include <thread>
#include <utility>
#include <vector>

#include "../../include/zh.h"
#include "zh_ctx.h"

using zh::Ctx;

// NVTX ranges around the ABI calls (header-only NVTX 3: free when no tool is attached), so nsys /
// ncu timelines show the paper's steps by name.
#ifndef ZH_NVTX
#define ZH_NVTX 1
#endif
#if ZH_NVTX
#include <nvtx3/nvToolsExt.h>
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
#define ZH_RANGE(name) NvtxRange zh_nvtx_range_(name)
#else
#define ZH_RANGE(name) (void)0
#endif

static thread_local char g_err[512] = "";

static zh_status fail(zh_status s, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
  return s;
}

static zh_status cuda_fail(cudaError_t e, const char* where) {
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    return fail(ZH_ERR_OOM, "%s: out of device memory", where);
  }
  return fail(ZH_ERR_CUDA, "%s: %s", where, cudaGetErrorString(e));
}

#define ZH_CU(call, where)                              \
  do {                                                  \
    cudaError_t _e = (call);                            \
    if (_e != cudaSuccess) return cuda_fail(_e, where); \
  } while (0)

static Ctx* C(zh_ctx c) { return reinterpret_cast<Ctx*>(c); }

// ---- process-wide cache of device blocks (zh_ctx.h) -------------------------------------------
namespace {
struct BlockCache {
  std::mutex m;
  std::multimap<size_t, std::pair<int, void*>> free_blocks;  // bytes -> (device, pointer)
  size_t cached = 0;
  bool enabled = true;
};
BlockCache& cache() {
  static BlockCache* c = new BlockCache();  // never destroyed: blocks may be returned at exit
  return *c;
}
void trim_locked(BlockCache& bc, int dev) {  // dev < 0: every device
  for (auto it = bc.free_blocks.begin(); it != bc.free_blocks.end();) {
    if (dev < 0 || it->second.first == dev) {
      if (it->second.first == -1) cudaFreeHost(it->second.second);
      else cudaFree(it->second.second);
      bc.cached -= it->first;
      it = bc.free_blocks.erase(it);
    } else {
      ++it;
    }
  }
}
}  // namespace

cudaError_t zh::cache_alloc(void** p, size_t* got, size_t need) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  BlockCache& bc = cache();
  std::lock_guard<std::mutex> lk(bc.m);
  // smallest cached block of this device that holds `need` without wasting more than half of it
  for (auto it = bc.free_blocks.lower_bound(need); it != bc.free_blocks.end() && it->first <= 2 * need + (1u << 20);
       ++it) {
    if (it->second.first != dev) continue;
    *p = it->second.second;
    *got = it->first;
    bc.cached -= it->first;
    bc.free_blocks.erase(it);
    return cudaSuccess;
  }
  e = cudaMalloc(p, need);
  if (e == cudaErrorMemoryAllocation && bc.cached > 0) {  // give the cache back and retry once
    cudaGetLastError();
    trim_locked(bc, dev);
    e = cudaMalloc(p, need);
  }
  if (e == cudaSuccess) *got = need;
  return e;
}

void zh::cache_free(void* p, size_t bytes) {
  BlockCache& bc = cache();
  int dev = 0;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) == cudaSuccess) dev = a.device;
  else cudaGetLastError();
  std::lock_guard<std::mutex> lk(bc.m);
  if (!bc.enabled) {
    cudaFree(p);
    return;
  }
  bc.free_blocks.emplace(bytes, std::make_pair(dev, p));
  bc.cached += bytes;
}

// Small pinned host buffers (list sizes, needed-tile flags) go through the same cache (device key
// -1): cudaFreeHost was measured taking 1 to 600 ms per call while a 40 GB host raster is pinned.
static cudaError_t pinned_alloc(void** p, size_t* got, size_t need) {
  BlockCache& bc = cache();
  {
    std::lock_guard<std::mutex> lk(bc.m);
    for (auto it = bc.free_blocks.lower_bound(need); it != bc.free_blocks.end() && it->first <= 2 * need + 4096;
         ++it) {
      if (it->second.first != -1) continue;
      *p = it->second.second;
      *got = it->first;
      bc.cached -= it->first;
      bc.free_blocks.erase(it);
      return cudaSuccess;
    }
  }
  cudaError_t e = cudaHostAlloc(p, need, cudaHostAllocDefault);
  if (e == cudaSuccess) *got = need;
  return e;
}

static void pinned_free(void* p, size_t bytes) {
  if (!p) return;
  BlockCache& bc = cache();
  std::lock_guard<std::mutex> lk(bc.m);
  if (!bc.enabled) {
    cudaFreeHost(p);
    return;
  }
  bc.free_blocks.emplace(bytes, std::make_pair(-1, p));
  bc.cached += bytes;
}

extern "C" int64_t zh_cache_bytes(void) {
  BlockCache& bc = cache();
  std::lock_guard<std::mutex> lk(bc.m);
  return (int64_t)bc.cached;
}

extern "C" void zh_trim_cache(int32_t keep_caching) {
  BlockCache& bc = cache();
  std::lock_guard<std::mutex> lk(bc.m);
  trim_locked(bc, -1);
  bc.enabled = keep_caching != 0;
}

extern "C" const char* zh_last_error(void) { return g_err; }
extern "C" int32_t zh_abi_version(void) { return ZH_ABI_VERSION; }

static const int32_t kMaxBins = 49152;  // shared-memory histogram limit (192 KB per CTA)

static zh_status validate(const zh_raster* r, const zh_polygons* p, const zh_bins* b, const zh_options* o) {
  if (!r || !p || !b || !o) return fail(ZH_ERR_INVALID_ARG, "null argument");
  if (r->rows < 1 || r->cols < 1) return fail(ZH_ERR_INVALID_ARG, "raster rows/cols must be >= 1");
  if (r->pitch < r->cols) return fail(ZH_ERR_INVALID_ARG, "pitch (%lld) < cols (%lld)", (long long)r->pitch,
                                      (long long)r->cols);
  if (r->row0 < 0 || r->nrows < 0 || r->row0 + r->nrows > r->rows)
    return fail(ZH_ERR_INVALID_ARG, "shard rows [row0, row0+nrows) outside the raster");
  if (o->tile < 1) return fail(ZH_ERR_INVALID_ARG, "tile must be >= 1");
  if (o->rep_custom && !(o->rep_x >= 0.0 && o->rep_x <= 1.0 && o->rep_y >= 0.0 && o->rep_y <= 1.0))
    return fail(ZH_ERR_INVALID_ARG, "representative point offsets must lie in [0, 1]");
  if (o->cover != 0 && o->cover != 1) return fail(ZH_ERR_INVALID_ARG, "cover must be 0 or 1");
  if (o->cover && o->rep_custom)
    return fail(ZH_ERR_UNSUPPORTED, "cover mode decides the cells no edge reaches by their centre (rep_custom = 0)");
  if (r->row0 % o->tile != 0) return fail(ZH_ERR_INVALID_ARG, "row0 must be a multiple of the tile size");
  for (int i = 0; i < 6; ++i)
    if (!isfinite(r->gt[i])) return fail(ZH_ERR_INVALID_ARG, "geotransform must be finite");
  if (r->gt[2] != 0.0 || r->gt[4] != 0.0) return fail(ZH_ERR_UNSUPPORTED, "rotated geotransforms are not supported");
  if (r->gt[1] == 0.0 || r->gt[5] == 0.0) return fail(ZH_ERR_INVALID_ARG, "gt[1] and gt[5] must be nonzero");
  if (r->nrows > 0 && !r->data) return fail(ZH_ERR_INVALID_ARG, "raster data is NULL");
  if (!r->on_host) {
    if (((uintptr_t)r->data & 15u) != 0) return fail(ZH_ERR_INVALID_ARG, "device raster must be 16-byte aligned");
    if (r->pitch % 8 != 0) return fail(ZH_ERR_INVALID_ARG, "device raster pitch must be a multiple of 8");
  }
  if (r->rows >= (1ll << 31) || r->cols >= (1ll << 31)) return fail(ZH_ERR_UNSUPPORTED, "raster dimension >= 2^31");
  if (b->nbins < 1 || b->nbins > kMaxBins) return fail(ZH_ERR_INVALID_ARG, "nbins must be in [1, %d]", kMaxBins);
  if (b->width < 1) return fail(ZH_ERR_INVALID_ARG, "width must be >= 1");
  if (b->lo > (1 << 30) || b->lo < -(1 << 30)) return fail(ZH_ERR_INVALID_ARG, "|lo| must be <= 2^30");
  if (b->use_nodata && (b->nodata < -32768 || b->nodata > 32767))
    return fail(ZH_ERR_INVALID_ARG, "nodata (%d) is not an int16 value", (int)b->nodata);
  // per-tile / per-pair shared histograms and the pure-run accumulator count in uint32: a tile must
  // hold < 2^32 cells, and the pure kernel caps its run of tiles accordingly (pure_params)
  if (o->tile > 46340) return fail(ZH_ERR_UNSUPPORTED, "tile size > 46340 (T^2 must stay below 2^31 cells)");
  if (p->n_poly < 0 || p->n_ring < 0 || p->n_vert < 0) return fail(ZH_ERR_INVALID_ARG, "negative polygon counts");
  if (p->n_vert >= (1ll << 31) - 1 || p->n_ring >= (1ll << 31) - 1 || p->n_poly >= (1ll << 31) - 1)
    return fail(ZH_ERR_UNSUPPORTED, "more than 2^31 vertices/rings/polygons");
  if (!p->poly_ring_off || !p->ring_vert_off) return fail(ZH_ERR_INVALID_ARG, "null offset array");
  if (p->n_vert > 0 && (!p->x || !p->y)) return fail(ZH_ERR_INVALID_ARG, "null coordinate array");
  if (p->poly_ring_off[0] != 0 || p->poly_ring_off[p->n_poly] != p->n_ring)
    return fail(ZH_ERR_INVALID_ARG, "poly_ring_off must start at 0 and end at n_ring");
  for (int64_t i = 0; i < p->n_poly; ++i)
    if (p->poly_ring_off[i + 1] < p->poly_ring_off[i])
      return fail(ZH_ERR_INVALID_ARG, "poly_ring_off not non-decreasing at %lld", (long long)i);
  if (p->ring_vert_off[0] != 0 || p->ring_vert_off[p->n_ring] != p->n_vert)
    return fail(ZH_ERR_INVALID_ARG, "ring_vert_off must start at 0 and end at n_vert");
  for (int64_t i = 0; i < p->n_ring; ++i)
    if (p->ring_vert_off[i + 1] < p->ring_vert_off[i])
      return fail(ZH_ERR_INVALID_ARG, "ring_vert_off not non-decreasing at %lld", (long long)i);
  return ZH_OK;
}

// Finiteness and max |coordinate| of the vertices (and with it the cell-size condition): one pass,
// split over host threads for large inputs (CONUS: 9.6 M vertices, ~25 ms on one core).  zh_create
// runs it before any CUDA call for small inputs, and for large ones while the vertex arrays are
// already on their way to the device (the DMA hides the scan).
static zh_status scan_verdict(const zh_raster* r, double amax, int64_t bad);

// Large inputs (ZH_DEVICE_SCAN): the same scan on the device right after the vertices' H2D (the host
// pass competed with the copy for host memory bandwidth: CONUS H2D 35 -> ~55 GB/s); the result comes
// back with zh_create's closing synchronisation.  out[0] = bits of max |coordinate| (non-negative
// doubles order like their bit patterns), out[1] = first non-finite vertex (INT64_MAX: none).
__global__ void k_scan_vertices(const double* __restrict__ x, const double* __restrict__ y, int64_t n,
                                unsigned long long* __restrict__ out) {
  double m = 0.0;
  long long bad = 0x7FFFFFFFFFFFFFFFll;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const double ax = fabs(x[i]), ay = fabs(y[i]);
    if (!(ax <= DBL_MAX) || !(ay <= DBL_MAX)) bad = min(bad, (long long)i);
    else m = fmax(m, fmax(ax, ay));
  }
  for (int o = 16; o > 0; o >>= 1) {
    m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
    bad = min(bad, __shfl_xor_sync(0xffffffffu, bad, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMax(&out[0], (unsigned long long)__double_as_longlong(m));
    atomicMin(reinterpret_cast<long long*>(&out[1]), bad);
  }
}

static zh_status scan_vertices(const zh_raster* r, const zh_polygons* p) {
  const int64_t nv = p->n_vert;
  const int nth = nv >= (1 << 20) ? (int)std::min<unsigned>(16u, std::max(1u, std::thread::hardware_concurrency())) : 1;
  std::vector<double> part_max(nth, 0.0);
  std::vector<int64_t> part_bad(nth, -1);
  auto scan = [&](int t) {
    const int64_t a = nv * t / nth, b = nv * (t + 1) / nth;
    double m = 0.0;
    for (int64_t i = a; i < b; ++i) {
      const double ax = fabs(p->x[i]), ay = fabs(p->y[i]);
      if (!(ax <= DBL_MAX) || !(ay <= DBL_MAX)) {  // NaN or infinite
        part_bad[t] = i;
        return;
      }
      m = std::max(m, std::max(ax, ay));
    }
    part_max[t] = m;
  };
  if (nth == 1) {
    scan(0);
  } else {
    std::vector<std::thread> th;
    for (int t = 0; t < nth; ++t) th.emplace_back(scan, t);
    for (auto& x : th) x.join();
  }
  double amax = 0.0;
  int64_t bad = -1;
  for (int t = 0; t < nth; ++t) {
    if (part_bad[t] >= 0 && bad < 0) bad = part_bad[t];
    amax = std::max(amax, part_max[t]);
  }
  return scan_verdict(r, amax, bad);
}

// bad >= 0: the first non-finite vertex
static zh_status scan_verdict(const zh_raster* r, double amax, int64_t bad) {
  if (bad >= 0) return fail(ZH_ERR_INVALID_ARG, "non-finite vertex %lld", (long long)bad);
  amax = std::max(amax, std::max(fabs(r->gt[0]), fabs(r->gt[3])));
  amax = std::max(amax, std::max(fabs(r->gt[0] + (double)r->cols * r->gt[1]), fabs(r->gt[3] + (double)r->rows * r->gt[5])));
  // The classification proof and the quick left/right edge tests need the cell size to dwarf the
  // rounding of coordinates: |gt1|, |gt5| >= 2^-30 * max |coordinate|.
  const double lim = ldexp(amax, -30);
  if (fabs(r->gt[1]) < lim || fabs(r->gt[5]) < lim)
    return fail(ZH_ERR_UNSUPPORTED, "cell size too small relative to the coordinate magnitude");
  return ZH_OK;
}

#if defined(ZH_DESTROY_TRACE) || defined(ZH_CREATE_TRACE)
#include <chrono>
static double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
#endif
#ifdef ZH_DESTROY_TRACE
#define ZH_TR(label) fprintf(stderr, "zh_destroy %-10s %8.3f ms\n", label, now_ms() - t_tr), t_tr = now_ms()
#else
#define ZH_TR(label) (void)0
#endif
#ifdef ZH_CREATE_TRACE
#define ZH_TRC(label) fprintf(stderr, "zh_create %-10s %8.3f ms\n", label, now_ms() - t_tr), t_tr = now_ms()
#else
#define ZH_TRC(label) (void)0
#endif

extern "C" zh_status zh_create(zh_ctx* out, const zh_raster* r, const zh_polygons* p, const zh_bins* b,
                               const zh_options* o) {
  ZH_RANGE("zh_create");
  if (!out) return fail(ZH_ERR_INVALID_ARG, "out is NULL");
#ifdef ZH_CREATE_TRACE
  double t_tr = now_ms();
#endif
  zh_status st = validate(r, p, b, o);
  if (st != ZH_OK) return st;
  const bool scan_during_h2d = p->n_vert >= (1 << 20);
  if (!scan_during_h2d && (st = scan_vertices(r, p)) != ZH_OK) return st;
  ZH_TRC("validate");
  const int64_t T = o->tile;
  const int64_t TC = (r->cols + T - 1) / T;
  const int64_t tr0 = r->row0 / T;
  const int64_t TRn = (r->nrows + T - 1) / T;
  const int64_t n_tiles = TC * TRn;
  if (n_tiles >= (1ll << 31) || TC >= (1ll << 31)) return fail(ZH_ERR_UNSUPPORTED, "more than 2^31 tiles");
  if (TC > (1ll << 20)) return fail(ZH_ERR_UNSUPPORTED, "more than 2^20 tile columns (step 2's row bitmaps)");
  if (!o->out_u64) {
    // uint32 output: a polygon's count is bounded by the cells of its MBB
    for (int64_t k = 0; k < p->n_poly; ++k) {
      int64_t vb = p->ring_vert_off[p->poly_ring_off[k]], ve = p->ring_vert_off[p->poly_ring_off[k + 1]];
      if (ve <= vb) continue;
      double xmn = INFINITY, xmx = -INFINITY, ymn = INFINITY, ymx = -INFINITY;
      for (int64_t i = vb; i < ve; ++i) {
        xmn = std::min(xmn, p->x[i]); xmx = std::max(xmx, p->x[i]);
        ymn = std::min(ymn, p->y[i]); ymx = std::max(ymx, p->y[i]);
      }
      double wc = std::min((xmx - xmn) / fabs(r->gt[1]) + 3.0, (double)r->cols);
      double hc = std::min((ymx - ymn) / fabs(r->gt[5]) + 3.0, (double)r->nrows);
      if (wc * hc >= 4294967295.0)
        return fail(ZH_ERR_OVERFLOW, "polygon %lld may hold >= 2^32 cells; use out_u64 = 1", (long long)k);
    }
  }

  Ctx* c = new (std::nothrow) Ctx();
  if (!c) return fail(ZH_ERR_OOM, "host allocation failed");
  c->rp.data = r->data;
  c->rp.rows = r->rows;
  c->rp.cols = r->cols;
  c->rp.pitch = r->pitch;
  c->rp.row0 = r->row0;
  c->rp.nrows = r->nrows;
  c->rp.T = (int32_t)T;
  c->rp.TC = (int32_t)TC;
  c->rp.tr0 = (int32_t)tr0;
  c->rp.TRn = (int32_t)TRn;
  zh::set_tc_div(c->rp);
  c->rp.wide = ((uintptr_t)c->rp.data % 32 == 0 && c->rp.pitch % 16 == 0) ? 1 : 0;
  c->geo = zh::Geo{r->gt[0], r->gt[1], r->gt[3], r->gt[5], o->rep_custom ? o->rep_x : 0.5,
                   o->rep_custom ? o->rep_y : 0.5, 1.0 / r->gt[1], 1.0 / r->gt[5]};
  c->on_host = r->on_host != 0;
  c->host_data = r->on_host ? r->data : nullptr;
  c->bp = zh::BinP{b->lo, b->width, b->nbins, b->use_nodata ? 1 : 0, b->nodata, b->oor_drop ? 1 : 0};
  c->B_pad = (b->nbins + 3) & ~3;
  c->out_u64 = o->out_u64 ? 1 : 0;
  c->force_isect = o->force_isect ? 1 : 0;
  c->cover = o->cover ? 1 : 0;
  c->fused = o->fused ? 1 : 0;
  c->stream = (cudaStream_t)o->stream;
  c->n_tiles = n_tiles;
  c->P = (int32_t)p->n_poly;
  c->R = (int32_t)p->n_ring;
  c->V = (int32_t)p->n_vert;

  auto cleanup_fail = [&](zh_status s) {
    zh_destroy(reinterpret_cast<zh_ctx>(c));
    return s;
  };
  cudaError_t e;
  ZH_TRC("setup");
  // polygons: int32 offsets + coordinates, copied H2D on the stream
  std::vector<int32_t> pro(p->n_poly + 1), rvo(p->n_ring + 1);
  for (int64_t i = 0; i <= p->n_poly; ++i) pro[i] = (int32_t)p->poly_ring_off[i];
  for (int64_t i = 0; i <= p->n_ring; ++i) rvo[i] = (int32_t)p->ring_vert_off[i];
  if ((e = c->d_pro.ensure(pro.size() * 4)) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create"));
  if ((e = c->d_rvo.ensure(rvo.size() * 4)) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create"));
  if ((e = c->d_x.ensure((size_t)p->n_vert * 8)) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create"));
  if ((e = c->d_y.ensure((size_t)p->n_vert * 8)) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create"));
  if ((e = cudaMemcpyAsync(c->d_pro.p, pro.data(), pro.size() * 4, cudaMemcpyHostToDevice, c->stream)) ||
      (e = cudaMemcpyAsync(c->d_rvo.p, rvo.data(), rvo.size() * 4, cudaMemcpyHostToDevice, c->stream)))
    return cleanup_fail(cuda_fail(e, "zh_create (polygon offsets H2D)"));
  if (p->n_vert > 0) {
    if ((e = cudaMemcpyAsync(c->d_x.p, p->x, (size_t)p->n_vert * 8, cudaMemcpyHostToDevice, c->stream)) ||
        (e = cudaMemcpyAsync(c->d_y.p, p->y, (size_t)p->n_vert * 8, cudaMemcpyHostToDevice, c->stream)))
      return cleanup_fail(cuda_fail(e, "zh_create (vertices H2D)"));
  }
#if ZH_DEVICE_SCAN
  if (scan_during_h2d) {  // on the device behind the copies; checked after the closing sync
    if ((e = c->d_scan.ensure(16)) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create (scan)"));
    const unsigned long long init[2] = {0ull, 0x7FFFFFFFFFFFFFFFull};
    if ((e = cudaMemcpyAsync(c->d_scan.p, init, sizeof(init), cudaMemcpyHostToDevice, c->stream)) != cudaSuccess)
      return cleanup_fail(cuda_fail(e, "zh_create (scan)"));
    k_scan_vertices<<<148 * 8, 256, 0, c->stream>>>(c->d_x.as<double>(), c->d_y.as<double>(), p->n_vert,
                                                     c->d_scan.as<unsigned long long>());
    c->launches += 1;
  }
#else
  if (scan_during_h2d && (st = scan_vertices(r, p)) != ZH_OK) return cleanup_fail(st);
#endif
  // output (the per-tile histograms of step 1 are allocated by the first zh_tile_hist)
  const size_t out_bytes = (size_t)p->n_poly * b->nbins * (c->out_u64 ? 8 : 4);
  if ((e = c->d_out_own.ensure(out_bytes)) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create (output)"));
  c->d_out = c->d_out_own.p;
  if ((e = cudaMemsetAsync(c->d_out, 0, out_bytes, c->stream)) != cudaSuccess)
    return cleanup_fail(cuda_fail(e, "zh_create"));
  ZH_TRC("h2d+out");
  if (c->on_host) {
    if ((e = c->raster_dev.ensure((size_t)std::max<int64_t>(r->nrows, 1) * r->pitch * 2 + 16)) != cudaSuccess)
      return cleanup_fail(cuda_fail(e, "zh_create (device raster copy)"));
    c->rp.data = c->raster_dev.as<int16_t>();
    if (r->pitch % 8 != 0) return cleanup_fail(fail(ZH_ERR_INVALID_ARG, "host raster pitch must be a multiple of 8"));
  }
  if ((e = pinned_alloc((void**)&c->pinned_counts, &c->pinned_counts_bytes, 16 * sizeof(int64_t))) != cudaSuccess)
    return cleanup_fail(cuda_fail(e, "zh_create (pinned counters)"));
  if ((e = c->d_flag.ensure(16)) != cudaSuccess || (e = cudaMemsetAsync(c->d_flag.p, 0, 16, c->stream)) != cudaSuccess)
    return cleanup_fail(cuda_fail(e, "zh_create (check flag)"));
  for (int i = 0; i < 16; ++i)
    if ((e = cudaEventCreate(&c->ev[i])) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create (events)"));
  if ((e = cudaStreamCreateWithFlags(&c->side, cudaStreamNonBlocking)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_counts, cudaEventDisableTiming)) != cudaSuccess)
    return cleanup_fail(cuda_fail(e, "zh_create (side stream)"));
  if ((e = cudaGetLastError()) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create"));
  // the polygon arrays are the caller's (zh.h: they may be freed or reused once zh_create
  // returns); with page-locked host arrays the copies above are truly asynchronous
  ZH_TRC("enqueue");
#if ZH_DEVICE_SCAN
  if (scan_during_h2d &&
      (e = cudaMemcpyAsync(c->pinned_counts, c->d_scan.p, 16, cudaMemcpyDeviceToHost, c->stream)) != cudaSuccess)
    return cleanup_fail(cuda_fail(e, "zh_create (scan)"));
#endif
  if ((e = cudaStreamSynchronize(c->stream)) != cudaSuccess) return cleanup_fail(cuda_fail(e, "zh_create (H2D)"));
  ZH_TRC("sync");
#if ZH_DEVICE_SCAN
  if (scan_during_h2d) {
    const uint64_t* sc = reinterpret_cast<const uint64_t*>(c->pinned_counts);
    double amax;
    memcpy(&amax, &sc[0], 8);
    const int64_t bad = sc[1] == 0x7FFFFFFFFFFFFFFFull ? -1 : (int64_t)sc[1];
    if ((st = scan_verdict(r, amax, bad)) != ZH_OK) return cleanup_fail(st);
  }
#endif
  *out = reinterpret_cast<zh_ctx>(c);
  return ZH_OK;
}

extern "C" void zh_destroy(zh_ctx h) {
  if (!h) return;
  Ctx* c = C(h);
#ifdef ZH_DESTROY_TRACE
  double t_tr = now_ms();
#endif
  cudaStreamSynchronize(c->stream);
  ZH_TR("sync");
  if (c->side) cudaStreamSynchronize(c->side);  // the blocks go back to the cache: nothing may still use them
  zh::DBuf* bufs[] = {&c->raster_dev, &c->d_pro, &c->d_rvo, &c->d_x, &c->d_y, &c->d_edges, &c->d_erows,
                      &c->d_mbb, &c->d_ncand, &c->d_nband, &c->d_cand_off,
                      &c->d_band_base, &c->d_band_cnt, &c->d_band_off, &c->d_band_cur, &c->d_band_edges,
                      &c->d_class, &c->d_flags, &c->d_flag_pos, &c->d_inside, &c->d_isect, &c->d_counts,
                      &c->d_cub, &c->d_tile_hist, &c->d_out_own, &c->d_mixed, &c->d_pure_cnt,
                      &c->d_pure_cur, &c->d_pure_pk, &c->d_pure_off, &c->d_pure_poly, &c->d_pure_tiles,
                      &c->d_extra, &c->d_extra_pos, &c->d_pip, &c->d_pip_cur, &c->d_pbits, &c->d_remap, &c->d_fcounts, &c->d_stats,
                      &c->d_pip_grp, &c->d_mixed_pk, &c->d_band_poly, &c->d_band_first, &c->d_scan, &c->d_flag, &c->d_need, &c->d_summary, &c->d_cdf, &c->d_dist, &c->d_ids};
  for (auto* b : bufs) b->release();
  ZH_TR("release");
  for (int i = 0; i < 16; ++i)
    if (c->ev[i]) cudaEventDestroy(c->ev[i]);
  ZH_TR("events");
  if (c->side) {
    cudaStreamSynchronize(c->side);
    cudaStreamDestroy(c->side);
  }
  if (c->gexec) cudaGraphExecDestroy(c->gexec);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  if (c->ev_counts) cudaEventDestroy(c->ev_counts);
  ZH_TR("streams");
  pinned_free(c->pinned_counts, c->pinned_counts_bytes);
  pinned_free(c->pinned_need, c->pinned_need_bytes);
  ZH_TR("freehost");
  delete c;
}

size_t zh::device_bytes(const Ctx& c) {
  const zh::DBuf* bufs[] = {&c.raster_dev, &c.d_pro, &c.d_rvo, &c.d_x, &c.d_y, &c.d_edges, &c.d_erows,
                            &c.d_mbb, &c.d_ncand, &c.d_nband, &c.d_cand_off,
                            &c.d_band_base, &c.d_band_cnt, &c.d_band_off, &c.d_band_cur, &c.d_band_edges,
                            &c.d_class, &c.d_flags, &c.d_flag_pos, &c.d_inside, &c.d_isect, &c.d_counts,
                            &c.d_cub, &c.d_tile_hist, &c.d_out_own, &c.d_mixed, &c.d_pure_cnt,
                            &c.d_pure_cur, &c.d_pure_pk, &c.d_pure_off, &c.d_pure_poly, &c.d_pure_tiles,
                            &c.d_extra, &c.d_extra_pos, &c.d_pip, &c.d_pip_cur, &c.d_pbits, &c.d_remap, &c.d_fcounts, &c.d_stats,
                            &c.d_pip_grp, &c.d_mixed_pk, &c.d_band_poly, &c.d_band_first, &c.d_scan, &c.d_flag, &c.d_need, &c.d_summary, &c.d_cdf, &c.d_dist, &c.d_ids};
  size_t s = 0;
  for (auto* b : bufs) s += b->bytes;
  return s;
}

static void tic(Ctx* c, int step) {
  if (c->timing) zh::rec_event(*c, c->ev[2 * step], c->stream);
}
static void toc(Ctx* c, int step) {
  if (c->timing) zh::rec_event(*c, c->ev[2 * step + 1], c->stream);
}

// After a sync point: did a step's counts differ from the context's known sizes?  (Never, for a
// fixed geometry; the check guards the host-sync-free steps.)
static zh_status check_flag(Ctx* c, const char* who) {
  if (!c->d_flag.p) return ZH_OK;
  ZH_CU(cudaMemcpyAsync(c->pinned_counts + 15, c->d_flag.p, 4, cudaMemcpyDeviceToHost, c->stream), who);
  ZH_CU(cudaStreamSynchronize(c->stream), who);
  if (*reinterpret_cast<uint32_t*>(c->pinned_counts + 15) != 0u)
    return fail(ZH_ERR_STATE, "%s: a step's list sizes differ from the context's known sizes", who);
  return ZH_OK;
}

extern "C" zh_status zh_upload_raster(zh_ctx h) {
  ZH_RANGE("zh_upload_raster");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (!c->on_host) return ZH_OK;
  if (c->rp.nrows > 0)
    ZH_CU(cudaMemcpyAsync(c->raster_dev.p, c->host_data, (size_t)c->rp.nrows * c->rp.pitch * 2, cudaMemcpyHostToDevice,
                          c->stream),
          "zh_upload_raster");
  c->h2d_bytes = c->rp.nrows * c->rp.pitch * 2;
  return ZH_OK;
}

// on_host + fused zh_run: after step 2, copy only the tiles that some pair needs (pure or mixed
// tiles; the fused kernels never read the others), one 2-D copy per run of consecutive needed
// tiles of a tile row.  The bytes copied are reported as zh_stats.h2d_bytes.
static zh_status upload_needed(Ctx* c) {
  const int64_t NT = c->n_tiles, T = c->rp.T, TC = c->rp.TC;
  c->h2d_bytes = 0;
  if (NT == 0 || c->rp.nrows == 0) return ZH_OK;
  if (!c->pinned_need) ZH_CU(pinned_alloc((void**)&c->pinned_need, &c->pinned_need_bytes, (size_t)NT + 1), "zh_run");
  ZH_CU(zh::launch_need_tiles(*c), "zh_run (needed tiles)");
  ZH_CU(cudaMemcpyAsync(c->pinned_need, c->d_need.p, (size_t)NT, cudaMemcpyDeviceToHost, c->stream), "zh_run");
  ZH_CU(cudaStreamSynchronize(c->stream), "zh_run (needed tiles)");
  const size_t pitch_b = (size_t)c->rp.pitch * 2;
  const char* src = reinterpret_cast<const char*>(c->host_data);
  char* dst = reinterpret_cast<char*>(c->raster_dev.p);
  for (int64_t tr = 0; tr < c->rp.TRn; ++tr) {
    const int64_t lr0 = tr * T;  // shard-local first row
    const int64_t h = std::min<int64_t>(T, c->rp.nrows - lr0);
    const uint8_t* nd = c->pinned_need + tr * TC;
    for (int64_t a = 0; a < TC;) {
      if (!nd[a]) { ++a; continue; }
      int64_t b = a;
      while (b < TC && nd[b]) ++b;
      // columns [a T, b T) rounded out to whole 16-byte vectors (the kernels read 8-cell vectors)
      const int64_t c0 = (a * T) & ~7ll, c1 = std::min<int64_t>((b * T + 7) & ~7ll, c->rp.pitch);
      const size_t off = (size_t)lr0 * pitch_b + (size_t)c0 * 2, wb = (size_t)(c1 - c0) * 2;
      if (c0 == 0 && c1 == c->rp.pitch) {
        ZH_CU(cudaMemcpyAsync(dst + off, src + off, (size_t)h * pitch_b, cudaMemcpyHostToDevice, c->stream),
              "zh_run (upload)");
      } else {
        ZH_CU(cudaMemcpy2DAsync(dst + off, pitch_b, src + off, pitch_b, wb, (size_t)h, cudaMemcpyHostToDevice,
                                c->stream),
              "zh_run (upload)");
      }
      c->h2d_bytes += (int64_t)(wb * (size_t)h);
      a = b;
    }
  }
  return ZH_OK;
}

extern "C" zh_status zh_tile_hist(zh_ctx h) {
  ZH_RANGE("zh_tile_hist");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  ZH_CU(c->d_tile_hist.ensure((size_t)c->n_tiles * c->B_pad * 4), "zh_tile_hist (allocating tile histograms)");
  tic(c, 0);
  ZH_CU(zh::launch_tile_hist(*c), "zh_tile_hist");
  toc(c, 0);
  c->have_hist = true;
  return ZH_OK;
}

extern "C" zh_status zh_pair_tiles(zh_ctx h, int64_t* n_inside, int64_t* n_isect) {
  ZH_RANGE("zh_pair_tiles");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  c->have_pairs = false;
  c->step3_done = false;
  c->step4_done = false;
  c->fused_done = false;
  tic(c, 1);
  const size_t out_bytes = (size_t)c->P * c->bp.nbins * (c->out_u64 ? 8 : 4);
  ZH_CU(cudaMemsetAsync(c->d_out, 0, out_bytes, c->stream), "zh_pair_tiles (zero output)");
  ZH_CU(zh::launch_pairs_phase1(*c), "zh_pair_tiles (phase 1)");
  if (c->sizes_known) {
    // the sizes are those of the first call (fixed geometry): no host round trip; the device
    // checks the recomputed counts against them
    ZH_CU(zh::launch_pairs_phase2(*c), "zh_pair_tiles (phase 2)");
    const int64_t want[6] = {c->n_cand + c->n_cand_check_bias, c->n_bands, c->n_band_entries, 0, c->n_inside,
                             c->n_isect};
    ZH_CU(zh::launch_check_counts(*c, c->d_counts.as<int64_t>(), want, 3), "zh_pair_tiles (check)");
    ZH_CU(zh::launch_check_counts(*c, c->d_counts.as<int64_t>() + 4, want + 4, 2), "zh_pair_tiles (check)");
    toc(c, 1);
  } else {
    ZH_CU(cudaMemcpyAsync(c->pinned_counts, c->d_counts.p, 3 * sizeof(int64_t), cudaMemcpyDeviceToHost, c->stream),
          "zh_pair_tiles (counts)");
    ZH_CU(cudaStreamSynchronize(c->stream), "zh_pair_tiles (sync 1)");
    c->n_cand = c->pinned_counts[0];
    c->n_bands = c->pinned_counts[1];
    c->n_band_entries = c->pinned_counts[2];
    if (c->n_cand >= (1ll << 31) || c->n_bands >= (1ll << 31) || c->n_band_entries >= (1ll << 31) ||
        c->n_band_entries < 0)
      return fail(ZH_ERR_UNSUPPORTED, "pair lists exceed 2^31 entries");
    ZH_CU(zh::launch_pairs_phase2(*c), "zh_pair_tiles (phase 2)");
    ZH_CU(cudaMemcpyAsync(c->pinned_counts + 4, c->d_counts.as<int64_t>() + 4, 2 * sizeof(int64_t),
                          cudaMemcpyDeviceToHost, c->stream),
          "zh_pair_tiles (counts)");
    toc(c, 1);
    ZH_CU(cudaStreamSynchronize(c->stream), "zh_pair_tiles (sync 2)");
    c->n_inside = c->pinned_counts[4];
    c->n_isect = c->pinned_counts[5];
    c->sizes_known = true;
    // ZH_TEST_BAD_SIZES=1 (testing the guard): remember a wrong candidate count, so that the next
    // host-sync-free step's device check must flag it
    const char* bad = getenv("ZH_TEST_BAD_SIZES");
    if (bad && bad[0] == '1') c->bad_sizes_pending = true;
  }
  if (c->bad_sizes_pending && c->sizes_known) {
    c->bad_sizes_pending = false;
    c->n_cand_check_bias = 1;
  }
  c->have_pairs = true;
  if (n_inside) *n_inside = c->n_inside;
  if (n_isect) *n_isect = c->n_isect;
  return ZH_OK;
}

extern "C" zh_status zh_aggregate(zh_ctx h) {
  ZH_RANGE("zh_aggregate");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (!c->have_pairs || !c->have_hist) return fail(ZH_ERR_STATE, "zh_aggregate needs zh_tile_hist and zh_pair_tiles");
  if (c->step3_done) return fail(ZH_ERR_STATE, "zh_aggregate already applied since the last zh_pair_tiles");
  if (c->fused_done) return fail(ZH_ERR_STATE, "zh_fused_update already covered step 3");
  tic(c, 2);
  ZH_CU(zh::launch_aggregate(*c), "zh_aggregate");
  toc(c, 2);
  c->step3_done = true;
  return ZH_OK;
}

extern "C" zh_status zh_pip_update(zh_ctx h) {
  ZH_RANGE("zh_pip_update");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (!c->have_pairs) return fail(ZH_ERR_STATE, "zh_pip_update needs zh_pair_tiles");
  if (c->step4_done) return fail(ZH_ERR_STATE, "zh_pip_update already applied since the last zh_pair_tiles");
  if (c->fused_done) return fail(ZH_ERR_STATE, "zh_fused_update already covered step 4");
  tic(c, 3);
  ZH_CU(zh::launch_pip(*c), "zh_pip_update");
  toc(c, 3);
  c->step4_done = true;
  return ZH_OK;
}

extern "C" zh_status zh_fused_update(zh_ctx h) {
  ZH_RANGE("zh_fused_update");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (!c->have_pairs) return fail(ZH_ERR_STATE, "zh_fused_update needs zh_pair_tiles");
  if (c->step3_done || c->step4_done || c->fused_done)
    return fail(ZH_ERR_STATE, "steps 3/4 already applied since the last zh_pair_tiles");
  tic(c, 4);
  ZH_CU(zh::launch_fused(*c), "zh_fused_update");
  toc(c, 4);
  c->fused_done = true;
  return ZH_OK;
}

extern "C" zh_status zh_run(zh_ctx h, void* host_out) {
  ZH_RANGE("zh_run");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  zh_status s;
  // the fused path reads only tiles with a pair: on_host rasters are uploaded after step 2 (which
  // needs the polygons only), tile runs that some pair needs; the four-step path's step 1 reads
  // every tile, so the whole shard goes up first
  const bool needed_only = c->on_host && c->fused;
  if (!needed_only && (s = zh_upload_raster(h)) != ZH_OK) return s;
  if ((s = zh_pair_tiles(h, nullptr, nullptr)) != ZH_OK) return s;
  if (needed_only && (s = upload_needed(c)) != ZH_OK) return s;
  if (c->fused) {
    if ((s = zh_fused_update(h)) != ZH_OK) return s;
  } else {
    if ((s = zh_tile_hist(h)) != ZH_OK) return s;
    if ((s = zh_aggregate(h)) != ZH_OK) return s;
    if ((s = zh_pip_update(h)) != ZH_OK) return s;
  }
  if (host_out) {
    const size_t out_bytes = (size_t)c->P * c->bp.nbins * (c->out_u64 ? 8 : 4);
    ZH_CU(cudaMemcpyAsync(host_out, c->d_out, out_bytes, cudaMemcpyDeviceToHost, c->stream), "zh_run (D2H)");
  }
  ZH_CU(cudaStreamSynchronize(c->stream), "zh_run (sync)");
  return check_flag(c, "zh_run");
}

// The step's calls (no upload, no D2H) on c->stream.
static zh_status run_step_calls(zh_ctx h) {
  Ctx* c = C(h);
  zh_status s;
  if ((s = zh_pair_tiles(h, nullptr, nullptr)) != ZH_OK) return s;
  if (c->fused) return zh_fused_update(h);
  if ((s = zh_tile_hist(h)) != ZH_OK) return s;
  if ((s = zh_aggregate(h)) != ZH_OK) return s;
  return zh_pip_update(h);
}

extern "C" zh_status zh_step_graph(zh_ctx h) {
  ZH_RANGE("zh_step_graph");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (c->on_host && c->rp.nrows > 0 && c->h2d_bytes == 0)
    return fail(ZH_ERR_STATE, "zh_step_graph on a host raster needs zh_upload_raster (or a zh_run) first");
  // the first call runs the step directly: it learns the list sizes (host syncs)
  if (!c->sizes_known || (c->fused && !c->fused_known)) return run_step_calls(h);
  if (c->gexec && c->graph_fused != c->fused) {
    cudaGraphExecDestroy(c->gexec);
    c->gexec = nullptr;
  }
  if (!c->gexec) {
    // capture on the context's own non-blocking stream (the caller's stream may be the legacy
    // default stream, which cannot be captured); the launches below fork/join it to c->stream
    cudaStream_t user = c->stream;
    ZH_CU(cudaStreamBeginCapture(c->side, cudaStreamCaptureModeThreadLocal), "zh_step_graph (capture)");
    c->stream = c->side;
    c->capturing = true;
    const int64_t before = c->launches;
    const zh_status st = run_step_calls(h);
    c->graph_kernels = c->launches - before;  // kernel nodes of the graph (recorded, not launched)
    c->launches = before;
    c->stream = user;
    c->capturing = false;
    cudaGraph_t g = nullptr;
    const cudaError_t e = cudaStreamEndCapture(c->side, &g);
    if (st != ZH_OK) {
      if (g) cudaGraphDestroy(g);
      return st;
    }
    if (e != cudaSuccess) return cuda_fail(e, "zh_step_graph (end capture)");
    const cudaError_t ei = cudaGraphInstantiate(&c->gexec, g, 0);
    cudaGraphDestroy(g);
    if (ei != cudaSuccess) {
      c->gexec = nullptr;
      return cuda_fail(ei, "zh_step_graph (instantiate)");
    }
    c->graph_fused = c->fused;
  }
  ZH_CU(cudaEventRecord(c->ev_fork, c->stream), "zh_step_graph");
  ZH_CU(cudaStreamWaitEvent(c->side, c->ev_fork, 0), "zh_step_graph");
  ZH_CU(cudaGraphLaunch(c->gexec, c->side), "zh_step_graph (launch)");
  ZH_CU(cudaEventRecord(c->ev_join, c->side), "zh_step_graph");
  ZH_CU(cudaStreamWaitEvent(c->stream, c->ev_join, 0), "zh_step_graph");
  c->launches += c->graph_kernels;
  c->have_pairs = true;
  if (c->fused) {
    c->fused_done = true;
  } else {
    c->have_hist = true;
    c->step3_done = c->step4_done = true;
  }
  return ZH_OK;
}

extern "C" zh_status zh_zonal_stats(zh_ctx h, int64_t* host_stats, int64_t** dptr) {
  ZH_RANGE("zh_zonal_stats");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (!c->have_pairs || !(c->fused_done || (c->step3_done && c->step4_done)))
    return fail(ZH_ERR_STATE, "zh_zonal_stats needs a completed histogram (zh_run, steps 2 + 3 + 4, or the fused update)");
  ZH_CU(c->d_stats.ensure((size_t)(c->P > 0 ? c->P : 1) * ZH_NSTATS * sizeof(int64_t)), "zh_zonal_stats");
  ZH_CU(zh::launch_zonal_stats(*c, c->d_stats.as<int64_t>()), "zh_zonal_stats");
  if (dptr) *dptr = c->d_stats.as<int64_t>();
  if (host_stats && c->P > 0) {
    ZH_CU(cudaMemcpyAsync(host_stats, c->d_stats.p, (size_t)c->P * ZH_NSTATS * sizeof(int64_t),
                          cudaMemcpyDeviceToHost, c->stream),
          "zh_zonal_stats (D2H)");
    ZH_CU(cudaStreamSynchronize(c->stream), "zh_zonal_stats");
  }
  return ZH_OK;
}

// Exact statistics of the current histogram into c->d_stats (a completed histogram required).
static zh_status stats_on_device(Ctx* c, const char* who) {
  if (!c->have_pairs || !(c->fused_done || (c->step3_done && c->step4_done)))
    return fail(ZH_ERR_STATE, "%s needs a completed histogram (zh_run, steps 2 + 3 + 4, or the fused update)", who);
  ZH_CU(c->d_stats.ensure((size_t)(c->P > 0 ? c->P : 1) * ZH_NSTATS * sizeof(int64_t)), who);
  ZH_CU(zh::launch_zonal_stats(*c, c->d_stats.as<int64_t>()), who);
  return ZH_OK;
}

extern "C" zh_status zh_zonal_summary(zh_ctx h, double* host_out, double** dptr) {
  ZH_RANGE("zh_zonal_summary");
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  zh_status s = stats_on_device(c, "zh_zonal_summary");
  if (s != ZH_OK) return s;
  ZH_CU(c->d_summary.ensure((size_t)(c->P > 0 ? c->P : 1) * ZH_NSUMMARY * sizeof(double)), "zh_zonal_summary");
  ZH_CU(zh::launch_zonal_summary(*c, c->d_stats.as<int64_t>(), c->d_summary.as<double>()), "zh_zonal_summary");
  if (dptr) *dptr = c->d_summary.as<double>();
  if (host_out && c->P > 0) {
    ZH_CU(cudaMemcpyAsync(host_out, c->d_summary.p, (size_t)c->P * ZH_NSUMMARY * sizeof(double),
                          cudaMemcpyDeviceToHost, c->stream),
          "zh_zonal_summary (D2H)");
    ZH_CU(cudaStreamSynchronize(c->stream), "zh_zonal_summary");
  }
  return ZH_OK;
}

extern "C" zh_status zh_hist_distance(zh_ctx h, int32_t kind, const int32_t* a_ids, const int32_t* b_ids, int64_t n,
                                      double* host_out) {
  ZH_RANGE("zh_hist_distance");
  if (!h || !host_out) return fail(ZH_ERR_INVALID_ARG, "null argument");
  Ctx* c = C(h);
  if (kind != ZH_DIST_L1 && kind != ZH_DIST_EMD && kind != ZH_DIST_CHI2)
    return fail(ZH_ERR_INVALID_ARG, "unknown distance kind %d", (int)kind);
  if ((a_ids == nullptr) != (b_ids == nullptr))
    return fail(ZH_ERR_INVALID_ARG, "a_ids and b_ids must both be given or both be NULL");
  const bool all = a_ids == nullptr;
  if (!all) {
    if (n < 0 || n >= (1ll << 31)) return fail(ZH_ERR_INVALID_ARG, "n must be in [0, 2^31)");
    for (int64_t i = 0; i < n; ++i)
      if (a_ids[i] < 0 || a_ids[i] >= c->P || b_ids[i] < 0 || b_ids[i] >= c->P)
        return fail(ZH_ERR_INVALID_ARG, "polygon id out of range at %lld", (long long)i);
  } else if ((int64_t)c->P * c->P >= (1ll << 40)) {
    return fail(ZH_ERR_UNSUPPORTED, "all-pairs matrix too large");
  }
  zh_status s = stats_on_device(c, "zh_hist_distance");
  if (s != ZH_OK) return s;
  // 32 x 32 -> 64-bit products when every count (and so every bin and running sum) is < 2^32
  std::vector<int64_t> st((size_t)std::max(c->P, 1) * ZH_NSTATS);
  if (c->P > 0) {
    ZH_CU(cudaMemcpyAsync(st.data(), c->d_stats.p, st.size() * 8, cudaMemcpyDeviceToHost, c->stream), "zh_hist_distance");
    ZH_CU(cudaStreamSynchronize(c->stream), "zh_hist_distance");
  }
  // ZH_DIST_WIDE=1 (testing): the general 64 x 64 -> 128-bit products even when narrow would do
  const char* wide_env = getenv("ZH_DIST_WIDE");
  bool narrow = !(wide_env && wide_env[0] == '1');
  for (int32_t k = 0; k < c->P; ++k)
    if ((uint64_t)st[(size_t)k * ZH_NSTATS] >= (1ull << 32)) narrow = false;
  const int64_t n_out = all ? (int64_t)c->P * c->P : n;
  ZH_CU(c->d_dist.ensure((size_t)std::max<int64_t>(n_out, 1) * sizeof(double)), "zh_hist_distance");
  const int32_t *ia = nullptr, *ib = nullptr;
  if (!all) {
    ZH_CU(c->d_ids.ensure((size_t)std::max<int64_t>(n, 1) * 2 * sizeof(int32_t)), "zh_hist_distance");
    if (n > 0) {
      ZH_CU(cudaMemcpyAsync(c->d_ids.p, a_ids, (size_t)n * 4, cudaMemcpyHostToDevice, c->stream), "zh_hist_distance");
      ZH_CU(cudaMemcpyAsync(c->d_ids.as<int32_t>() + n, b_ids, (size_t)n * 4, cudaMemcpyHostToDevice, c->stream),
            "zh_hist_distance");
    }
    ia = c->d_ids.as<int32_t>();
    ib = ia + n;
  }
  ZH_CU(zh::launch_hist_distance(*c, kind, c->d_stats.as<int64_t>(), narrow, ia, ib, all ? 0 : n,
                                 c->d_dist.as<double>()),
        "zh_hist_distance");
  if (n_out > 0)
    ZH_CU(cudaMemcpyAsync(host_out, c->d_dist.p, (size_t)n_out * sizeof(double), cudaMemcpyDeviceToHost, c->stream),
          "zh_hist_distance (D2H)");
  ZH_CU(cudaStreamSynchronize(c->stream), "zh_hist_distance");
  return ZH_OK;
}

extern "C" zh_status zh_plan_rows(const zh_raster* r, const zh_polygons* p, const zh_options* o, int32_t n_shards,
                                  int64_t* row_bounds, double* shard_cost) {
  ZH_RANGE("zh_plan_rows");
  if (!r || !p || !o || !row_bounds) return fail(ZH_ERR_INVALID_ARG, "null argument");
  if (n_shards < 1) return fail(ZH_ERR_INVALID_ARG, "n_shards must be >= 1");
  // Geometry only: the raster values are never read by step 2, so a placeholder pointer stands in
  // for the data and a single bin for the histograms.
  zh_raster g = *r;
  g.row0 = 0;
  g.nrows = r->rows;
  g.on_host = 0;
  g.pitch = (r->cols + 7) / 8 * 8;
  g.data = reinterpret_cast<const int16_t*>(static_cast<uintptr_t>(256));
  zh_bins b1 = {0, 1, 1, 0, 0, 0};
  zh_options go = *o;
  go.out_u64 = 1;
  go.force_isect = 0;
  go.fused = 0;
  zh_ctx h = nullptr;
  zh_status s = zh_create(&h, &g, p, &b1, &go);
  if (s != ZH_OK) return s;
  Ctx* c = C(h);
  const int64_t TR = c->rp.TRn;
  std::vector<double> cost(TR > 0 ? TR : 1, 0.0);
  s = zh_pair_tiles(h, nullptr, nullptr);
  if (s == ZH_OK) {
    zh::DBuf d;
    cudaError_t e = d.ensure(sizeof(double) * (size_t)(TR > 0 ? TR : 1));
    if (e == cudaSuccess) e = zh::launch_row_cost(*c, d.as<double>());
    if (e == cudaSuccess && TR > 0)
      e = cudaMemcpyAsync(cost.data(), d.p, sizeof(double) * (size_t)TR, cudaMemcpyDeviceToHost, c->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
    d.release();
    if (e != cudaSuccess) s = cuda_fail(e, "zh_plan_rows");
  }
  zh_destroy(h);
  if (s != ZH_OK) return s;
  // contiguous split of the tile rows at equal prefix cost; a small per-row floor keeps empty rows
  // (ocean) from collapsing all of them into one shard
  const int64_t T = o->tile;
  double total = 0.0;
  for (int64_t i = 0; i < TR; ++i) total += cost[i];
  const double floor_cost = total > 0 ? 1e-3 * total / (double)TR : 1.0;
  for (int64_t i = 0; i < TR; ++i) cost[i] += floor_cost;
  total += floor_cost * (double)TR;
  row_bounds[0] = 0;
  double run = 0.0;
  int64_t tr = 0;
  for (int i = 1; i < n_shards; ++i) {
    const double target = total * (double)i / (double)n_shards;
    while (tr < TR && run + cost[tr] * 0.5 < target) run += cost[tr++];
    row_bounds[i] = std::min(tr * T, r->rows);
  }
  row_bounds[n_shards] = r->rows;
  if (shard_cost) {
    for (int i = 0; i < n_shards; ++i) {
      double sc = 0.0;
      for (int64_t t = row_bounds[i] / T; t < (row_bounds[i + 1] + T - 1) / T && t < TR; ++t) sc += cost[t];
      shard_cost[i] = sc;
    }
  }
  return ZH_OK;
}

extern "C" zh_status zh_output_device(zh_ctx h, void** dptr, int64_t* n) {
  if (!h || !dptr) return fail(ZH_ERR_INVALID_ARG, "null argument");
  Ctx* c = C(h);
  *dptr = c->d_out;
  if (n) *n = (int64_t)c->P * c->bp.nbins;
  return ZH_OK;
}

extern "C" zh_status zh_set_output(zh_ctx h, void* dptr) {
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (dptr && ((uintptr_t)dptr & 7u)) return fail(ZH_ERR_INVALID_ARG, "output buffer must be 8-byte aligned");
  c->d_out = dptr ? dptr : c->d_out_own.p;
  if (c->gexec) {  // the captured step writes the old buffer
    cudaGraphExecDestroy(c->gexec);
    c->gexec = nullptr;
  }
  c->have_pairs = false;  // the new buffer must be zeroed by zh_pair_tiles before accumulation
  c->have_hist = c->have_hist;
  return ZH_OK;
}

extern "C" zh_status zh_copy_tile_hist(zh_ctx h, uint32_t* host, int64_t n_elems) {
  if (!h || !host) return fail(ZH_ERR_INVALID_ARG, "null argument");
  Ctx* c = C(h);
  if (n_elems < c->n_tiles * c->bp.nbins) return fail(ZH_ERR_INVALID_ARG, "host buffer too small");
  if (!c->have_hist) return fail(ZH_ERR_STATE, "zh_copy_tile_hist needs zh_tile_hist");
  if (c->n_tiles == 0) return ZH_OK;
  ZH_CU(cudaMemcpy2DAsync(host, (size_t)c->bp.nbins * 4, c->d_tile_hist.p, (size_t)c->B_pad * 4,
                          (size_t)c->bp.nbins * 4, (size_t)c->n_tiles, cudaMemcpyDeviceToHost, c->stream),
        "zh_copy_tile_hist");
  ZH_CU(cudaStreamSynchronize(c->stream), "zh_copy_tile_hist");
  return ZH_OK;
}

extern "C" zh_status zh_copy_pairs(zh_ctx h, int32_t* inside, int32_t* isect) {
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (!c->have_pairs) return fail(ZH_ERR_STATE, "zh_copy_pairs needs zh_pair_tiles");
  if (inside && c->n_inside)
    ZH_CU(cudaMemcpyAsync(inside, c->d_inside.p, (size_t)c->n_inside * 8, cudaMemcpyDeviceToHost, c->stream),
          "zh_copy_pairs");
  if (isect && c->n_isect)
    ZH_CU(cudaMemcpyAsync(isect, c->d_isect.p, (size_t)c->n_isect * 8, cudaMemcpyDeviceToHost, c->stream),
          "zh_copy_pairs");
  ZH_CU(cudaStreamSynchronize(c->stream), "zh_copy_pairs");
  return ZH_OK;
}

extern "C" zh_status zh_get_stats(zh_ctx h, zh_stats* s) {
  if (!h || !s) return fail(ZH_ERR_INVALID_ARG, "null argument");
  Ctx* c = C(h);
  s->n_tiles = c->n_tiles;
  s->n_candidates = c->n_cand;
  s->n_inside = c->n_inside;
  s->n_isect = c->n_isect;
  s->n_band_entries = c->n_band_entries;
  s->n_edges = c->V;
  s->device_bytes = (int64_t)zh::device_bytes(*c);
  s->h2d_bytes = c->h2d_bytes;
  s->n_pure_tiles = s->n_pip_pairs = s->n_pure_cells = s->n_pip_cells = s->n_mixed_groups = s->n_group_cells = 0;
  s->n_mixed_cells = 0;
  zh_status fs = check_flag(c, "zh_get_stats");
  if (fs != ZH_OK) return fs;
  if (c->fused_done) {
    ZH_CU(cudaMemcpyAsync(c->pinned_counts, c->d_fcounts.p, 7 * sizeof(int64_t), cudaMemcpyDeviceToHost, c->stream),
          "zh_get_stats");
    ZH_CU(cudaStreamSynchronize(c->stream), "zh_get_stats");
    s->n_pure_tiles = c->pinned_counts[0];
    s->n_pip_pairs = c->pinned_counts[1];
    s->n_pure_cells = c->pinned_counts[2];
    s->n_pip_cells = c->pinned_counts[3];
    s->n_mixed_groups = c->pinned_counts[4];
    s->n_group_cells = c->pinned_counts[5];
    s->n_mixed_cells = c->pinned_counts[6];
  }
  return ZH_OK;
}

extern "C" zh_status zh_set_timing(zh_ctx h, int32_t enable) {
  if (!h) return fail(ZH_ERR_INVALID_ARG, "null context");
  Ctx* c = C(h);
  if (c->gexec && c->timing != (enable != 0)) {  // the captured step records (or not) the events
    cudaGraphExecDestroy(c->gexec);
    c->gexec = nullptr;
  }
  c->timing = enable != 0;
  return ZH_OK;
}

extern "C" zh_status zh_get_step_ms(zh_ctx h, float* ms, int32_t n) {
  if (!h || !ms) return fail(ZH_ERR_INVALID_ARG, "null argument");
  Ctx* c = C(h);
  if (!c->timing) return fail(ZH_ERR_STATE, "timing is disabled");
  {
    zh_status fs = check_flag(c, "zh_get_step_ms");
    if (fs != ZH_OK) return fs;
  }
  // (start, stop) event pairs: steps 1..4, fused, fused pure-tile kernel, fused cell-in-polygon
  // (cell) kernel, fused parity kernel (second stream, overlapping the pure-tile kernel)
  const int pairs[8][2] = {{0, 1}, {2, 3}, {4, 5}, {6, 7}, {8, 9}, {10, 11}, {15, 12}, {13, 14}};
  for (int i = 0; i < n && i < 8; ++i) {
    float v = 0.f;
    if (cudaEventElapsedTime(&v, c->ev[pairs[i][0]], c->ev[pairs[i][1]]) != cudaSuccess) {
      cudaGetLastError();
      v = -1.f;
    }
    ms[i] = v;
  }
  return ZH_OK;
}

extern "C" int64_t zh_launch_count(zh_ctx h) { return h ? C(h)->launches : 0; }
