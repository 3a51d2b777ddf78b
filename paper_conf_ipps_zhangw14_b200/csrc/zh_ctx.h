// zh_ctx.h — host-side context of libzh and the launchers of its kernels (internal).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "zh_internal.cuh"

#ifndef ZH_PIP_GROUP_DEFAULT
#define ZH_PIP_GROUP_DEFAULT 1
#endif

namespace zh {

// Process-wide cache of device blocks (zh_api.cu), like PyTorch's caching allocator: a context's
// buffers go back to the cache when it is destroyed (after its streams are synchronised) and the
// next context of the same device reuses them, so a zh_create / zh_run / zh_destroy cycle does not
// pay cudaMalloc + cudaFree of a 40 GB raster copy every time.  zh_trim_cache() frees the cache.
cudaError_t cache_alloc(void** p, size_t* got, size_t need);
void cache_free(void* p, size_t bytes);

// Grow-only device buffer owned by the context.
struct DBuf {
  void* p = nullptr;
  size_t bytes = 0;
  cudaError_t ensure(size_t need) {
    if (need <= bytes && p) return cudaSuccess;
    if (p) cudaFree(p);  // growth: cudaFree waits for the work already enqueued on the old block
    p = nullptr;
    bytes = 0;
    if (need == 0) need = 16;
    return cache_alloc(&p, &bytes, need);
  }
  void release() {  // callers have synchronised every stream that used the block
    if (p) cache_free(p, bytes);
    p = nullptr;
    bytes = 0;
  }
  template <class T>
  T* as() const { return reinterpret_cast<T*>(p); }
};

struct Ctx {
  // raster shard
  RasterP rp;
  Geo geo;
  const int16_t* host_data = nullptr;  // on_host rasters: borrowed host pointer
  bool on_host = false;
  DBuf raster_dev;                     // on_host rasters: device copy of the shard
  // bins / options
  BinP bp;
  int32_t B_pad = 0;
  int32_t out_u64 = 1;
  int32_t force_isect = 0;
  int32_t cover = 0;  // R15: closed cell rectangle meets the closed polygon (k_touch.cu)
  int32_t pip_group = ZH_PIP_GROUP_DEFAULT;  // fused path: mixed-tile groups of <= 2 pairs (k_mixed_cells) or one CTA per pair
  cudaStream_t stream = nullptr;
  // polygons (device)
  int32_t P = 0, R = 0, V = 0;
  DBuf d_pro, d_rvo, d_x, d_y;
  // step 2 products
  DBuf d_edges, d_erows, d_mbb, d_ncand, d_nband, d_cand_off, d_band_base;
  DBuf d_band_cnt, d_band_off, d_band_cur, d_band_edges, d_class, d_flags, d_flag_pos;
  DBuf d_inside, d_isect, d_counts, d_cub;
  DBuf d_band_poly;  // band -> polygon
  DBuf d_scan;  // zh_create: device vertex scan (max |coordinate| bits, first non-finite vertex)
  DBuf d_band_first;  // band -> #edges straddling its first row (at the front of its list), -1: unsorted
  // fused path lists (k_fused.cu)
  DBuf d_mixed, d_pure_cnt, d_pure_cur, d_pure_pk, d_pure_off, d_pure_poly, d_pure_tiles, d_extra, d_extra_pos,
      d_pip, d_pip_cur, d_fcounts, d_pbits, d_remap, d_pip_grp, d_mixed_pk;
  DBuf d_stats;  // zonal statistics [P][8] (k_stats.cu)
  DBuf d_summary, d_cdf, d_dist, d_ids;  // zonal summary [P][6], row CDFs, distances, pair ids (k_features.cu)
  int64_t n_cand = 0, n_bands = 0, n_band_entries = 0, n_inside = 0, n_isect = 0;
  // step 1 product and output
  DBuf d_tile_hist;
  DBuf d_out_own;
  void* d_out = nullptr;  // own or borrowed
  int64_t n_tiles = 0;
  // state
  bool have_hist = false, have_pairs = false, step3_done = false, step4_done = false, fused_done = false;
  int32_t fused = 0;
  // timing
  bool timing = false;
  cudaEvent_t ev[16] = {};  // start/stop per timed call: steps 1..4, fused; + fused inner marks 10..15
  cudaStream_t side = nullptr;            // second stream of the fused path (k_parity beside k_fused_pure)
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  cudaEvent_t ev_counts = nullptr;        // fused path: list sizes copied to pinned_counts[8..13]
  int64_t fused_counts[4] = {0, 0, 0, 0};  // pure tiles, pip pairs, pure cells, pip cells
  int64_t launches = 0;
  int64_t host_count_buf[4] = {0, 0, 0, 0};
  int64_t* pinned_counts = nullptr;
  int64_t h2d_bytes = 0;               // bytes of raster copied host->device by the last upload
  uint8_t* pinned_need = nullptr;       // on_host + fused zh_run: per-tile 'needed' flags (host copy)
  size_t pinned_counts_bytes = 0, pinned_need_bytes = 0;  // sizes of the cached pinned blocks
  DBuf d_need;
  // Sizes of the step's lists are a function of the context's fixed geometry (polygons, raster
  // extent, tile): the first zh_pair_tiles / zh_fused_update learn them with host syncs, later calls
  // reuse them and run with no host round trip (capturable in a CUDA graph, zh_step_graph); a
  // device check (k_check_counts) flags any step whose counts differ, reported at the next sync.
  bool sizes_known = false, fused_known = false;
  int64_t n_pip_known = 0, n_grp_known = 0;
  DBuf d_flag;
  bool capturing = false;                 // recording a CUDA graph: events become external records
  cudaGraphExec_t gexec = nullptr;
  int32_t graph_fused = -1;               // the path the graph was captured for
  int64_t graph_kernels = 0;              // kernel launches one replay performs
  bool bad_sizes_pending = false;         // ZH_TEST_BAD_SIZES: test hook of the device size check
  int64_t n_cand_check_bias = 0;
};

// Kernel attributes set before a launch: the dynamic shared memory beyond 48 KB it needs, and (with
// ZH_CARVEOUT >= 0) the preferred shared-memory carveout, the same for every kernel of the step so
// that consecutive kernels do not reconfigure the SMs' L1 / shared split.
#ifndef ZH_CARVEOUT
#define ZH_CARVEOUT -1
#endif
template <class K>
inline void prep_kernel(K k, size_t smem) {
  if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (ZH_CARVEOUT >= 0) cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, ZH_CARVEOUT);
}

// Timing event on stream s (an external record node while a graph is being captured).
inline void rec_event(const Ctx& c, cudaEvent_t e, cudaStream_t s) {
  cudaEventRecordWithFlags(e, s, c.capturing ? cudaEventRecordExternal : cudaEventRecordDefault);
}
// Device check of counts[i] == want[i] (i < n <= 6); sets *flag (k_pairs.cu).
cudaError_t launch_check_counts(Ctx& c, const int64_t* counts, const int64_t* want, int n);

// kernels / launchers (k_*.cu)
cudaError_t launch_tile_hist(Ctx& c);
cudaError_t launch_pairs_phase1(Ctx& c);   // edges, MBBs, scans, count totals -> d_counts
cudaError_t launch_pairs_phase2(Ctx& c);   // bands, marking, classification, compaction
cudaError_t launch_aggregate(Ctx& c);
cudaError_t launch_pip(Ctx& c);
cudaError_t launch_pip_list(Ctx& c, const int2* pairs, int64_t grid, const int64_t* n_dev);
cudaError_t pip_prepare(Ctx& c, int64_t grid);  // split form: per-pair parity bitmap buffer
cudaError_t launch_parity(Ctx& c, const int2* pairs, int64_t grid, const int64_t* n_dev, cudaStream_t s);
cudaError_t launch_pip_cells(Ctx& c, const int2* pairs, int64_t grid, const int64_t* n_dev);
size_t mixed_smem(Ctx& c);  // 0: the grouped cell kernel does not apply
cudaError_t launch_mixed_cells(Ctx& c, const int2* pairs, const int2* grp, int64_t grid, const int64_t* n_dev);
cudaError_t launch_touch(Ctx& c, const int32_t* remap, cudaStream_t s);  // k_touch.cu (cover mode)
cudaError_t launch_fused(Ctx& c);  // steps 1 + 3 + 4 fused (k_fused.cu)
cudaError_t launch_need_tiles(Ctx& c);  // d_need[t] = tile t has a pair (k_fused.cu)
cudaError_t launch_zonal_stats(Ctx& c, int64_t* dstats);  // k_stats.cu
cudaError_t launch_zonal_summary(Ctx& c, const int64_t* dstats, double* dout);  // k_features.cu
cudaError_t launch_hist_distance(Ctx& c, int kind, const int64_t* dstats, bool narrow, const int32_t* ia,
                                 const int32_t* ib, int64_t n, double* dout);  // k_features.cu
cudaError_t launch_row_cost(Ctx& c, double* d_row_cost);  // k_fused.cu (shard planning)

size_t device_bytes(const Ctx& c);

}  // namespace zh
