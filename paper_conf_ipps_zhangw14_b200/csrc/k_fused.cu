// k_fused.cu — fused, needed-tiles-only histogramming (SURVEY.md §8f-1 "NEXT 1").
//
// Step 1 is independent of the polygons (§III ¶1), so after step 2 the tiles split into
//   * outside-only tiles  — no pair: never read;
//   * pure tiles          — >= 1 inside pair and no intersecting pair: the tile is histogrammed in
//                           shared memory exactly as in step 1 and the histogram is added straight
//                           into each inside polygon's row (steps 1 + 3 fused: no per-tile histogram
//                           array, no second pass);
//   * mixed tiles         — >= 1 intersecting pair: every pair of the tile (intersecting, and the rare
//                           inside pair of a mixed tile, e.g. overlapping polygons) goes through the
//                           step-4 cell-in-polygon kernel, which is exact for any pair.
// Each raster cell is therefore read once from HBM, and only when some polygon may contain it.
// The result is bit-identical to steps 1 + 3 + 4 (integer sums; tests/test_gpu_fused.py).
#include <algorithm>

#include <cub/device/device_scan.cuh>

#include "zh_ctx.h"
#include "zh_pip.cuh"
#include "zh_tilehist.cuh"

#ifndef ZH_PURE_MINB
#define ZH_PURE_MINB 3  // CTAs of 512 threads per SM the pure-tile kernel is compiled for (register cap)
#endif


namespace zh {

// pip_cnt[t] = #pairs of tile t for the cell-in-polygon kernel: its intersecting pairs, then (below)
// the inside pairs of the tiles that have one (a tile is "mixed" iff it has an intersecting pair)
__global__ void k_mark_mixed(const int2* __restrict__ isect, int64_t n, uint32_t* __restrict__ pip_cnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&pip_cnt[isect[i].x], 1u);
}

// inside pairs of pure tiles are counted per tile; inside pairs of mixed tiles are flagged "extra"
// and join the tile's cell-in-polygon pairs (pip_cnt of a tile is either 0 throughout — pure — or
// > 0 before and after this kernel's increments, so the test below does not race)
__global__ void k_inside_split(const int2* __restrict__ inside, int64_t n, uint32_t* __restrict__ pip_cnt,
                               uint32_t* __restrict__ pure_cnt, uint32_t* __restrict__ extra) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int t = inside[i].x;
    if (*(volatile uint32_t*)&pip_cnt[t]) {
      extra[i] = 1;
      atomicAdd(&pip_cnt[t], 1u);
    } else {
      extra[i] = 0;
      atomicAdd(&pure_cnt[t], 1u);
    }
  }
}

// packed per-tile value for one scan: low 32 = #inside polygons, high 32 = (tile is pure)
__global__ void k_pack_tiles(const uint32_t* __restrict__ pure_cnt, int64_t n, uint64_t* __restrict__ pk) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t c = pure_cnt[i];
    pk[i] = (uint64_t)c | ((uint64_t)(c > 0) << 32);
  }
}

__global__ void k_pure_fill(const int2* __restrict__ inside, int64_t n, const uint32_t* __restrict__ extra,
                            const uint64_t* __restrict__ pure_off, uint32_t* __restrict__ cursor,
                            int32_t* __restrict__ pure_poly) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (extra[i]) continue;
    const int2 p = inside[i];
    const uint32_t pos = (uint32_t)(pure_off[p.x] & 0xFFFFFFFFull) + atomicAdd(&cursor[p.x], 1u);
    pure_poly[pos] = p.y;
  }
}

__device__ __forceinline__ int64_t tile_cells(const RasterP& rp, int tile) {
  const int trl = tile_row(rp, tile), tc = tile - trl * rp.TC;
  const int64_t r0 = (int64_t)(rp.tr0 + trl) * rp.T, c0 = (int64_t)tc * rp.T;
  return min((int64_t)rp.T, rp.row0 + rp.nrows - r0) * min((int64_t)rp.T, rp.cols - c0);
}

// counts[0] = #pure tiles, counts[2] = their cells (bench: algorithmic bytes)
__global__ void k_pure_tiles(const uint32_t* __restrict__ pure_cnt, int64_t n, const uint64_t* __restrict__ pure_off,
                             RasterP rp, int32_t* __restrict__ pure_tiles, int64_t* __restrict__ counts) {
  int64_t cells = 0;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    if (pure_cnt[t]) {
      pure_tiles[pure_off[t] >> 32] = (int32_t)t;
      cells += tile_cells(rp, (int)t);
    }
    if (t == n - 1) counts[0] = (int64_t)(pure_off[t] >> 32) + (pure_cnt[t] ? 1 : 0);
  }
  for (int o = 16; o > 0; o >>= 1) cells += __shfl_xor_sync(0xffffffffu, cells, o);
  if ((threadIdx.x & 31) == 0 && cells) atomicAdd(reinterpret_cast<unsigned long long*>(&counts[2]),
                                                  (unsigned long long)cells);
}

// counts[1] = #pairs for the cell-in-polygon kernel, counts[3] = their tiles' cells.  The list is
// grouped BY TILE (pip_off = exclusive scan of pip_cnt), so the 2-3 pairs that read the same mixed
// tile run back to back and all but the first find its cells in L2 (grouped by polygon, as step 2
// emits them, the L2 hit rate of the per-pair cell pass was 15 %).
__global__ void k_pip_list(const int2* __restrict__ isect, int64_t n_isect, const int2* __restrict__ inside,
                           int64_t n_inside, const uint32_t* __restrict__ extra, const uint64_t* __restrict__ pip_off,
                           uint32_t* __restrict__ cursor, int64_t n_tiles, RasterP rp, int2* __restrict__ pip,
                           int32_t* __restrict__ remap, int64_t* __restrict__ counts) {
  const int64_t n = n_isect + n_inside;
  int64_t cells = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int2 pr;
    if (i < n_isect) {
      pr = isect[i];
    } else {
      if (!extra[i - n_isect]) continue;
      pr = inside[i - n_isect];
    }
    const uint32_t pos = (uint32_t)pip_off[pr.x] + atomicAdd(&cursor[pr.x], 1u);
    pip[pos] = pr;
    if (remap && i < n_isect) remap[i] = (int32_t)pos;  // isect index -> list index (k_touch)
    cells += tile_cells(rp, pr.x);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) counts[1] = (int64_t)(uint32_t)pip_off[n_tiles];
  for (int o = 16; o > 0; o >>= 1) cells += __shfl_xor_sync(0xffffffffu, cells, o);
  if ((threadIdx.x & 31) == 0 && cells) atomicAdd(reinterpret_cast<unsigned long long*>(&counts[3]),
                                                  (unsigned long long)cells);
}

// Tile groups of the grouped cell kernel (k_mixed_cells): a mixed tile with c cell-in-polygon pairs
// forms ceil(c / 2) groups of <= 2 consecutive pairs.  pk[t] = c | ceil(c / 2) << 32, so one
// exclusive scan gives both the tile's first pair (low half) and its first group (high half).
__global__ void k_pack_mixed(const uint32_t* __restrict__ cnt, int64_t n, uint64_t* __restrict__ pk) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t c = cnt[i];
    pk[i] = (uint64_t)c | ((uint64_t)((c + 1) >> 1) << 32);
  }
}


// grp[g] = {first pair index, #pairs}; counts[4] = #groups, counts[5] = cells read by the groups
// (a mixed tile once per group), counts[6] = cells of the mixed tiles (each once: the HBM bytes the
// grouped cell kernel must read — later groups of a tile find it in L2)
__global__ void k_pip_groups(const uint32_t* __restrict__ cnt, const uint64_t* __restrict__ off, int64_t n_tiles,
                             RasterP rp, int2* __restrict__ grp, int64_t* __restrict__ counts) {
  int64_t cells = 0, tcells = 0;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n_tiles; t += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t c = cnt[t];
    if (!c) continue;
    const uint32_t p0 = (uint32_t)off[t], g0 = (uint32_t)(off[t] >> 32);
    for (uint32_t q = 0; 2 * q < c; ++q) grp[g0 + q] = make_int2((int)(p0 + 2 * q), (int)min(2u, c - 2 * q));
    cells += tile_cells(rp, (int)t) * (int64_t)((c + 1) >> 1);
    tcells += tile_cells(rp, (int)t);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) counts[4] = (int64_t)(off[n_tiles] >> 32);
  for (int o = 16; o > 0; o >>= 1) {
    cells += __shfl_xor_sync(0xffffffffu, cells, o);
    tcells += __shfl_xor_sync(0xffffffffu, tcells, o);
  }
  if ((threadIdx.x & 31) == 0 && cells) {
    atomicAdd(reinterpret_cast<unsigned long long*>(&counts[5]), (unsigned long long)cells);
    atomicAdd(reinterpret_cast<unsigned long long*>(&counts[6]), (unsigned long long)tcells);
  }
}

struct PureP {
  RasterP rp;
  BinP bp;
  FastBins fb;
  const int32_t* pure_tiles;
  const int64_t* counts;
  const uint64_t* pure_off;
  const uint32_t* pure_cnt;
  const int32_t* pure_poly;
  void* out;
  int run;  // pure tiles per CTA (k_fused_pure)
};

// Same inside-polygon set for two pure tiles (lists compared in stored order: a permuted list only
// costs an extra flush)?
__device__ __forceinline__ bool same_polys(const PureP& f, int ta, int tb) {
  const uint32_t ca = f.pure_cnt[ta];
  if (ca != f.pure_cnt[tb]) return false;
  const uint32_t a0 = (uint32_t)(f.pure_off[ta] & 0xFFFFFFFFull), b0 = (uint32_t)(f.pure_off[tb] & 0xFFFFFFFFull);
  for (uint32_t j = 0; j < ca; ++j)
    if (f.pure_poly[a0 + j] != f.pure_poly[b0 + j]) return false;
  return true;
}

// Add the shared histogram into the row of each inside polygon of `tile` (one global atomic per
// non-zero bin; 16-byte reads of the histogram skip whole zero vectors — a tile touches a few
// hundred of 5,000 bins).
template <bool kU64>
__device__ __forceinline__ void pure_flush(const PureP& f, int tile, const uint32_t* __restrict__ sh) {
  const uint32_t beg = (uint32_t)(f.pure_off[tile] & 0xFFFFFFFFull), cnt = f.pure_cnt[tile];
  const int nbins = f.bp.nbins;
  for (uint32_t j = 0; j < cnt; ++j) {
    const int64_t row = (int64_t)f.pure_poly[beg + j] * nbins;
    for (int b = threadIdx.x * 4; b < nbins; b += blockDim.x * 4) {
      const uint4 v = *reinterpret_cast<const uint4*>(&sh[kOff + b]);
      if (!(v.x | v.y | v.z | v.w)) continue;
      const uint32_t vs[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        if (vs[q] && b + q < nbins) {
          if (kU64) atomicAdd(reinterpret_cast<unsigned long long*>(f.out) + row + b + q, (unsigned long long)vs[q]);
          else atomicAdd(reinterpret_cast<uint32_t*>(f.out) + row + b + q, vs[q]);
        }
      }
    }
  }
}

// A CTA takes f.run (<= ZH_PURE_RUN) consecutive entries of the pure-tile list (tile order:
// neighbouring tiles, mostly of the same county) and keeps ONE shared histogram across consecutive
// tiles with the same inside-polygon set: no barrier between them (the loads of the next tile
// follow the last atomics of the previous one) and one flush per run instead of one per tile.
// The host lowers the run when the list is short, so that the grid still fills the GPU.
#ifndef ZH_PURE_RUN
#define ZH_PURE_RUN 8
#endif
constexpr int kPureRun = ZH_PURE_RUN;

constexpr int kPureRunMax = 256;  // pure_params caps the run at this many tiles

template <int kMode, bool kU64>
__global__ void __launch_bounds__(512, ZH_PURE_MINB) k_fused_pure(PureP f) {
  const int64_t n = f.counts[0];
  const int64_t i0 = (int64_t)blockIdx.x * f.run;
  if (i0 >= n) return;
  const int nrun = (int)(min(n, i0 + (int64_t)f.run) - i0);
  extern __shared__ __align__(16) uint32_t sh[];
  // the run's tiles and where its inside-polygon set changes (a flush), decided by all threads at
  // once: the per-tile list reads are one round of latency per CTA instead of one per tile
  __shared__ int s_tile[kPureRunMax];
  __shared__ uint8_t s_flush[kPureRunMax];
  for (int j = threadIdx.x; j < nrun; j += blockDim.x) {
    const int t = f.pure_tiles[i0 + j];
    s_tile[j] = t;
    s_flush[j] = (j == nrun - 1 || !same_polys(f, t, f.pure_tiles[i0 + j + 1])) ? 1 : 0;
  }
  const int HW = hist_words(f.bp.nbins);
  auto zero = [&]() {
    for (int i = threadIdx.x * 4; i < HW; i += blockDim.x * 4)
      *reinterpret_cast<uint4*>(&sh[i]) = make_uint4(0, 0, 0, 0);
  };
  zero();
  __syncthreads();
  for (int j = 0; j < nrun; ++j) {
    const int tile = s_tile[j];
    const int trl = tile_row(f.rp, tile), tc = tile - trl * f.rp.TC;
    tile_histogram<kMode, ZH_PURE_WROWS>(sh, f.rp, f.bp, f.fb, trl, tc);
    if (s_flush[j]) {  // uniform over the CTA
      __syncthreads();
      pure_flush<kU64>(f, tile, sh);
      if (j + 1 < nrun) {
        __syncthreads();
        zero();
        __syncthreads();
      }
    }
  }
}

// ---- work-balanced shard planning: estimated cost of every tile row of the
// raster from step 2's pair lists — cells of inside pairs (read once, histogrammed) and cells of
// intersecting pairs (read per pair, tested) plus a fixed cost per intersecting pair.  Weights
// are the measured per-cell times of the fused kernels.
__global__ void k_row_cost(const int2* __restrict__ inside, int64_t n_inside, const int2* __restrict__ isect,
                           int64_t n_isect, RasterP rp, double w_in, double w_x, double w_pair,
                           double* __restrict__ row_cost) {
  const int64_t n = n_inside + n_isect;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const bool in = i < n_inside;
    const int tile = in ? inside[i].x : isect[i - n_inside].x;
    const double cells = (double)tile_cells(rp, tile);
    atomicAdd(&row_cost[tile / rp.TC], in ? w_in * cells : w_x * cells + w_pair);
  }
}

cudaError_t launch_row_cost(Ctx& c, double* d_row_cost) {
  cudaMemsetAsync(d_row_cost, 0, sizeof(double) * (size_t)c.rp.TRn, c.stream);
  const int64_t n = c.n_inside + c.n_isect;
  if (n > 0) {
    int64_t b = (n + 255) / 256;
    if (b > 148 * 32) b = 148 * 32;
    k_row_cost<<<(unsigned)b, 256, 0, c.stream>>>(c.d_inside.as<int2>(), c.n_inside, c.d_isect.as<int2>(),
                                                   c.n_isect, c.rp, 0.37, 0.53, 2000.0 * 0.37, d_row_cost);
    c.launches += 1;
  }
  return cudaGetLastError();
}

// need[t] = 1 for every tile of some inside or intersecting pair (on_host zh_run of the fused path
// uploads only those tiles: the others are read by no kernel)
__global__ void k_need_tiles(const int2* __restrict__ inside, int64_t n_inside, const int2* __restrict__ isect,
                             int64_t n_isect, uint8_t* __restrict__ need) {
  const int64_t n = n_inside + n_isect;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    need[i < n_inside ? inside[i].x : isect[i - n_inside].x] = 1;
}

static int grid_for(int64_t n, int threads) {
  int64_t b = (n + threads - 1) / threads;
  if (b > 148 * 32) b = 148 * 32;
  if (b < 1) b = 1;
  return (int)b;
}

template <class T>
static cudaError_t excl_scan(Ctx& c, const T* in, T* out, int64_t n) {
  size_t need = 0;
  cudaError_t e = cub::DeviceScan::ExclusiveSum(nullptr, need, in, out, (int)n, c.stream);
  if (e != cudaSuccess) return e;
  if ((e = c.d_cub.ensure(need)) != cudaSuccess) return e;
  size_t have = c.d_cub.bytes;
  c.launches += 2;  // CUB init + scan kernels
  return cub::DeviceScan::ExclusiveSum(c.d_cub.p, have, in, out, (int)n, c.stream);
}

static PureP pure_params(Ctx& c) {
  PureP f;
  f.rp = c.rp;
  f.bp = c.bp;
  f.fb = make_fast_bins(c.bp);
  f.pure_tiles = c.d_pure_tiles.as<int32_t>();
  f.counts = c.d_fcounts.as<int64_t>();
  f.pure_off = c.d_pure_off.as<uint64_t>();
  f.pure_cnt = c.d_pure_cnt.as<uint32_t>();
  f.pure_poly = c.d_pure_poly.as<int32_t>();
  f.out = c.d_out;
  // enough CTAs for >= 4 waves of 3 per SM (148 SMs), at most kPureRun tiles of 256^2 cells each
  // (more tiles when they are smaller: the zeroing and the flush are per run, not per cell)
  const int64_t T2 = (int64_t)c.rp.T * c.rp.T;
  const int64_t cap = std::max<int64_t>(kPureRun, std::min<int64_t>(kPureRunMax, kPureRun * 65536 / std::max<int64_t>(T2, 1)));
  const int64_t run = c.n_inside / (148 * 3 * 4);
  // the shared uint32 histogram is kept across a run of tiles: run * T^2 < 2^32 (zh_create caps T)
  const int64_t no_wrap = std::max<int64_t>(1, (int64_t)0xFFFFFFFFll / std::max<int64_t>(T2, 1));
  f.run = (int)std::max<int64_t>(1, std::min<int64_t>(std::min<int64_t>(cap, run), no_wrap));
  return f;
}

template <int kMode, bool kU64>
static void launch_pure(Ctx& c, size_t smem, unsigned grid) {
  auto k = k_fused_pure<kMode, kU64>;
  prep_kernel(k, smem);
  k<<<grid, 512, smem, c.stream>>>(pure_params(c));
}

cudaError_t launch_need_tiles(Ctx& c) {
  cudaError_t e;
  if ((e = c.d_need.ensure((size_t)c.n_tiles + 1)) != cudaSuccess) return e;
  if ((e = cudaMemsetAsync(c.d_need.p, 0, (size_t)c.n_tiles + 1, c.stream)) != cudaSuccess) return e;
  const int64_t n = c.n_inside + c.n_isect;
  if (n > 0) {
    k_need_tiles<<<grid_for(n, 256), 256, 0, c.stream>>>(c.d_inside.as<int2>(), c.n_inside, c.d_isect.as<int2>(),
                                                         c.n_isect, c.d_need.as<uint8_t>());
    c.launches += 1;
  }
  return cudaGetLastError();
}

cudaError_t launch_fused(Ctx& c) {
  cudaError_t e;
  const int64_t NT = c.n_tiles, NI = c.n_inside, NX = c.n_isect;
  if ((e = c.d_mixed.ensure(sizeof(uint32_t) * ((size_t)NT + 1))) != cudaSuccess) return e;
  if ((e = c.d_pip_cur.ensure(sizeof(uint32_t) * ((size_t)NT + 1))) != cudaSuccess) return e;
  if ((e = c.d_pure_cnt.ensure(sizeof(uint32_t) * ((size_t)NT + 1))) != cudaSuccess) return e;
  if ((e = c.d_pure_cur.ensure(sizeof(uint32_t) * ((size_t)NT + 1))) != cudaSuccess) return e;
  if ((e = c.d_pure_pk.ensure(sizeof(uint64_t) * ((size_t)NT + 1))) != cudaSuccess) return e;
  if ((e = c.d_pure_off.ensure(sizeof(uint64_t) * ((size_t)NT + 1))) != cudaSuccess) return e;
  if ((e = c.d_pure_poly.ensure(sizeof(int32_t) * ((size_t)NI + 1))) != cudaSuccess) return e;
  if ((e = c.d_pure_tiles.ensure(sizeof(int32_t) * ((size_t)NI + 1))) != cudaSuccess) return e;
  if ((e = c.d_extra.ensure(sizeof(uint32_t) * ((size_t)NI + 1))) != cudaSuccess) return e;
  if ((e = c.d_extra_pos.ensure(sizeof(uint64_t) * ((size_t)NT + 1))) != cudaSuccess) return e;
  if ((e = c.d_mixed_pk.ensure(sizeof(uint64_t) * ((size_t)NT + 1))) != cudaSuccess) return e;
  if ((e = c.d_pip.ensure(sizeof(int2) * ((size_t)NI + NX + 1))) != cudaSuccess) return e;
  if ((e = c.d_fcounts.ensure(sizeof(int64_t) * 7)) != cudaSuccess) return e;
  if (c.cover && (e = c.d_remap.ensure(sizeof(int32_t) * ((size_t)NX + 1))) != cudaSuccess) return e;
  cudaMemsetAsync(c.d_fcounts.p, 0, sizeof(int64_t) * 7, c.stream);
  if (NT == 0 || NI + NX == 0) {
    if (c.timing)
      for (int i = 10; i < 16; ++i) rec_event(c, c.ev[i], c.stream);
    return cudaGetLastError();
  }

  cudaMemsetAsync(c.d_mixed.p, 0, sizeof(uint32_t) * ((size_t)NT + 1), c.stream);
  cudaMemsetAsync(c.d_pip_cur.p, 0, sizeof(uint32_t) * ((size_t)NT + 1), c.stream);
  cudaMemsetAsync(c.d_pure_cnt.p, 0, sizeof(uint32_t) * ((size_t)NT + 1), c.stream);
  cudaMemsetAsync(c.d_pure_cur.p, 0, sizeof(uint32_t) * ((size_t)NT + 1), c.stream);
  if (NX > 0) {
    k_mark_mixed<<<grid_for(NX, 256), 256, 0, c.stream>>>(c.d_isect.as<int2>(), NX, c.d_mixed.as<uint32_t>());
    c.launches += 1;
  }
  if (NI > 0) {
    k_inside_split<<<grid_for(NI, 256), 256, 0, c.stream>>>(c.d_inside.as<int2>(), NI, c.d_mixed.as<uint32_t>(),
                                                           c.d_pure_cnt.as<uint32_t>(), c.d_extra.as<uint32_t>());
    c.launches += 1;
  }
  k_pack_tiles<<<grid_for(NT + 1, 256), 256, 0, c.stream>>>(c.d_pure_cnt.as<uint32_t>(), NT + 1,
                                                            c.d_pure_pk.as<uint64_t>());
  c.launches += 1;
  if ((e = excl_scan<uint64_t>(c, c.d_pure_pk.as<uint64_t>(), c.d_pure_off.as<uint64_t>(), NT + 1)) != cudaSuccess)
    return e;
  if (NI > 0) {
    k_pure_fill<<<grid_for(NI, 256), 256, 0, c.stream>>>(c.d_inside.as<int2>(), NI, c.d_extra.as<uint32_t>(),
                                                        c.d_pure_off.as<uint64_t>(), c.d_pure_cur.as<uint32_t>(),
                                                        c.d_pure_poly.as<int32_t>());
    c.launches += 1;
  }
  k_pure_tiles<<<grid_for(NT, 256), 256, 0, c.stream>>>(c.d_pure_cnt.as<uint32_t>(), NT, c.d_pure_off.as<uint64_t>(),
                                                        c.rp, c.d_pure_tiles.as<int32_t>(), c.d_fcounts.as<int64_t>());
  c.launches += 1;
  k_pack_mixed<<<grid_for(NT + 1, 256), 256, 0, c.stream>>>(c.d_mixed.as<uint32_t>(), NT + 1,
                                                            c.d_mixed_pk.as<uint64_t>());
  c.launches += 1;
  if ((e = excl_scan<uint64_t>(c, c.d_mixed_pk.as<uint64_t>(), c.d_extra_pos.as<uint64_t>(), NT + 1)) != cudaSuccess)
    return e;
  k_pip_list<<<grid_for(NI + NX, 256), 256, 0, c.stream>>>(c.d_isect.as<int2>(), NX, c.d_inside.as<int2>(), NI,
                                                          c.d_extra.as<uint32_t>(), c.d_extra_pos.as<uint64_t>(),
                                                          c.d_pip_cur.as<uint32_t>(), NT, c.rp, c.d_pip.as<int2>(),
                                                          c.cover ? c.d_remap.as<int32_t>() : nullptr,
                                                          c.d_fcounts.as<int64_t>());
  c.launches += 1;

  // grouped cell kernel: tile groups of <= 2 pairs (every cell read once per group)
  const bool grouped = c.pip_group != 0 && mixed_smem(c) > 0;
  if (grouped) {
    if ((e = c.d_pip_grp.ensure(sizeof(int2) * ((size_t)NI + NX + 1))) != cudaSuccess) return e;
    k_pip_groups<<<grid_for(NT, 256), 256, 0, c.stream>>>(c.d_mixed.as<uint32_t>(), c.d_extra_pos.as<uint64_t>(), NT,
                                                          c.rp, c.d_pip_grp.as<int2>(), c.d_fcounts.as<int64_t>());
    c.launches += 1;
  }

  const int mode = fast_bins_ok(c.bp) ? (make_fast_bins(c.bp).bias ? 4 : (c.bp.use_nodata ? 3 : 2))
                                      : (c.bp.width == 1 ? 0 : 1);
  // mixed tiles, split form: the parity bitmaps of every cell-in-polygon pair are built on the side
  // stream WHILE the pure-tile kernel streams the pure tiles (FP64-latency work beside HBM-bound
  // work), then the cell kernel runs once both are done
  // exact grid for the cell kernel: the list sizes are copied to the host behind the list kernels
  // and read while the pure-tile kernel runs (no CTAs that only find they have no work)
  if ((e = pip_prepare(c, NI + NX)) != cudaSuccess) return e;
  if (!c.fused_known) {
    cudaMemcpyAsync(c.pinned_counts + 8, c.d_fcounts.p, 6 * sizeof(int64_t), cudaMemcpyDeviceToHost, c.stream);
    cudaEventRecord(c.ev_counts, c.stream);
  } else {  // known sizes (fixed geometry): the device checks the recomputed counts
    const int64_t want[4] = {c.n_pip_known, 0, 0, c.n_grp_known};
    if ((e = launch_check_counts(c, c.d_fcounts.as<int64_t>() + 1, want, 1)) != cudaSuccess) return e;
    if ((e = launch_check_counts(c, c.d_fcounts.as<int64_t>() + 4, want + 3, 1)) != cudaSuccess) return e;
  }
  auto parity = [&](int64_t grid) -> cudaError_t {
    cudaError_t pe;
    if (c.timing) rec_event(c, c.ev[13], c.stream);
    if ((pe = launch_parity(c, c.d_pip.as<int2>(), grid, c.d_fcounts.as<int64_t>() + 1, c.stream)) != cudaSuccess)
      return pe;
    if (c.cover) {  // R15: cells an edge reaches join the parity bits (k_touch.cu)
      if ((pe = launch_touch(c, c.d_remap.as<int32_t>(), c.stream)) != cudaSuccess) return pe;
    }
    if (c.timing) rec_event(c, c.ev[14], c.stream);
    return cudaSuccess;
  };
  // pure tiles: steps 1 + 3 fused (grid = upper bound, surplus CTAs exit at once)
  if (c.timing) rec_event(c, c.ev[10], c.stream);
  if (NI > 0) {
    const size_t smem = (size_t)hist_words(c.bp.nbins) * 4;
    const int run = pure_params(c).run;
    const unsigned grid = (unsigned)((NI + run - 1) / run);
    if (c.out_u64) {
      switch (mode) {
        case 0: launch_pure<0, true>(c, smem, grid); break;
        case 1: launch_pure<1, true>(c, smem, grid); break;
        case 2: launch_pure<2, true>(c, smem, grid); break;
        case 3: launch_pure<3, true>(c, smem, grid); break;
        default: launch_pure<4, true>(c, smem, grid); break;
      }
    } else {
      switch (mode) {
        case 0: launch_pure<0, false>(c, smem, grid); break;
        case 1: launch_pure<1, false>(c, smem, grid); break;
        case 2: launch_pure<2, false>(c, smem, grid); break;
        case 3: launch_pure<3, false>(c, smem, grid); break;
        default: launch_pure<4, false>(c, smem, grid); break;
      }
    }
    c.launches += 1;
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  if (c.timing) rec_event(c, c.ev[11], c.stream);
  if (!c.fused_known) {
    if ((e = cudaEventSynchronize(c.ev_counts)) != cudaSuccess) return e;
    c.n_pip_known = c.pinned_counts[8 + 1];
    c.n_grp_known = c.pinned_counts[8 + 4];
    c.fused_known = true;
  }
  const int64_t n_pip = c.n_pip_known;
  const int64_t n_grp = c.n_grp_known;
  if (n_pip > 0) {
    if ((e = parity(n_pip)) != cudaSuccess) return e;
  } else if (c.timing) {
    rec_event(c, c.ev[13], c.stream);
    rec_event(c, c.ev[14], c.stream);
  }
  if (c.timing) rec_event(c, c.ev[15], c.stream);
  if (grouped)
    e = n_grp > 0 ? launch_mixed_cells(c, c.d_pip.as<int2>(), c.d_pip_grp.as<int2>(), n_grp,
                                       c.d_fcounts.as<int64_t>() + 4)
                  : cudaSuccess;
  else
    e = n_pip > 0 ? launch_pip_cells(c, c.d_pip.as<int2>(), n_pip, c.d_fcounts.as<int64_t>() + 1) : cudaSuccess;
  if (c.timing) rec_event(c, c.ev[12], c.stream);
  return e;
}

}  // namespace zh
