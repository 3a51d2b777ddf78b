// k_pairs.cu — step 2: pair raster tiles with polygons and classify each pair
// (§III.B, Fig. 3; segment bookkeeping of PAPER.md:16-18 §III.C / Fig. 4 left).
//
// Paper design (prior art): MBB rasterisation with the GPU grid-file of [19]; the tile-in-polygon
// test on the CPU "using well-established computational geometry libraries", then Thrust
// stable_sort_by_key / stable_partition / reduce_by_key / scan to build per-polygon segments.
// B200 design, all on the GPU:
//   1. k_mbb_edges — one CTA per polygon: vertex MBB -> covered tile rectangle (1-cell margin);
//                  then one thread per vertex: the ring edge it starts, in canonical orientation,
//                  and the exact half-open interval of centre rows it straddles (ya <= yc(r) < yb),
//                  found with the same yc(r) expression the PIP test uses;
//   3. scans     — candidate offsets and band (polygon, tile-row) bases (CUB);
//   4. k_poly_bands — per (polygon, tile row) lists of the edges whose row interval meets it (the
//                  step-4 edge lists and the classifier's input), counted in shared memory;
//   5. k_mark    — a tile is INTERSECT if some edge's bounding box comes within one cell of
//                  its cell rectangle (conservative; DESIGN.md §4 proof);
//   6. k_classify— every other candidate tile has a uniform computed PIP status, evaluated exactly
//                  at its first cell with a scanline over the band's edges (INSIDE / OUTSIDE);
//   7. compaction— packed (inside, intersect) exclusive scan -> (tile, polygon) lists sorted by
//                  (polygon, tile).
#include <algorithm>

#include <cub/device/device_scan.cuh>

#include "zh_ctx.h"

#ifndef ZH_MARK_RCP
#define ZH_MARK_RCP 1
#endif

namespace zh {

__device__ __forceinline__ int64_t upper_bound_i64(const int64_t* a, int64_t n, int64_t v) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t m = (lo + hi) >> 1;
    if (a[m] <= v) lo = m + 1; else hi = m;
  }
  return lo;
}

__device__ __forceinline__ int64_t clamp_est(double v, int64_t lo, int64_t hi) {
  if (!(v > (double)lo)) return lo;  // also NaN
  if (v > (double)hi) return hi;
  return (int64_t)ceil(v);
}

// Rows r in [rA, rB) with ya <= yc(r) < yb, exactly (monotone predicates + first_false).
__device__ __forceinline__ int2 straddle_rows(const Geo& g, double ya, double yb, int64_t rA, int64_t rB) {
  if (!(ya < yb)) return make_int2(0, 0);
  // first guesses only (first_false makes the rows exact): reciprocal instead of a division
  const double ea = (ya - g.gt3) * g.igt5 - g.oy, eb = (yb - g.gt3) * g.igt5 - g.oy;
  int64_t ra, rb;
  if (g.gt5 < 0) {  // yc decreasing in r
    // B(r): yc(r) < yb  is false then true -> ra = first r with B true
    ra = first_false(rA, rB, clamp_est(eb, rA, rB), [&](int64_t r) { return !(row_centre(g, r) < yb); });
    // A(r): ya <= yc(r) is true then false -> rb = first r with A false
    rb = first_false(rA, rB, clamp_est(ea, rA, rB), [&](int64_t r) { return ya <= row_centre(g, r); });
  } else {          // yc increasing in r
    ra = first_false(rA, rB, clamp_est(ea, rA, rB), [&](int64_t r) { return !(ya <= row_centre(g, r)); });
    rb = first_false(rA, rB, clamp_est(eb, rA, rB), [&](int64_t r) { return row_centre(g, r) < yb; });
  }
  if (ra >= rb) return make_int2(0, 0);
  return make_int2((int)ra, (int)rb);
}

// MBB of polygon k's vertices -> covered tile rectangle (global tile indices), clipped to the raster
// columns and the shard rows, from each thread's partial min / max.  Empty -> (1, 0, 1, 0).
// Returned to every thread of the CTA.
__device__ __forceinline__ int4 mbb_reduce(int k, int nv, double xmn, double xmx, double ymn, double ymx, const Geo& g,
                                           const RasterP& rp, int4* __restrict__ mbb, int64_t* __restrict__ ncand,
                                           int64_t* __restrict__ nband) {
  __shared__ int4 s_m;
  __shared__ double s[4][8];
  for (int o = 16; o > 0; o >>= 1) {
    xmn = fmin(xmn, __shfl_xor_sync(0xffffffffu, xmn, o));
    xmx = fmax(xmx, __shfl_xor_sync(0xffffffffu, xmx, o));
    ymn = fmin(ymn, __shfl_xor_sync(0xffffffffu, ymn, o));
    ymx = fmax(ymx, __shfl_xor_sync(0xffffffffu, ymx, o));
  }
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) { s[0][wid] = xmn; s[1][wid] = xmx; s[2][wid] = ymn; s[3][wid] = ymx; }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < (int)(blockDim.x >> 5); ++w) {
      xmn = fmin(xmn, s[0][w]); xmx = fmax(xmx, s[1][w]);
      ymn = fmin(ymn, s[2][w]); ymx = fmax(ymx, s[3][w]);
    }
    int4 m = make_int4(1, 0, 1, 0);
    int64_t nc = 0, nb = 0;
    if (nv > 0) {
      double ca = (xmn - g.gt0) / g.gt1, cb = (xmx - g.gt0) / g.gt1;
      double ra = (ymn - g.gt3) / g.gt5, rb = (ymx - g.gt3) / g.gt5;
      if (ca > cb) { double t = ca; ca = cb; cb = t; }
      if (ra > rb) { double t = ra; ra = rb; rb = t; }
      // 1-cell margin; clip in double first (coordinates may be far off the raster)
      double clo = fmax(floor(ca) - 1.0, 0.0), chi = fmin(floor(cb) + 1.0, (double)(rp.cols - 1));
      double rlo = fmax(floor(ra) - 1.0, (double)rp.row0);
      double rhi = fmin(floor(rb) + 1.0, (double)(rp.row0 + rp.nrows - 1));
      if (clo <= chi && rlo <= rhi) {
        m.x = cell_tile(rp, (int64_t)clo);
        m.y = cell_tile(rp, (int64_t)chi);
        m.z = cell_tile(rp, (int64_t)rlo);
        m.w = cell_tile(rp, (int64_t)rhi);
        nc = (int64_t)(m.y - m.x + 1) * (m.w - m.z + 1);
        nb = m.w - m.z + 1;
      }
    }
    mbb[k] = m;
    ncand[k] = nc;
    nband[k] = nb;
    s_m = m;
  }
  __syncthreads();
  return s_m;
}

// One CTA per polygon (step 2, first pass), one pass over its vertices: each vertex v starts the
// edge v -> next(v) (implicit closure), written in canonical orientation with its exact straddled
// row interval within the shard, and joins the MBB's partial min / max; then the MBB's tile
// rectangle.  The polygon's (edge, tile row) band entries count towards *n_entries only when the
// rectangle meets the shard (nothing downstream reads the edges of the others).  (Rings are
// contiguous, so no search is needed.)
__global__ void __launch_bounds__(256) k_mbb_edges(const int32_t* __restrict__ pro, const int32_t* __restrict__ rvo,
                                                   const double* __restrict__ x, const double* __restrict__ y, Geo g,
                                                   RasterP rp, int4* __restrict__ mbb, int64_t* __restrict__ ncand,
                                                   int64_t* __restrict__ nband, int64_t rA, int64_t rB,
                                                   Edge* __restrict__ edges, int2* __restrict__ erows,
                                                   int64_t* __restrict__ n_entries) {
  const int k = blockIdx.x;
  const int T = rp.T;
  double xmn = INFINITY, xmx = -INFINITY, ymn = INFINITY, ymx = -INFINITY;
  int span = 0;
  for (int ring = pro[k]; ring < pro[k + 1]; ++ring) {
    const int a = rvo[ring], b = rvo[ring + 1];
    for (int v = a + threadIdx.x; v < b; v += blockDim.x) {
      const int nxt = (v + 1 < b) ? v + 1 : a;
      const double x0 = x[v], y0 = y[v], x1 = x[nxt], y1 = y[nxt];
      xmn = fmin(xmn, x0); xmx = fmax(xmx, x0);
      ymn = fmin(ymn, y0); ymx = fmax(ymx, y0);
      Edge e;
      if (y0 <= y1) { e.xa = x0; e.ya = y0; e.xb = x1; e.yb = y1; }
      else          { e.xa = x1; e.ya = y1; e.xb = x0; e.yb = y0; }
      edges[v] = e;
      const int2 rr = straddle_rows(g, e.ya, e.yb, rA, rB);
      erows[v] = rr;
      span += (rr.x < rr.y) ? (cell_tile(rp, rr.y - 1) - cell_tile(rp, rr.x) + 1) : 0;
    }
  }
  const int4 m = mbb_reduce(k, rvo[pro[k + 1]] - rvo[pro[k]], xmn, xmx, ymn, ymx, g, rp, mbb, ncand, nband);
  if (m.x > m.y) return;
  for (int o = 16; o > 0; o >>= 1) span += __shfl_xor_sync(0xffffffffu, span, o);
  if ((threadIdx.x & 31) == 0 && span) atomicAdd(reinterpret_cast<unsigned long long*>(n_entries),
                                                 (unsigned long long)span);
}

// Band lists, one CTA per polygon: its vertices (= edges) are contiguous, and the counters of its
// bands (one per tile row of its MBB) live in shared memory, so the heavily repeated increments of
// consecutive edges never leave the SM.  mode 0: counts -> band_cnt, and band_first = how many of
// them straddle the band's FIRST row (the row k_classify tests; -1: not sorted, polygons with more
// bands than kSmemBands, which use global atomics directly); mode 1: fill band_edges from band_off,
// those first-row edges at the front of the list.
constexpr int kSmemBands = 2048;
__global__ void __launch_bounds__(256) k_poly_bands(const int32_t* __restrict__ pro, const int32_t* __restrict__ rvo,
                                                    const int2* __restrict__ erows, const int4* __restrict__ mbb,
                                                    const int64_t* __restrict__ band_base, int T, uint32_t tmul,
                                                    uint32_t tsh, int mode,
                                                    int32_t* __restrict__ band_cnt, const int32_t* __restrict__ band_off,
                                                    int32_t* __restrict__ band_edges, int32_t* __restrict__ band_poly,
                                                    int32_t* __restrict__ band_first) {
  __shared__ int32_t sc[kSmemBands];
  __shared__ int32_t sb[kSmemBands];  // first-row edges (mode 0) / cursor of the rest (mode 1)
  const int k = blockIdx.x;
  const int4 m = mbb[k];
  if (m.x > m.y) return;
  const int nb = m.w - m.z + 1;
  const int64_t bb = band_base[k];
  const bool in_smem = nb <= kSmemBands;
  if (mode == 0)
    for (int i = threadIdx.x; i < nb; i += blockDim.x) band_poly[bb + i] = k;  // band -> polygon
  if (in_smem) {
    for (int i = threadIdx.x; i < nb; i += blockDim.x) {
      sc[i] = 0;
      sb[i] = 0;
    }
    __syncthreads();
  } else if (mode == 0) {
    for (int i = threadIdx.x; i < nb; i += blockDim.x) band_first[bb + i] = -1;
  }
  const int vb = rvo[pro[k]], ve = rvo[pro[k + 1]];
  for (int v = vb + threadIdx.x; v < ve; v += blockDim.x) {
    const int2 rr = erows[v];
    if (rr.x >= rr.y) continue;
    const int tr1 = magic_q((uint32_t)(rr.y - 1), tmul, tsh);
    for (int tr = magic_q((uint32_t)rr.x, tmul, tsh); tr <= tr1; ++tr) {
      const int i = tr - m.z;
      const int64_t r = (int64_t)tr * T;  // the band's first row
      const bool first = rr.x <= r && r < rr.y;
      if (mode == 0) {
        if (in_smem) {
          atomicAdd(&sc[i], 1);
          if (first) atomicAdd(&sb[i], 1);
        } else {
          atomicAdd(&band_cnt[bb + i], 1);
        }
      } else if (in_smem) {
        const int pos = first ? band_off[bb + i] + atomicAdd(&sc[i], 1)
                              : band_off[bb + i] + band_first[bb + i] + atomicAdd(&sb[i], 1);
        band_edges[pos] = v;
      } else {
        band_edges[atomicAdd(&band_cnt[bb + i], 1)] = v;  // band_cnt = cursors
      }
    }
  }
  if (in_smem && mode == 0) {
    __syncthreads();
    for (int i = threadIdx.x; i < nb; i += blockDim.x) {
      band_cnt[bb + i] = sc[i];
      band_first[bb + i] = sb[i];
    }
  }
}

// Mark INTERSECT: every tile whose cell rectangle comes within one cell of the edge's bounding
// box (x AND y extent — an edge lying between two centre rows straddles none of them but still
// separates them).  A tile touched by no edge box is crossed by no part of the boundary, so the
// exact parity is constant on it, and every straddling edge is >= 1 cell left/right of its
// centres, so the computed parity equals the exact one at every centre.
// class: 0 = not yet classified, 1 = inside, 2 = intersect, 3 = outside.
__global__ void __launch_bounds__(256) k_mark(const int32_t* __restrict__ pro, const int32_t* __restrict__ rvo,
                                              const Edge* __restrict__ edges, Geo g, RasterP rp,
                                              const int4* __restrict__ mbb, const int64_t* __restrict__ cand_off,
                                              uint8_t* __restrict__ cls) {
  const int k = blockIdx.x;
  const int4 m = mbb[k];
  if (m.x > m.y) return;
  const int wk = m.y - m.x + 1;
  const int64_t base = cand_off[k];
  const int vb = rvo[pro[k]], ve = rvo[pro[k + 1]];
  for (int v = vb + threadIdx.x; v < ve; v += blockDim.x) {
    const Edge e = edges[v];
    // fractional cell coordinates of the edge's bbox: reciprocals instead of divisions (a few ulp
    // of a coordinate, far inside the one-cell margin below)
#if ZH_MARK_RCP
    double ca = (fmin(e.xa, e.xb) - g.gt0) * g.igt1, cb = (fmax(e.xa, e.xb) - g.gt0) * g.igt1;
    double ra = (e.ya - g.gt3) * g.igt5, rb = (e.yb - g.gt3) * g.igt5;
#else
    double ca = (fmin(e.xa, e.xb) - g.gt0) / g.gt1, cb = (fmax(e.xa, e.xb) - g.gt0) / g.gt1;
    double ra = (e.ya - g.gt3) / g.gt5, rb = (e.yb - g.gt3) / g.gt5;
#endif
    if (ca > cb) { double t = ca; ca = cb; cb = t; }
    if (ra > rb) { double t = ra; ra = rb; rb = t; }
    const double clo = fmax(floor(ca) - 1.0, (double)m.x * rp.T);
    const double chi = fmin(floor(cb) + 1.0, (double)(m.y + 1) * rp.T - 1.0);
    const double rlo = fmax(floor(ra) - 1.0, (double)m.z * rp.T);
    const double rhi = fmin(floor(rb) + 1.0, (double)(m.w + 1) * rp.T - 1.0);
    if (clo > chi || rlo > rhi) continue;
    const int tc_lo = cell_tile(rp, (int64_t)clo), tc_hi = cell_tile(rp, (int64_t)chi);
    const int tr_lo = cell_tile(rp, (int64_t)rlo), tr_hi = cell_tile(rp, (int64_t)rhi);
    for (int tr = tr_lo; tr <= tr_hi; ++tr)
      for (int tc = tc_lo; tc <= tc_hi; ++tc) cls[base + (int64_t)(tr - m.z) * wk + (tc - m.x)] = 2;
  }
}

// One WARP per band (polygon k, tile row tr; 4 bands per CTA): classify the unmarked tiles of the
// row by the exact PIP status of their first cell (r = tr*T, c = tc*T).  For each band edge
// straddling r the toggled tiles {tc : xc(tc*T) < xi} form a prefix (gt1 > 0) or a suffix (gt1 < 0)
// of the row, recorded as flips of a difference bitmap D (per warp, shared memory);
// parity(j) = XOR_{i > j} D[i].  (A band's work is a few hundred edges and a handful of tiles: a
// warp, not a CTA, and no block-wide barrier.)
constexpr int kClassifyWarps = 4;
__global__ void __launch_bounds__(32 * kClassifyWarps) k_classify(
    const Edge* __restrict__ edges, const int2* __restrict__ erows, const int32_t* __restrict__ band_off,
    const int32_t* __restrict__ band_edges, const int64_t* __restrict__ band_base,
    const int32_t* __restrict__ band_poly, const int32_t* __restrict__ band_first, int64_t n_bands, Geo g, RasterP rp,
    const int4* __restrict__ mbb,
    const int64_t* __restrict__ cand_off, uint8_t* __restrict__ cls, int dwords) {
  extern __shared__ uint32_t Dall[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t band = (int64_t)blockIdx.x * (blockDim.x >> 5) + wid;
  if (band >= n_bands) return;  // whole warps exit: only __syncwarp below
  uint32_t* D = Dall + wid * dwords;
  const int k = band_poly[band];
  const int4 m = mbb[k];
  const int tr = m.z + (int)(band - band_base[k]);
  const int wk = m.y - m.x + 1;
  const int64_t rrep = (int64_t)tr * rp.T;
  const double yc = row_centre(g, rrep);
  const bool s = g.gt1 > 0;
  const int nd = (wk >> 5) + 1;
  for (int i = lane; i < nd; i += 32) D[i] = 0;
  __syncwarp();
  const int e0 = band_off[band], nf = band_first[band];
  const int e1 = nf >= 0 ? e0 + nf : band_off[band + 1];  // the edges straddling row rrep come first
  for (int i = e0 + lane; i < e1; i += 32) {
    const int v = band_edges[i];
    const int2 rr = erows[v];
    if (!(rr.x <= rrep && rrep < rr.y)) continue;
    const Edge e = edges[v];
    const double xi = intercept(e, yc);
    // pred(j) = ((xc(c_j) < xi) == s), true on a prefix of j in [0, wk)
    const double est = ((xi - g.gt0) * g.igt1 - g.ox) / rp.T - (double)m.x;  // a guess (first_false is exact)
    const int64_t jb = first_false(0, wk, clamp_est(est, 0, wk), [&](int64_t j) {
      return (col_centre(g, (int64_t)(m.x + j) * rp.T) < xi) == s;
    });
    if (jb > 0) atomicXor(&D[jb >> 5], 1u << (jb & 31));
    if (!s) atomicXor(&D[wk >> 5], 1u << (wk & 31));
  }
  __syncwarp();
  if (lane == 0) {
    uint32_t carry = 0;
    for (int wi = (wk >> 5); wi >= 0; --wi) {
      uint32_t t = D[wi];
      t ^= t >> 1; t ^= t >> 2; t ^= t >> 4; t ^= t >> 8; t ^= t >> 16;
      D[wi] = (t >> 1) ^ (carry ? 0xFFFFFFFFu : 0u);
      carry ^= (t & 1u);
    }
  }
  __syncwarp();
  uint8_t* c = cls + cand_off[k] + (int64_t)(tr - m.z) * wk;
  for (int j = lane; j < wk; j += 32) {
    if (c[j] == 0) c[j] = ((D[j >> 5] >> (j & 31)) & 1u) ? 1 : 3;
  }
}

__global__ void k_force_isect(uint8_t* cls, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    cls[i] = 2;
}

__global__ void k_flags(const uint8_t* __restrict__ cls, int64_t n, uint64_t* __restrict__ flags) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint8_t c = cls[i];
    flags[i] = (c == 1 ? 1ull : 0ull) | (c == 2 ? (1ull << 32) : 0ull);
  }
}

__global__ void k_compact(const uint8_t* __restrict__ cls, const uint64_t* __restrict__ pos, int64_t n,
                          const int64_t* __restrict__ cand_off, int P, const int4* __restrict__ mbb, RasterP rp,
                          int2* __restrict__ inside, int2* __restrict__ isect, int64_t* __restrict__ totals) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint8_t c = cls[i];
    if (i == n - 1) {
      const uint64_t tot = pos[i] + ((c == 1) ? 1ull : 0ull) + ((c == 2) ? (1ull << 32) : 0ull);
      totals[0] = (int64_t)(tot & 0xFFFFFFFFull);
      totals[1] = (int64_t)(tot >> 32);
    }
    if (c != 1 && c != 2) continue;
    const int k = (int)(upper_bound_i64(cand_off, P + 1, i) - 1);
    const int4 m = mbb[k];
    const int wk = m.y - m.x + 1;
    const int64_t j = i - cand_off[k];
    const int tr = m.z + (int)(j / wk), tc = m.x + (int)(j % wk);
    const int tile = (tr - rp.tr0) * rp.TC + tc;
    const uint64_t p = pos[i];
    if (c == 1) inside[p & 0xFFFFFFFFull] = make_int2(tile, k);
    else isect[p >> 32] = make_int2(tile, k);
  }
}

__global__ void k_totals1(const int64_t* cand_off, const int64_t* band_base, int P, int64_t* out) {
  out[0] = cand_off[P];
  out[1] = band_base[P];
}

struct Want6 {
  int64_t v[6];
};
__global__ void k_check_counts(const int64_t* __restrict__ counts, Want6 want, int n, uint32_t* __restrict__ flag) {
  for (int i = 0; i < n; ++i)
    if (counts[i] != want.v[i]) *flag = 1u;
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

}  // namespace zh


namespace zh {

cudaError_t launch_check_counts(Ctx& c, const int64_t* counts, const int64_t* want, int n) {
  if (!c.d_flag.p) return cudaErrorInvalidValue;  // allocated and zeroed by zh_create
  Want6 w = {};
  for (int i = 0; i < n && i < 6; ++i) w.v[i] = want[i];
  k_check_counts<<<1, 1, 0, c.stream>>>(counts, w, n < 6 ? n : 6, c.d_flag.as<uint32_t>());
  c.launches += 1;
  return cudaGetLastError();
}

// Threads per CTA of the one-CTA-per-polygon step-2 kernels (k_mbb_edges, k_poly_bands, k_mark):
// about one edge per thread or more — 256 for county-sized rings (CONUS: ~3,000 vertices), fewer
// for small ones (PIP-stress: ~760), where a 256-thread CTA mostly waits at its barriers.
static int s2_threads(const Ctx& c) {
#ifdef ZH_S2_THREADS
  return ZH_S2_THREADS;
#else
  const int64_t avg = c.P > 0 ? (int64_t)c.V / c.P : 0;
  return avg >= 1536 ? 256 : (avg >= 384 ? 128 : 64);
#endif
}

cudaError_t launch_pairs_phase1(Ctx& c) {
  cudaError_t e;
  const int V = c.V, P = c.P;
  if ((e = c.d_edges.ensure(sizeof(Edge) * (size_t)V)) != cudaSuccess) return e;
  if ((e = c.d_erows.ensure(sizeof(int2) * (size_t)V)) != cudaSuccess) return e;
  if ((e = c.d_mbb.ensure(sizeof(int4) * (size_t)P)) != cudaSuccess) return e;
  if ((e = c.d_ncand.ensure(sizeof(int64_t) * ((size_t)P + 1))) != cudaSuccess) return e;
  if ((e = c.d_nband.ensure(sizeof(int64_t) * ((size_t)P + 1))) != cudaSuccess) return e;
  if ((e = c.d_cand_off.ensure(sizeof(int64_t) * ((size_t)P + 1))) != cudaSuccess) return e;
  if ((e = c.d_band_base.ensure(sizeof(int64_t) * ((size_t)P + 1))) != cudaSuccess) return e;
  if ((e = c.d_counts.ensure(sizeof(int64_t) * 8)) != cudaSuccess) return e;
  const int64_t rA = c.rp.row0, rB = c.rp.row0 + c.rp.nrows;
  // one trailing zero so that the exclusive scans over P + 1 entries end with the totals
  cudaMemsetAsync(c.d_ncand.as<int64_t>() + P, 0, sizeof(int64_t), c.stream);
  cudaMemsetAsync(c.d_nband.as<int64_t>() + P, 0, sizeof(int64_t), c.stream);
  cudaMemsetAsync(c.d_counts.p, 0, sizeof(int64_t) * 8, c.stream);
  if (ZH_CARVEOUT >= 0) {
    prep_kernel(k_mbb_edges, 0);
    prep_kernel(k_poly_bands, 0);
    prep_kernel(k_mark, 0);
    prep_kernel(k_classify, 0);
  }
  if (P > 0) {
    k_mbb_edges<<<P, s2_threads(c), 0, c.stream>>>(c.d_pro.as<int32_t>(), c.d_rvo.as<int32_t>(), c.d_x.as<double>(),
                                         c.d_y.as<double>(), c.geo, c.rp, c.d_mbb.as<int4>(), c.d_ncand.as<int64_t>(),
                                         c.d_nband.as<int64_t>(), rA, rB, c.d_edges.as<Edge>(), c.d_erows.as<int2>(),
                                         c.d_counts.as<int64_t>() + 2);
    c.launches += 1;
  }
  if ((e = excl_scan<int64_t>(c, c.d_ncand.as<int64_t>(), c.d_cand_off.as<int64_t>(), P + 1)) != cudaSuccess) return e;
  if ((e = excl_scan<int64_t>(c, c.d_nband.as<int64_t>(), c.d_band_base.as<int64_t>(), P + 1)) != cudaSuccess) return e;
  k_totals1<<<1, 1, 0, c.stream>>>(c.d_cand_off.as<int64_t>(), c.d_band_base.as<int64_t>(), P,
                                   c.d_counts.as<int64_t>());
  c.launches += 1;
  return cudaGetLastError();
}

cudaError_t launch_pairs_phase2(Ctx& c) {
  cudaError_t e;
  const int V = c.V, P = c.P;
  const int64_t nc = c.n_cand, nb = c.n_bands, ne = c.n_band_entries;
  if ((e = c.d_band_cnt.ensure(sizeof(int32_t) * ((size_t)nb + 1))) != cudaSuccess) return e;
  if ((e = c.d_band_off.ensure(sizeof(int32_t) * ((size_t)nb + 1))) != cudaSuccess) return e;
  if ((e = c.d_band_cur.ensure(sizeof(int32_t) * ((size_t)nb + 1))) != cudaSuccess) return e;
  if ((e = c.d_band_edges.ensure(sizeof(int32_t) * (size_t)ne)) != cudaSuccess) return e;
  if ((e = c.d_band_poly.ensure(sizeof(int32_t) * ((size_t)nb + 1))) != cudaSuccess) return e;
  if ((e = c.d_band_first.ensure(sizeof(int32_t) * ((size_t)nb + 1))) != cudaSuccess) return e;
  if ((e = c.d_class.ensure((size_t)nc)) != cudaSuccess) return e;
  if ((e = c.d_flags.ensure(sizeof(uint64_t) * (size_t)nc)) != cudaSuccess) return e;
  if ((e = c.d_flag_pos.ensure(sizeof(uint64_t) * (size_t)nc)) != cudaSuccess) return e;
  // The band (polygon, tile-row) edge lists.
  cudaMemsetAsync(c.d_band_cnt.p, 0, sizeof(int32_t) * ((size_t)nb + 1), c.stream);
  if (V > 0 && nb > 0) {
    k_poly_bands<<<P, s2_threads(c), 0, c.stream>>>(c.d_pro.as<int32_t>(), c.d_rvo.as<int32_t>(), c.d_erows.as<int2>(),
                                          c.d_mbb.as<int4>(), c.d_band_base.as<int64_t>(), c.rp.T, c.rp.t_mul, c.rp.t_sh, 0,
                                          c.d_band_cnt.as<int32_t>(), nullptr, nullptr, c.d_band_poly.as<int32_t>(),
                                          c.d_band_first.as<int32_t>());
    c.launches += 1;
  }
  if (nb > 0) {
    if ((e = excl_scan<int32_t>(c, c.d_band_cnt.as<int32_t>(), c.d_band_off.as<int32_t>(), nb + 1)) != cudaSuccess)
      return e;
    cudaMemcpyAsync(c.d_band_cur.p, c.d_band_off.p, sizeof(int32_t) * (size_t)nb, cudaMemcpyDeviceToDevice, c.stream);
    if (V > 0) {
      k_poly_bands<<<P, s2_threads(c), 0, c.stream>>>(c.d_pro.as<int32_t>(), c.d_rvo.as<int32_t>(), c.d_erows.as<int2>(),
                                            c.d_mbb.as<int4>(), c.d_band_base.as<int64_t>(), c.rp.T, c.rp.t_mul, c.rp.t_sh, 1,
                                            c.d_band_cur.as<int32_t>(), c.d_band_off.as<int32_t>(),
                                            c.d_band_edges.as<int32_t>(), nullptr, c.d_band_first.as<int32_t>());
      c.launches += 1;
    }
  }
  if (nc > 0) {
    if (c.force_isect) {
      k_force_isect<<<grid_for(nc, 256), 256, 0, c.stream>>>(c.d_class.as<uint8_t>(), nc);
      c.launches += 1;
    } else {
      cudaMemsetAsync(c.d_class.p, 0, (size_t)nc, c.stream);
      if (V > 0) {
        k_mark<<<P, s2_threads(c), 0, c.stream>>>(c.d_pro.as<int32_t>(), c.d_rvo.as<int32_t>(), c.d_edges.as<Edge>(), c.geo,
                                       c.rp, c.d_mbb.as<int4>(),
                                                      c.d_cand_off.as<int64_t>(), c.d_class.as<uint8_t>());
        c.launches += 1;
      }
      const int dwords = c.rp.TC / 32 + 2;
      // warps (bands) per CTA: 4, fewer when a band's bitmap is large (TC <= 2^20: zh_create)
      const int nw = (int)std::max<int64_t>(1, std::min<int64_t>(kClassifyWarps, 48 * 1024 / (4 * dwords)));
      const size_t smem = sizeof(uint32_t) * (size_t)dwords * nw;
      prep_kernel(k_classify, smem);
      k_classify<<<(unsigned)((nb + nw - 1) / nw), 32 * nw, smem, c.stream>>>(
          c.d_edges.as<Edge>(), c.d_erows.as<int2>(), c.d_band_off.as<int32_t>(), c.d_band_edges.as<int32_t>(),
          c.d_band_base.as<int64_t>(), c.d_band_poly.as<int32_t>(), c.d_band_first.as<int32_t>(), nb, c.geo, c.rp,
          c.d_mbb.as<int4>(),
          c.d_cand_off.as<int64_t>(), c.d_class.as<uint8_t>(), dwords);
      c.launches += 1;
    }
    k_flags<<<grid_for(nc, 256), 256, 0, c.stream>>>(c.d_class.as<uint8_t>(), nc, c.d_flags.as<uint64_t>());
    c.launches += 1;
    if ((e = excl_scan<uint64_t>(c, c.d_flags.as<uint64_t>(), c.d_flag_pos.as<uint64_t>(), nc)) != cudaSuccess)
      return e;
    // lists are sized by the candidate count (an upper bound of both)
    if ((e = c.d_inside.ensure(sizeof(int2) * (size_t)nc)) != cudaSuccess) return e;
    if ((e = c.d_isect.ensure(sizeof(int2) * (size_t)nc)) != cudaSuccess) return e;
    k_compact<<<grid_for(nc, 256), 256, 0, c.stream>>>(c.d_class.as<uint8_t>(), c.d_flag_pos.as<uint64_t>(), nc,
                                                      c.d_cand_off.as<int64_t>(), P, c.d_mbb.as<int4>(), c.rp,
                                                      c.d_inside.as<int2>(), c.d_isect.as<int2>(),
                                                      c.d_counts.as<int64_t>() + 4);
    c.launches += 1;
  } else {
    cudaMemsetAsync(c.d_counts.as<int64_t>() + 4, 0, 2 * sizeof(int64_t), c.stream);
  }
  return cudaGetLastError();
}

}  // namespace zh
