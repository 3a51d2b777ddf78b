// zh_internal.cuh — device-side building blocks shared by libzh's kernels (sm_100a).
//
// Nothing here is shared with oracle/ (the CPU oracle is written independently from the paper).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/zh.h"

namespace zh {

// ----------------------------------------------------------------------------------------------
// Geometry: cell centres and Franklin's intercept, each operation an explicit IEEE binary64
// round-to-nearest op (__d*_rn) so that nvcc cannot contract them into FMAs (DESIGN.md §3 R7).
// ----------------------------------------------------------------------------------------------
struct Geo {
  double gt0, gt1, gt3, gt5;
};

__device__ __forceinline__ double col_centre(const Geo& g, int64_t c) {
  return __dadd_rn(g.gt0, __dmul_rn(__dadd_rn((double)c, 0.5), g.gt1));
}
__device__ __forceinline__ double row_centre(const Geo& g, int64_t r) {
  return __dadd_rn(g.gt3, __dmul_rn(__dadd_rn((double)r, 0.5), g.gt5));
}

// Canonical edge (ya <= yb), Fig. 5 predicate in lower-endpoint-first orientation (R8).
struct Edge {
  double xa, ya, xb, yb;
};

// xi = (xb - xa) * (yc - ya) / (yb - ya) + xa, left to right (R8).
__device__ __forceinline__ double intercept(const Edge& e, double yc) {
  const double t1 = __dsub_rn(e.xb, e.xa);
  const double t2 = __dsub_rn(yc, e.ya);
  const double t3 = __dmul_rn(t1, t2);
  const double t4 = __dsub_rn(e.yb, e.ya);
  const double t5 = __ddiv_rn(t3, t4);
  return __dadd_rn(t5, e.xa);
}

// Smallest i in [lo, hi] with pred(i) == false, for a predicate that is true on a prefix of
// [lo, hi) and false after it (returns hi when it is true on all of [lo, hi)).  `est` is a guess;
// a short walk from it usually lands on the answer, otherwise bisection finds it, so the result
// is exact whatever the guess.
template <class Pred>
__device__ __forceinline__ int64_t first_false(int64_t lo, int64_t hi, int64_t est, Pred pred) {
  int64_t i = est < lo ? lo : (est > hi ? hi : est);
#pragma unroll 1
  for (int s = 0; s < 4; ++s) {
    if (i > lo && !pred(i - 1)) --i;
    else if (i < hi && pred(i)) ++i;
    else return i;
  }
  int64_t a = lo - 1, b = hi;  // pred(a) true (or a = lo-1), pred(b) false (or b = hi)
#pragma unroll 1
  while (b - a > 1) {
    const int64_t m = a + ((b - a) >> 1);
    if (pred(m)) a = m; else b = m;
  }
  return b;
}

// ----------------------------------------------------------------------------------------------
// Bin mapping (R3/R4): -1 = not counted.
// ----------------------------------------------------------------------------------------------
struct BinP {
  int32_t lo, width, nbins, use_nodata, nodata, drop;
};

template <bool kW1>
__device__ __forceinline__ int bin_of(int v, const BinP& b) {
  if (b.use_nodata && v == b.nodata) return -1;
  int d = v - b.lo;
  if (d < 0) return b.drop ? -1 : 0;
  int q = kW1 ? d : d / b.width;
  if (q >= b.nbins) return b.drop ? -1 : b.nbins - 1;
  return q;
}

// 16-byte streaming load (read-once raster data: do not allocate in L1).
__device__ __forceinline__ uint4 ld_stream16(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ int cell_of(const uint4& q, int j) {
  const uint32_t w = (j < 2) ? q.x : (j < 4) ? q.y : (j < 6) ? q.z : q.w;
  return (int)(int16_t)(w >> ((j & 1) * 16));
}

// Count the valid cells (bit j of `valid`) of an 8-cell vector into a shared-memory histogram.
// Runs of equal bins inside the vector are merged first (DEM neighbours are often equal, so this
// removes same-address serialisation of the shared atomics).
template <bool kW1>
__device__ __forceinline__ void count8(uint32_t* __restrict__ hist, const uint4& q, uint32_t valid,
                                       const BinP& bp) {
  int prev = -1;
  uint32_t run = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    int b = ((valid >> j) & 1u) ? bin_of<kW1>(cell_of(q, j), bp) : -1;
    if (b == prev) {
      ++run;
    } else {
      if (prev >= 0) atomicAdd(&hist[prev], run);
      prev = b;
      run = 1;
    }
  }
  if (prev >= 0) atomicAdd(&hist[prev], run);
}

// ----------------------------------------------------------------------------------------------
// Kernel parameter blocks
// ----------------------------------------------------------------------------------------------
struct RasterP {
  const int16_t* data;  // points at row `row0` of the full raster (device)
  int64_t rows, cols, pitch, row0, nrows;
  int32_t T, TC, tr0, TRn;  // tile size, tile columns, first tile row, tile rows in shard
};

}  // namespace zh
