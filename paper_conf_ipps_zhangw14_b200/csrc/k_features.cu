// k_features.cu — what the per-polygon histograms are for (SURVEY.md §8f-4, §I ¶1):
// the classic zonal summary ("min, max, average, count and standard deviation") and histogram
// feature distances ("these histograms can further be used as feature vectors for ... computing
// various distance measurements which can be used for subsequent clustering").
//
// Everything is computed from the exact integer histogram with a stated rounding sequence, so the
// results are reproducible bit for bit (zh.h documents each formula):
//   * zonal summary: k_zonal_summary, from k_zonal_stats' exact integers (count, S1 = sum b H[b],
//     S2 = sum b^2 H[b] as 128 bits): mean = lo + width * (S1 / n); std = width * (sqrt(D) / n)
//     with D = n S2 - S1^2 exact in 128 bits — no cancellation anywhere;
//   * L1 / EMD-1D between normalised histograms: N / n_a / n_b with the exact 128-bit integer
//     N = sum_b |X_a[b] n_b - X_b[b] n_a| (X = H for L1, the cumulative counts for EMD);
//   * chi^2: per-bin doubles from exact integer numerators (order of the sum unspecified).
// All pairs (the clustering input) run as a tiled P x P kernel: 32 x 32 polygon pairs per CTA,
// 32-bin chunks of both row blocks staged in shared memory, 4 pairs per thread.  When every
// count is < 2^32 (any county-sized zone) the products are single 32 x 32 -> 64-bit multiplies.
#include <type_traits>

#include "zh_ctx.h"

namespace zh {

struct U128 {
  unsigned long long lo, hi;
};

__device__ __forceinline__ void add128(U128& a, unsigned long long v) {
  const unsigned long long s = a.lo + v;
  a.hi += (s < v) ? 1ull : 0ull;
  a.lo = s;
}

__device__ __forceinline__ void add128(U128& a, const U128& b) {
  const unsigned long long s = a.lo + b.lo;
  a.hi += b.hi + ((s < b.lo) ? 1ull : 0ull);
  a.lo = s;
}

__device__ __forceinline__ U128 mul64x64(unsigned long long a, unsigned long long b) {
  U128 r;
  r.lo = a * b;
  r.hi = __umul64hi(a, b);
  return r;
}

// |x - y| for 128-bit x, y
__device__ __forceinline__ U128 absdiff128(const U128& x, const U128& y) {
  const bool ge = (x.hi > y.hi) || (x.hi == y.hi && x.lo >= y.lo);
  const U128& a = ge ? x : y;
  const U128& b = ge ? y : x;
  U128 r;
  r.lo = a.lo - b.lo;
  r.hi = a.hi - b.hi - ((a.lo < b.lo) ? 1ull : 0ull);
  return r;
}

// Round-to-nearest-even conversion of a 128-bit unsigned integer to double: the top 64 bits with
// a sticky bit for everything below (it lies under the half-ulp bit of the 53-bit result, so the
// rounding decision is that of the exact value), then an exact power-of-two scaling.
__device__ __forceinline__ double u128_to_double_rn(const U128& v) {
  if (v.hi == 0) return __ull2double_rn(v.lo);
  const int lz = __clzll((long long)v.hi);
  const int s = 64 - lz;  // bits to drop
  unsigned long long m = (v.hi << lz) | (lz ? (v.lo >> s) : 0ull);
  const unsigned long long below = lz ? (v.lo << lz) : v.lo;  // the dropped low bits
  if (below) m |= 1ull;
  return ldexp(__ull2double_rn(m), s);
}

// ---- zonal summary -------------------------------------------------------------------------
__global__ void k_zonal_summary(const int64_t* __restrict__ stats, int P, double lo, double width,
                                double* __restrict__ out) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= P) return;
  const int64_t* st = stats + (int64_t)k * ZH_NSTATS;
  double* o = out + (int64_t)k * ZH_NSUMMARY;
  const unsigned long long n = (unsigned long long)st[0];
  o[0] = __ull2double_rn(n);
  if (n == 0) {
    const double nan = __longlong_as_double(0x7ff8000000000000ll);
    o[1] = o[2] = o[3] = o[4] = o[5] = nan;
    return;
  }
  // bins are small integers: lo + b * width is exact in double (|lo| <= 2^30, b < 2^16, width < 2^31)
  o[1] = __dadd_rn(lo, __dmul_rn((double)st[1], width));
  o[2] = __dadd_rn(lo, __dmul_rn((double)st[2], width));
  o[3] = __dadd_rn(lo, __dmul_rn((double)st[3], width));
  const unsigned long long s1 = (unsigned long long)st[4];
  const double nd = __ull2double_rn(n);
  o[4] = __dadd_rn(lo, __dmul_rn(width, __ddiv_rn(__ull2double_rn(s1), nd)));
  // D = n * S2 - S1^2 >= 0 (Cauchy-Schwarz), exactly; S2 < 2^72 and n < 2^40 keep it in 128 bits
  const unsigned long long s2lo = (unsigned long long)st[5], s2hi = (unsigned long long)st[6];
  U128 a = mul64x64(n, s2lo);
  a.hi += n * s2hi;
  const U128 b = mul64x64(s1, s1);
  const U128 d = absdiff128(a, b);
  o[5] = __dmul_rn(width, __ddiv_rn(__dsqrt_rn(u128_to_double_rn(d)), nd));
}

// ---- histogram rows as 64-bit counts: H (or its running sum along the bins, for EMD) --------
template <bool kU64>
__device__ __forceinline__ unsigned long long hval(const void* h, int64_t i) {
  return kU64 ? reinterpret_cast<const unsigned long long*>(h)[i]
              : (unsigned long long)reinterpret_cast<const uint32_t*>(h)[i];
}

// cdf[k][b] = sum_{b' <= b} H[k][b'] — one CTA per polygon, 1024-bin chunks scanned by a warp
// shuffle scan per warp and a carry across the chunk.
template <bool kU64>
__global__ void __launch_bounds__(1024) k_row_cdf(const void* __restrict__ h, int nbins,
                                                  unsigned long long* __restrict__ cdf) {
  const int64_t row = (int64_t)blockIdx.x * nbins;
  __shared__ unsigned long long wsum[32];
  __shared__ unsigned long long carry;
  if (threadIdx.x == 0) carry = 0;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (int base = 0; base < nbins; base += blockDim.x) {
    const int b = base + threadIdx.x;
    unsigned long long v = b < nbins ? hval<kU64>(h, row + b) : 0ull;
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long t = __shfl_up_sync(0xffffffffu, v, o);
      if (lane >= o) v += t;
    }
    if (lane == 31) wsum[wid] = v;
    __syncthreads();
    if (wid == 0) {
      unsigned long long s = lane < (int)(blockDim.x >> 5) ? wsum[lane] : 0ull;
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long t = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o) s += t;
      }
      wsum[lane] = s;  // inclusive warp prefix
    }
    __syncthreads();
    const unsigned long long c0 = carry;
    const unsigned long long pre = (wid ? wsum[wid - 1] : 0ull) + c0;
    if (b < nbins) cdf[row + b] = v + pre;
    __syncthreads();
    if (threadIdx.x == 0) carry = c0 + wsum[(blockDim.x >> 5) - 1];
    __syncthreads();
  }
}

// ---- per-bin terms of one (a, b) pair --------------------------------------------------------
// x = X_a[bin] * n_b, y = X_b[bin] * n_a (exact); L1/EMD accumulate |x - y|, chi^2 adds
// RN(RN(d)^2 / RN(s)) with d = x - y, s = x + y.
template <int kKind, bool kNarrow>
struct PairAcc {
  U128 n{0, 0};
  double c = 0.0;
  __device__ __forceinline__ void add(unsigned long long xa, unsigned long long xb, unsigned long long na,
                                      unsigned long long nb) {
    U128 x, y;
    if (kNarrow) {  // everything < 2^32: one 32x32 -> 64-bit product each
      x.lo = (unsigned long long)(uint32_t)xa * (uint32_t)nb;
      y.lo = (unsigned long long)(uint32_t)xb * (uint32_t)na;
      x.hi = y.hi = 0;
      if (kKind != ZH_DIST_CHI2) {
        add128(n, x.lo >= y.lo ? x.lo - y.lo : y.lo - x.lo);
        return;
      }
    } else {
      x = mul64x64(xa, nb);
      y = mul64x64(xb, na);
      if (kKind != ZH_DIST_CHI2) {
        add128(n, absdiff128(x, y));
        return;
      }
    }
    if (xa == 0 && xb == 0) return;
    const double d = u128_to_double_rn(absdiff128(x, y));
    U128 s = x;
    add128(s, y);
    c = __dadd_rn(c, __ddiv_rn(__dmul_rn(d, d), u128_to_double_rn(s)));
  }
};

template <int kKind>
__device__ __forceinline__ double finish(const U128& n, double c, unsigned long long na, unsigned long long nb) {
  if (na == 0 || nb == 0) return __longlong_as_double(0x7ff8000000000000ll);
  // divide by the smaller count first: the rounding is then symmetric in (a, b)
  const double d1 = __ull2double_rn(na < nb ? na : nb), d2 = __ull2double_rn(na < nb ? nb : na);
  if (kKind == ZH_DIST_CHI2) return 0.5 * __ddiv_rn(__ddiv_rn(c, d1), d2);
  return __ddiv_rn(__ddiv_rn(u128_to_double_rn(n), d1), d2);
}

// List mode: one warp per (a, b) pair, lanes over bins; partial sums combined in a fixed order.
template <int kKind, bool kNarrow>
__global__ void __launch_bounds__(256) k_dist_list(const void* __restrict__ X, int kind_src_u64, int nbins,
                                                   const int64_t* __restrict__ stats,
                                                   const int32_t* __restrict__ ia, const int32_t* __restrict__ ib,
                                                   int64_t n, double* __restrict__ out) {
  const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (i >= n) return;
  const int a = ia[i], b = ib[i];
  const unsigned long long na = (unsigned long long)stats[(int64_t)a * ZH_NSTATS];
  const unsigned long long nb = (unsigned long long)stats[(int64_t)b * ZH_NSTATS];
  const bool wide = kind_src_u64 != 0;  // X holds uint64 (H in u64 mode, or the CDF)
  PairAcc<kKind, kNarrow> acc;
  const int64_t ra = (int64_t)a * nbins, rb = (int64_t)b * nbins;
  for (int bin = lane; bin < nbins; bin += 32) {
    const unsigned long long xa = wide ? hval<true>(X, ra + bin) : hval<false>(X, ra + bin);
    const unsigned long long xb = wide ? hval<true>(X, rb + bin) : hval<false>(X, rb + bin);
    acc.add(xa, xb, na, nb);
  }
  for (int o = 16; o > 0; o >>= 1) {
    U128 t;
    t.lo = __shfl_down_sync(0xffffffffu, acc.n.lo, o);
    t.hi = __shfl_down_sync(0xffffffffu, acc.n.hi, o);
    add128(acc.n, t);
    acc.c = __dadd_rn(acc.c, __shfl_down_sync(0xffffffffu, acc.c, o));
  }
  if (lane == 0) out[i] = finish<kKind>(acc.n, acc.c, na, nb);
}

// All pairs: CTA (bx, by) with by <= bx computes the 32 x 32 block of pairs (a in rows of by,
// b in rows of bx) and writes it and its mirror.  256 threads (16 x 16), 4 pairs each.
constexpr int kDT = 32;  // polygons per block side
constexpr int kDB = 32;  // bins per staged chunk
template <int kKind, bool kNarrow>
__global__ void __launch_bounds__(256) k_dist_all(const void* __restrict__ X, int src_u64, int nbins,
                                                  const int64_t* __restrict__ stats, int P,
                                                  double* __restrict__ out) {
  const int bx = blockIdx.x, by = blockIdx.y;
  if (by > bx) return;
  using V = typename std::conditional<kNarrow, uint32_t, unsigned long long>::type;
  __shared__ V sa[kDB][kDT + 1], sb[kDB][kDT + 1];
  __shared__ unsigned long long sna[kDT], snb[kDT];
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const int a0 = by * kDT, b0 = bx * kDT;
  if (threadIdx.x < kDT) {
    const int a = a0 + threadIdx.x, b = b0 + threadIdx.x;
    sna[threadIdx.x] = a < P ? (unsigned long long)stats[(int64_t)a * ZH_NSTATS] : 0ull;
    snb[threadIdx.x] = b < P ? (unsigned long long)stats[(int64_t)b * ZH_NSTATS] : 0ull;
  }
  __syncthreads();
  unsigned long long na[2], nb[2];
  for (int i = 0; i < 2; ++i) {
    na[i] = sna[ty + 16 * i];
    nb[i] = snb[tx + 16 * i];
  }
  PairAcc<kKind, kNarrow> acc[2][2];
  for (int c0 = 0; c0 < nbins; c0 += kDB) {
    // stage X[a0 .. a0+31][c0 .. c0+31] and X[b0 ..][..] transposed (bin-major): lanes read
    // consecutive bins of one row (coalesced)
    for (int e = threadIdx.x; e < kDT * kDB; e += blockDim.x) {
      const int r = e / kDB, cb = e % kDB;
      const int bin = c0 + cb;
      const int a = a0 + r, b = b0 + r;
      unsigned long long va = 0, vb = 0;
      if (bin < nbins) {
        if (a < P) va = src_u64 ? hval<true>(X, (int64_t)a * nbins + bin) : hval<false>(X, (int64_t)a * nbins + bin);
        if (b < P) vb = src_u64 ? hval<true>(X, (int64_t)b * nbins + bin) : hval<false>(X, (int64_t)b * nbins + bin);
      }
      sa[cb][r] = (V)va;
      sb[cb][r] = (V)vb;
    }
    __syncthreads();
#pragma unroll 4
    for (int cb = 0; cb < kDB; ++cb) {
      const unsigned long long xa0 = sa[cb][ty], xa1 = sa[cb][ty + 16];
      const unsigned long long xb0 = sb[cb][tx], xb1 = sb[cb][tx + 16];
      acc[0][0].add(xa0, xb0, na[0], nb[0]);
      acc[0][1].add(xa0, xb1, na[0], nb[1]);
      acc[1][0].add(xa1, xb0, na[1], nb[0]);
      acc[1][1].add(xa1, xb1, na[1], nb[1]);
    }
    __syncthreads();
  }
  for (int i = 0; i < 2; ++i)
    for (int j = 0; j < 2; ++j) {
      const int a = a0 + ty + 16 * i, b = b0 + tx + 16 * j;
      if (a >= P || b >= P) continue;
      const double d = finish<kKind>(acc[i][j].n, acc[i][j].c, na[i], nb[j]);
      out[(int64_t)a * P + b] = d;
      out[(int64_t)b * P + a] = d;
    }
}

cudaError_t launch_zonal_summary(Ctx& c, const int64_t* dstats, double* dout) {
  if (c.P == 0) return cudaSuccess;
  k_zonal_summary<<<(c.P + 127) / 128, 128, 0, c.stream>>>(dstats, c.P, (double)c.bp.lo, (double)c.bp.width, dout);
  c.launches += 1;
  return cudaGetLastError();
}

template <int kKind, bool kNarrow>
static void launch_dist_kind(Ctx& c, const void* X, int src_u64, const int64_t* dstats, const int32_t* ia,
                             const int32_t* ib, int64_t n, double* dout) {
  if (ia) {
    const int64_t blocks = (n * 32 + 255) / 256;
    k_dist_list<kKind, kNarrow><<<(unsigned)blocks, 256, 0, c.stream>>>(X, src_u64, c.bp.nbins, dstats, ia, ib, n, dout);
  } else {
    const unsigned nt = (unsigned)((c.P + kDT - 1) / kDT);
    k_dist_all<kKind, kNarrow><<<dim3(nt, nt), 256, 0, c.stream>>>(X, src_u64, c.bp.nbins, dstats, c.P, dout);
  }
  c.launches += 1;
}

// X: the output histogram (kind L1 / CHI2) or, for EMD, its row CDFs built here in d_cdf.
cudaError_t launch_hist_distance(Ctx& c, int kind, const int64_t* dstats, bool narrow, const int32_t* ia,
                                 const int32_t* ib, int64_t n, double* dout) {
  cudaError_t e;
  const void* X = c.d_out;
  int src_u64 = c.out_u64;
  if (kind == ZH_DIST_EMD) {
    if ((e = c.d_cdf.ensure((size_t)c.P * c.bp.nbins * 8)) != cudaSuccess) return e;
    if (c.P > 0) {
      if (c.out_u64) k_row_cdf<true><<<c.P, 1024, 0, c.stream>>>(c.d_out, c.bp.nbins, c.d_cdf.as<unsigned long long>());
      else k_row_cdf<false><<<c.P, 1024, 0, c.stream>>>(c.d_out, c.bp.nbins, c.d_cdf.as<unsigned long long>());
      c.launches += 1;
    }
    X = c.d_cdf.p;
    src_u64 = 1;
  }
  if (c.P == 0 || (ia && n == 0)) return cudaGetLastError();
  switch (kind) {
    case ZH_DIST_L1:
      if (narrow) launch_dist_kind<ZH_DIST_L1, true>(c, X, src_u64, dstats, ia, ib, n, dout);
      else launch_dist_kind<ZH_DIST_L1, false>(c, X, src_u64, dstats, ia, ib, n, dout);
      break;
    case ZH_DIST_EMD:
      if (narrow) launch_dist_kind<ZH_DIST_EMD, true>(c, X, src_u64, dstats, ia, ib, n, dout);
      else launch_dist_kind<ZH_DIST_EMD, false>(c, X, src_u64, dstats, ia, ib, n, dout);
      break;
    default:
      if (narrow) launch_dist_kind<ZH_DIST_CHI2, true>(c, X, src_u64, dstats, ia, ib, n, dout);
      else launch_dist_kind<ZH_DIST_CHI2, false>(c, X, src_u64, dstats, ia, ib, n, dout);
      break;
  }
  return cudaGetLastError();
}

}  // namespace zh
