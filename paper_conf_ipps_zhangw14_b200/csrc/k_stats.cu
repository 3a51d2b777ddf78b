// k_stats.cu — zonal statistics from the per-polygon histograms.
//
// The paper motivates zonal histograms as an extension of classic zonal statistics — "min, max,
// average, count and standard deviation" per zone (§I ¶1) — and as feature vectors
// for further analysis.  Everything here is derived from the histogram in exact integer
// arithmetic, in units of bin indices b (value of a bin = lo + b * width), so the GPU result is
// bit-identical to any other exact evaluation:
//   [0] count   = sum_b H[b]
//   [1] min_bin = smallest b with H[b] > 0 (-1 if count = 0)
//   [2] max_bin = largest  b with H[b] > 0 (-1 if count = 0)
//   [3] median  = smallest b with sum_{b' <= b} H[b'] >= (count + 1) / 2 (lower median; -1 if empty)
//   [4] sum_b   = sum_b b * H[b]                    (< 2^63 for any raster that fits in HBM)
//   [5] sumsq_lo, [6] sumsq_hi = sum_b b^2 * H[b]   (128-bit, two 64-bit words)
//   [7] nonzero = number of bins with H[b] > 0
// Mean and variance in value units follow exactly from these (zh.py: ZonalHistogram.zonal_stats).
#include "zh_ctx.h"

namespace zh {

template <bool kU64>
__global__ void __launch_bounds__(256) k_zonal_stats(const void* __restrict__ out, int nbins,
                                                     int64_t* __restrict__ stats) {
  const int k = blockIdx.x;
  const int64_t row = (int64_t)k * nbins;
  __shared__ unsigned long long s_cnt[256];
  __shared__ int s_min[256], s_max[256], s_nz[256];
  __shared__ unsigned long long s_sum[256];
  __shared__ unsigned __int128 s_sq[256];
  // pass 1: moments, extremes
  unsigned long long cnt = 0, sum = 0;
  unsigned __int128 sq = 0;
  int mn = 0x7FFFFFFF, mx = -1, nz = 0;
  for (int b = threadIdx.x; b < nbins; b += blockDim.x) {
    const unsigned long long h = kU64 ? reinterpret_cast<const unsigned long long*>(out)[row + b]
                                      : (unsigned long long)reinterpret_cast<const uint32_t*>(out)[row + b];
    if (!h) continue;
    cnt += h;
    sum += (unsigned long long)b * h;
    sq += (unsigned __int128)((unsigned long long)b * (unsigned long long)b) * h;
    mn = min(mn, b);
    mx = max(mx, b);
    ++nz;
  }
  s_cnt[threadIdx.x] = cnt;
  s_sum[threadIdx.x] = sum;
  s_sq[threadIdx.x] = sq;
  s_min[threadIdx.x] = mn;
  s_max[threadIdx.x] = mx;
  s_nz[threadIdx.x] = nz;
  __syncthreads();
  for (int o = blockDim.x / 2; o > 0; o >>= 1) {
    if ((int)threadIdx.x < o) {
      s_cnt[threadIdx.x] += s_cnt[threadIdx.x + o];
      s_sum[threadIdx.x] += s_sum[threadIdx.x + o];
      s_sq[threadIdx.x] += s_sq[threadIdx.x + o];
      s_min[threadIdx.x] = min(s_min[threadIdx.x], s_min[threadIdx.x + o]);
      s_max[threadIdx.x] = max(s_max[threadIdx.x], s_max[threadIdx.x + o]);
      s_nz[threadIdx.x] += s_nz[threadIdx.x + o];
    }
    __syncthreads();
  }
  const unsigned long long total = s_cnt[0];
  // pass 2: lower median by a blocked prefix sum (thread t owns a contiguous run of bins)
  __shared__ int s_med;
  if (threadIdx.x == 0) s_med = -1;
  __syncthreads();
  if (total > 0) {
    const unsigned long long target = (total + 1) / 2;
    const int per = (nbins + blockDim.x - 1) / blockDim.x;
    const int b0 = threadIdx.x * per, b1 = min(nbins, b0 + per);
    unsigned long long mine = 0;
    for (int b = b0; b < b1; ++b)
      mine += kU64 ? reinterpret_cast<const unsigned long long*>(out)[row + b]
                   : (unsigned long long)reinterpret_cast<const uint32_t*>(out)[row + b];
    s_cnt[threadIdx.x] = mine;
    __syncthreads();
    if (threadIdx.x == 0) {  // exclusive scan of 256 partial counts (cheap, once per polygon)
      unsigned long long run = 0;
      for (int i = 0; i < (int)blockDim.x; ++i) {
        const unsigned long long v = s_cnt[i];
        s_cnt[i] = run;
        run += v;
      }
    }
    __syncthreads();
    unsigned long long run = s_cnt[threadIdx.x];
    if (run < target) {
      for (int b = b0; b < b1; ++b) {
        run += kU64 ? reinterpret_cast<const unsigned long long*>(out)[row + b]
                    : (unsigned long long)reinterpret_cast<const uint32_t*>(out)[row + b];
        if (run >= target) {  // exactly one thread's run crosses the target
          s_med = b;
          break;
        }
      }
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int64_t* st = stats + (int64_t)k * 8;
    st[0] = (int64_t)total;
    st[1] = total ? s_min[0] : -1;
    st[2] = total ? s_max[0] : -1;
    st[3] = s_med;
    st[4] = (int64_t)s_sum[0];
    st[5] = (int64_t)(unsigned long long)(s_sq[0] & 0xFFFFFFFFFFFFFFFFull);
    st[6] = (int64_t)(unsigned long long)(s_sq[0] >> 64);
    st[7] = s_nz[0];
  }
}

cudaError_t launch_zonal_stats(Ctx& c, int64_t* dstats) {
  if (c.P == 0) return cudaSuccess;
  if (c.out_u64) k_zonal_stats<true><<<c.P, 256, 0, c.stream>>>(c.d_out, c.bp.nbins, dstats);
  else k_zonal_stats<false><<<c.P, 256, 0, c.stream>>>(c.d_out, c.bp.nbins, dstats);
  c.launches += 1;
  return cudaGetLastError();
}

}  // namespace zh
