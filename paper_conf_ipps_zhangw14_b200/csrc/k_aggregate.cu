// k_aggregate.cu — step 3: out[k][b] += sum of tile_hist[t][b] over the inside tiles t of k
// (§III.C, Fig. 4 right, UpdateHistKernel).
//
// Paper design (prior art): one block per polygon, a serial loop over all of the polygon's inside
// tiles — a big western county with hundreds of inside tiles is one long block.  B200 design:
// the (polygon, tile)-sorted inside list is cut into flat chunks of CH entries (chunks may span
// polygon boundaries), crossed with 1024-bin slices; a thread owns 4 consecutive bins (one 16-byte
// load per tile row slice), keeps running sums in registers and adds them to `out` with one
// global atomic per non-zero bin whenever the polygon changes (most DEM bins of a tile are zero).
// HBM-bound: 4*B_pad bytes read per inside pair.
#include "zh_ctx.h"

namespace zh {

template <bool kU64>
__global__ void __launch_bounds__(256) k_aggregate(const uint32_t* __restrict__ tile_hist, int B_pad,
                                                   const int2* __restrict__ inside, int64_t n_inside, int chunk,
                                                   void* __restrict__ out, int nbins) {
  const int64_t start = (int64_t)blockIdx.x * chunk;
  const int64_t end = min(start + chunk, n_inside);
  const int b = (blockIdx.y * blockDim.x + threadIdx.x) * 4;
  if (b >= B_pad) return;
  uint32_t a0 = 0, a1 = 0, a2 = 0, a3 = 0;
  int cur = inside[start].y;
  auto flush = [&](int k) {
    const int64_t row = (int64_t)k * nbins;
    const uint32_t v[4] = {a0, a1, a2, a3};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (v[j] && b + j < nbins) {
        if (kU64) atomicAdd(reinterpret_cast<unsigned long long*>(out) + row + b + j, (unsigned long long)v[j]);
        else atomicAdd(reinterpret_cast<uint32_t*>(out) + row + b + j, v[j]);
      }
    }
  };
  int64_t i = start;
  for (; i + 4 <= end; i += 4) {
    const int2 p0 = inside[i], p1 = inside[i + 1], p2 = inside[i + 2], p3 = inside[i + 3];
    const uint4 q0 = __ldg(reinterpret_cast<const uint4*>(tile_hist + (int64_t)p0.x * B_pad + b));
    const uint4 q1 = __ldg(reinterpret_cast<const uint4*>(tile_hist + (int64_t)p1.x * B_pad + b));
    const uint4 q2 = __ldg(reinterpret_cast<const uint4*>(tile_hist + (int64_t)p2.x * B_pad + b));
    const uint4 q3 = __ldg(reinterpret_cast<const uint4*>(tile_hist + (int64_t)p3.x * B_pad + b));
    const int2 ps[4] = {p0, p1, p2, p3};
    const uint4 qs[4] = {q0, q1, q2, q3};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (ps[j].y != cur) {
        flush(cur);
        a0 = a1 = a2 = a3 = 0;
        cur = ps[j].y;
      }
      a0 += qs[j].x; a1 += qs[j].y; a2 += qs[j].z; a3 += qs[j].w;
    }
  }
  for (; i < end; ++i) {
    const int2 p = inside[i];
    const uint4 q = __ldg(reinterpret_cast<const uint4*>(tile_hist + (int64_t)p.x * B_pad + b));
    if (p.y != cur) {
      flush(cur);
      a0 = a1 = a2 = a3 = 0;
      cur = p.y;
    }
    a0 += q.x; a1 += q.y; a2 += q.z; a3 += q.w;
  }
  flush(cur);
}

cudaError_t launch_aggregate(Ctx& c) {
  if (c.n_inside == 0) return cudaSuccess;
  // chunk so that a uint32 running sum cannot overflow: chunk * T^2 < 2^32
  const double cells = (double)c.rp.T * (double)c.rp.T;
  int chunk = 64;
  while (chunk > 1 && (double)chunk * cells >= 4294967295.0) chunk >>= 1;
  const int threads = 256;
  dim3 grid((unsigned)((c.n_inside + chunk - 1) / chunk), (unsigned)((c.B_pad + threads * 4 - 1) / (threads * 4)));
  if (c.out_u64)
    k_aggregate<true><<<grid, threads, 0, c.stream>>>(c.d_tile_hist.as<uint32_t>(), c.B_pad, c.d_inside.as<int2>(),
                                                       c.n_inside, chunk, c.d_out, c.bp.nbins);
  else
    k_aggregate<false><<<grid, threads, 0, c.stream>>>(c.d_tile_hist.as<uint32_t>(), c.B_pad, c.d_inside.as<int2>(),
                                                        c.n_inside, chunk, c.d_out, c.bp.nbins);
  c.launches += 1;
  return cudaGetLastError();
}

}  // namespace zh
