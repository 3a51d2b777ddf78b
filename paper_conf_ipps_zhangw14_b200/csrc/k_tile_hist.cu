// k_tile_hist.cu — step 1: per-tile histograms (§III.A, Fig. 2).
//
// tile_hist[t][b] = #{ cells of tile t : bin(v) = b }, t = local tile row * TC + tile column.
//
// Paper design (prior art): one thread block per tile, 256 threads, a global-memory atomicAdd per
// cell.  B200 design: one CTA per tile with the tile's histogram privatised in SHARED memory
// (20 KB at B = 5000); the raster is read as 16-byte streaming vectors (8 int16 cells,
// ld.global.nc.L1::no_allocate), 4 independent vectors in flight per thread; bins are computed
// two cells at a time with packed 16x2 min/max/add (VIMNMX.S16x2 / VIADD.16x2) and a zero-detect
// for nodata; every cell then issues exactly one shared atomic with no predicate or branch —
// cells that are not counted go to one of 32 per-lane dummy slots (zh_internal.cuh, HistLayout).
// The histogram leaves with one coalesced 16-byte store pass per tile (no global zeroing pass).
// HBM-bound: 2 B/cell read + 4*B_pad/T^2 B/cell written.
#include "zh_ctx.h"
#include "zh_tilehist.cuh"

namespace zh {

template <int kMode>
__global__ void __launch_bounds__(512, 3) k_tile_hist(RasterP rp, BinP bp, FastBins fb, int B_pad,
                                                      uint32_t* __restrict__ tile_hist) {
  extern __shared__ __align__(16) uint32_t sh[];
  const int HW = hist_words(bp.nbins);
  const int tile = blockIdx.x;
  const int trl = tile_row(rp, tile), tc = tile - trl * rp.TC;
  for (int i = threadIdx.x * 4; i < HW; i += blockDim.x * 4)
    *reinterpret_cast<uint4*>(&sh[i]) = make_uint4(0, 0, 0, 0);
  __syncthreads();
  tile_histogram<kMode>(sh, rp, bp, fb, trl, tc);
  __syncthreads();
  uint32_t* dst = tile_hist + (int64_t)tile * B_pad;
  for (int i = threadIdx.x * 4; i < B_pad; i += blockDim.x * 4)
    *reinterpret_cast<uint4*>(&dst[i]) = *reinterpret_cast<const uint4*>(&sh[kOff + i]);
}

template <int kMode>
static void launch_mode(Ctx& c, size_t smem, int threads) {
  auto k = k_tile_hist<kMode>;
  prep_kernel(k, smem);
  k<<<(unsigned)c.n_tiles, threads, smem, c.stream>>>(c.rp, c.bp, make_fast_bins(c.bp), c.B_pad,
                                                      c.d_tile_hist.as<uint32_t>());
}

cudaError_t launch_tile_hist(Ctx& c) {
  if (c.n_tiles == 0) return cudaSuccess;
  const size_t smem = (size_t)hist_words(c.bp.nbins) * 4;
  const int threads = 512;
  if (fast_bins_ok(c.bp)) {
    const FastBins f = make_fast_bins(c.bp);
    if (f.bias) launch_mode<4>(c, smem, threads);
    else if (c.bp.use_nodata) launch_mode<3>(c, smem, threads);
    else launch_mode<2>(c, smem, threads);
  } else {
    if (c.bp.width == 1) launch_mode<0>(c, smem, threads);
    else launch_mode<1>(c, smem, threads);
  }
  c.launches += 1;
  return cudaGetLastError();
}

}  // namespace zh
