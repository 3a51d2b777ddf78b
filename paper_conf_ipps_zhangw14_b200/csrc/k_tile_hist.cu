// k_tile_hist.cu — step 1: per-tile histograms (§III.A, Fig. 2).
//
// tile_hist[t][b] = #{ cells of tile t : bin(v) = b }, t = local tile row * TC + tile column.
//
// Paper design (prior art): one thread block per tile, 256 threads, a global-memory atomicAdd per
// cell.  B200 design: one CTA per tile with the tile's histogram privatised in SHARED memory
// (B_pad x 4 bytes, 20 KB at B = 5000), raster read as 16-byte streaming vectors (8 int16 cells,
// ld.global.nc.L1::no_allocate), 4 independent 16-byte loads in flight per thread, runs of equal
// bins inside each vector merged in registers before the shared atomic, and one coalesced 16-byte
// store pass per tile (no global zeroing pass).  HBM-bound: 2 B/cell read + 4*B_pad/T^2 B/cell
// written.
#include "zh_ctx.h"

namespace zh {

template <bool kW1>
__global__ void __launch_bounds__(512) k_tile_hist(RasterP rp, BinP bp, int B_pad,
                                                   uint32_t* __restrict__ tile_hist) {
  extern __shared__ __align__(16) uint32_t sh[];
  const int tile = blockIdx.x;
  const int tr = tile / rp.TC, tc = tile - tr * rp.TC;
  const int64_t r0 = (int64_t)(rp.tr0 + tr) * rp.T;
  const int h = (int)min((int64_t)rp.T, rp.row0 + rp.nrows - r0);
  const int64_t c0 = (int64_t)tc * rp.T;
  const int w = (int)min((int64_t)rp.T, rp.cols - c0);

  for (int i = threadIdx.x * 4; i < B_pad; i += blockDim.x * 4)
    *reinterpret_cast<uint4*>(&sh[i]) = make_uint4(0, 0, 0, 0);
  __syncthreads();

  const int64_t k0 = c0 >> 3, k1 = (c0 + w + 7) >> 3;
  const int nk = (int)(k1 - k0);
  const int16_t* base = rp.data + (r0 - rp.row0) * rp.pitch + k0 * 8;
  const int64_t pitch = rp.pitch;

  if (nk <= (int)blockDim.x) {
    const int rpi = blockDim.x / nk;  // rows per block iteration
    const int kk = threadIdx.x % nk, rs = threadIdx.x / nk;
    if (rs < rpi) {
      const int64_t cs = (k0 + kk) * 8;
      uint32_t valid = 0xFFu;
      if (cs < c0) valid &= (0xFFu << (int)(c0 - cs)) & 0xFFu;
      if (cs + 8 > c0 + w) valid &= 0xFFu >> (int)(cs + 8 - (c0 + w));
      const int16_t* p = base + kk * 8;
      int r = rs;
      for (; r + 3 * rpi < h; r += 4 * rpi) {
        const uint4 q0 = ld_stream16(p + (int64_t)r * pitch);
        const uint4 q1 = ld_stream16(p + (int64_t)(r + rpi) * pitch);
        const uint4 q2 = ld_stream16(p + (int64_t)(r + 2 * rpi) * pitch);
        const uint4 q3 = ld_stream16(p + (int64_t)(r + 3 * rpi) * pitch);
        count8<kW1>(sh, q0, valid, bp);
        count8<kW1>(sh, q1, valid, bp);
        count8<kW1>(sh, q2, valid, bp);
        count8<kW1>(sh, q3, valid, bp);
      }
      for (; r < h; r += rpi) count8<kW1>(sh, ld_stream16(p + (int64_t)r * pitch), valid, bp);
    }
  } else {
    for (int r = 0; r < h; ++r) {
      for (int kk = threadIdx.x; kk < nk; kk += blockDim.x) {
        const int64_t cs = (k0 + kk) * 8;
        uint32_t valid = 0xFFu;
        if (cs < c0) valid &= (0xFFu << (int)(c0 - cs)) & 0xFFu;
        if (cs + 8 > c0 + w) valid &= 0xFFu >> (int)(cs + 8 - (c0 + w));
        count8<kW1>(sh, ld_stream16(base + (int64_t)r * pitch + kk * 8), valid, bp);
      }
    }
  }
  __syncthreads();
  uint32_t* dst = tile_hist + (int64_t)tile * B_pad;
  for (int i = threadIdx.x * 4; i < B_pad; i += blockDim.x * 4)
    *reinterpret_cast<uint4*>(&dst[i]) = *reinterpret_cast<const uint4*>(&sh[i]);
}

cudaError_t launch_tile_hist(Ctx& c) {
  if (c.n_tiles == 0) return cudaSuccess;
  const size_t smem = (size_t)c.B_pad * 4;
  const int threads = 512;
  if (c.bp.width == 1) {
    auto k = k_tile_hist<true>;
    if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    k<<<(unsigned)c.n_tiles, threads, smem, c.stream>>>(c.rp, c.bp, c.B_pad, c.d_tile_hist.as<uint32_t>());
  } else {
    auto k = k_tile_hist<false>;
    if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    k<<<(unsigned)c.n_tiles, threads, smem, c.stream>>>(c.rp, c.bp, c.B_pad, c.d_tile_hist.as<uint32_t>());
  }
  c.launches += 1;
  return cudaGetLastError();
}

}  // namespace zh
