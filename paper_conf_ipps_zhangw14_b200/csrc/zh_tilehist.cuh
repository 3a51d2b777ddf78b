// zh_tilehist.cuh — the per-tile histogram pass shared by step 1 and the fused pure-tile kernel.
#pragma once
#include "zh_internal.cuh"

#ifndef ZH_TILE_WIDE
#define ZH_TILE_WIDE 1
#endif
#ifndef ZH_TILE_WROWS
#define ZH_TILE_WROWS 2  // rows (32-byte loads) in flight per thread in the wide tile pass (step 1)
#endif
#ifndef ZH_PURE_WROWS
#define ZH_PURE_WROWS 4  // the same for k_fused_pure (A/B: 2 / 3 / 4 rows -> 2.95 / 2.98 / 2.88 ms)
#endif

namespace zh {

// Histogram of one tile (tile-row trl, tile-column tc of the shard) into the shared histogram
// `sh` (HistLayout, zeroed and synchronised by the caller).  Shared by step 1 (k_tile_hist) and
// the fused pure-tile kernel (k_fused.cu).
// kMode: 0 generic bins (width 1), 1 generic bins (width > 1), 2 + kForm: packed bins (fast_idx2)
template <int kMode, int WR = ZH_TILE_WROWS>
__device__ __forceinline__ void tile_histogram(uint32_t* __restrict__ sh, const RasterP& rp, const BinP& bp,
                                               const FastBins& fb, int trl, int tc) {
  const int64_t r0 = (int64_t)(rp.tr0 + trl) * rp.T;
  const int h = (int)min((int64_t)rp.T, rp.row0 + rp.nrows - r0);
  const int64_t c0 = (int64_t)tc * rp.T;
  const int w = (int)min((int64_t)rp.T, rp.cols - c0);

  const uint32_t dummy = (uint32_t)hist_dummy(bp.nbins) + (threadIdx.x & 31);
  const uint32_t dum2 = dummy * 0x10001u;
  auto count = [&](const uint4& q, uint32_t skip) {
    if (kMode >= 2) {
      if (skip == 0) count8_fast<kMode - 2, false>(sh, q, 0, fb, dum2);
      else count8_fast<kMode - 2, true>(sh, q, skip, fb, dum2);
    } else {
      count8_generic<kMode == 0>(sh, q, skip, bp, dummy);
    }
  };

  const int64_t k0 = c0 >> 3, k1 = (c0 + w + 7) >> 3;
  const int nk = (int)(k1 - k0);
  const int16_t* base = rp.data + (r0 - rp.row0) * rp.pitch + k0 * 8;
  const int64_t pitch = rp.pitch;

#if ZH_TILE_WIDE
  // 16-cell segments, one 32-byte load each (sm_100 LDG.256), two rows in flight: the same bytes
  // and registers as four 16-byte vectors with half the load instructions (full, aligned tiles)
  if (kMode >= 2 && rp.wide && (c0 & 15) == 0 && (w & 15) == 0 && (w >> 4) <= (int)blockDim.x) {
    const int nk2 = w >> 4, rpi2 = blockDim.x / nk2;
    const int kk2 = threadIdx.x % nk2, rs2 = threadIdx.x / nk2;
    if (rs2 < rpi2) {
      const int16_t* p = rp.data + (r0 - rp.row0 + rs2) * rp.pitch + c0 + kk2 * 16;
      const int64_t step = (int64_t)rpi2 * rp.pitch;
      int r = rs2;
      for (; r + (WR - 1) * rpi2 < h; r += WR * rpi2, p += WR * step) {
        uint4 a[WR], b[WR];
#pragma unroll
        for (int u = 0; u < WR; ++u) ld_stream32(p + u * step, a[u], b[u]);
#pragma unroll
        for (int u = 0; u < WR; ++u) {
          count8_fast<kMode - 2, false>(sh, a[u], 0, fb, dum2);
          count8_fast<kMode - 2, false>(sh, b[u], 0, fb, dum2);
        }
      }
      for (; r < h; r += rpi2, p += step) {
        uint4 a0, a1;
        ld_stream32(p, a0, a1);
        count8_fast<kMode - 2, false>(sh, a0, 0, fb, dum2);
        count8_fast<kMode - 2, false>(sh, a1, 0, fb, dum2);
      }
    }
    return;
  }
#endif
  if (nk <= (int)blockDim.x) {
    const int rpi = blockDim.x / nk;  // rows per block iteration
    const int kk = threadIdx.x % nk, rs = threadIdx.x / nk;
    if (rs < rpi) {
      const uint32_t skip = cols_skip8((k0 + kk) * 8, c0, w);
      const int16_t* p = base + (int64_t)rs * pitch + kk * 8;
      const int64_t step = (int64_t)rpi * pitch;
      int r = rs;
      for (; r + 3 * rpi < h; r += 4 * rpi) {
        const uint4 q0 = ld_stream16(p);
        const uint4 q1 = ld_stream16(p + step);
        const uint4 q2 = ld_stream16(p + 2 * step);
        const uint4 q3 = ld_stream16(p + 3 * step);
        p += 4 * step;
        count(q0, skip);
        count(q1, skip);
        count(q2, skip);
        count(q3, skip);
      }
      for (; r < h; r += rpi, p += step) count(ld_stream16(p), skip);
    }
  } else {
    for (int r = 0; r < h; ++r) {
      for (int kk = threadIdx.x; kk < nk; kk += blockDim.x)
        count(ld_stream16(base + (int64_t)r * pitch + kk * 8), cols_skip8((k0 + kk) * 8, c0, w));
    }
  }
}

}  // namespace zh
