// k_pip.cu — step 4: cell-in-polygon test and histogram update for intersecting pairs
// (§III.D, Fig. 5, pip_test_kernel).
//
// For each intersecting (tile, polygon k) pair and each cell of the tile whose centre passes the
// even-odd ray-crossing test against all rings of k, out[k][bin(v)] += 1.
//
// Paper design (prior art): one block per polygon, one thread per cell, and for every cell a loop
// over ALL polygon vertices in global memory with float coordinates; the histogram update is a
// non-atomic read-modify-write (a race).  B200 design, bit-identical to the per-cell test:
//   * one CTA per intersecting pair; only the edges of the pair's band (edges that straddle one
//     of the tile's centre rows, built in step 2) are visited;
//   * the crossing test `xc < xi` depends on the cell only through xc, and xc is monotone in the
//     column, so for each (edge, row) the crossed cells form a prefix (gt1 > 0) or suffix
//     (gt1 < 0) of the row: the exact boundary column is found with the SAME xc(c) expression
//     (first_false), and recorded as a flip in a per-row difference bitmap in shared memory;
//     a suffix-XOR turns it into the per-cell parity (inside) bits.  Work per pair is
//     O(#(edge,row) crossings + cells) instead of O(cells x edges);
//   * edges entirely left / right of the tile's centres (with half a cell of margin, far above
//     the intercept's rounding) skip the division;
//   * the cells are then streamed exactly like step 1 (16-byte vectors, packed 16x2 bin mapping,
//     one branch-free shared atomic per cell; vectors with no inside cell are not even loaded)
//     into a CTA-private shared histogram, flushed once per pair with one global atomic per
//     non-zero bin (no race).
#include "zh_ctx.h"
#include "zh_parity.cuh"

namespace zh {

struct PipP {
  RasterP rp;
  Geo g;
  BinP bp;
  const int2* isect;
  const int4* mbb;
  const int64_t* band_base;
  const int32_t* band_off;
  const int32_t* band_edges;
  const Edge* edges;
  const int2* erows;
  void* out;
  FastBins fb;
  int B_pad;
  int wpr;  // bitmap words per row = T/32 + 1
  int rc;   // rows per chunk
  const int64_t* n_dev;  // device count of pairs (grid may be an upper bound), or nullptr
};

template <int kMode, bool kU64>  // kMode as in k_tile_hist: 0/1 generic (w1 / w>1), 2 + kForm packed
__global__ void __launch_bounds__(256) k_pip(PipP p) {
  if (p.n_dev && (int64_t)blockIdx.x >= *p.n_dev) return;
  extern __shared__ __align__(16) uint32_t sh[];
  __shared__ LongQ lq;
  const int HW = hist_words(p.bp.nbins);
  uint32_t* hist = sh;
  uint32_t* bm = sh + HW;
  if (threadIdx.x == 0) lq.n = 0;
  const RasterP& rp = p.rp;
  const Geo& g = p.g;

  const int2 pr = p.isect[blockIdx.x];
  const int tile = pr.x, k = pr.y;
  const TileGeom t = tile_geom(rp, g, tile);
  const int64_t r0 = t.r0, c0 = t.c0;
  const int h = t.h, w = t.w;
  const int4 m = p.mbb[k];
  const int64_t band = p.band_base[k] + ((int)(r0 / rp.T) - m.z);
  const int e0 = p.band_off[band], e1 = p.band_off[band + 1];

  for (int i = threadIdx.x * 4; i < HW; i += blockDim.x * 4)
    *reinterpret_cast<uint4*>(&hist[i]) = make_uint4(0, 0, 0, 0);
  const uint32_t dummy = (uint32_t)hist_dummy(p.bp.nbins) + (threadIdx.x & 31);
  const uint32_t dum2 = dummy * 0x10001u;

  const int64_t k0 = c0 >> 3, k1 = (c0 + w + 7) >> 3;
  const int nk = (int)(k1 - k0);
  const int64_t pitch = rp.pitch;
  const FastBins fb = p.fb;

  for (int cr = 0; cr < h; cr += p.rc) {
    const int ch = min(p.rc, h - cr);
    const int64_t rlo = r0 + cr, rhi = rlo + ch;  // global rows of this chunk
    for (int i = threadIdx.x; i < ch * p.wpr; i += blockDim.x) bm[i] = 0;
    __syncthreads();
    crossings_to_bitmap(bm, p.wpr, e0, e1, p.band_edges, p.edges, p.erows, g, t, rlo, rhi, &lq);
    suffix_xor_rows(bm, p.wpr, ch);
    __syncthreads();
    // ---- cells: stream the chunk's rows, count inside cells (fully-outside vectors are not read)
    const int16_t* base = rp.data + (rlo - rp.row0) * pitch + k0 * 8;
    if (nk <= (int)blockDim.x) {
      const int rpi = blockDim.x / nk;
      const int kk = threadIdx.x % nk, rs = threadIdx.x / nk;
      if (rs < rpi) {
        const int64_t cs = (k0 + kk) * 8;
        const uint32_t cskip = cols_skip8(cs, c0, w);
        const int lc0 = (int)(cs - c0);
        const int16_t* ptr = base + (int64_t)rs * pitch + kk * 8;
        const int64_t step = (int64_t)rpi * pitch;
        int lr = rs;
        // two rows per iteration: both skip masks first, then both loads in flight
        for (; lr + rpi < ch; lr += 2 * rpi, ptr += 2 * step) {
          const uint32_t s0 = cskip | (~bits8(bm + lr * p.wpr, p.wpr, lc0) & 0xFFu);
          const uint32_t s1 = cskip | (~bits8(bm + (lr + rpi) * p.wpr, p.wpr, lc0) & 0xFFu);
          uint4 q0 = make_uint4(0, 0, 0, 0), q1 = make_uint4(0, 0, 0, 0);
          if (s0 != 0xFFu) q0 = ld_stream16(ptr);
          if (s1 != 0xFFu) q1 = ld_stream16(ptr + step);
          if (s0 != 0xFFu) {
            if (kMode >= 2) count8_fast<kMode - 2, true>(hist, q0, s0, fb, dum2);
            else count8_generic<kMode == 0>(hist, q0, s0, p.bp, dummy);
          }
          if (s1 != 0xFFu) {
            if (kMode >= 2) count8_fast<kMode - 2, true>(hist, q1, s1, fb, dum2);
            else count8_generic<kMode == 0>(hist, q1, s1, p.bp, dummy);
          }
        }
        for (; lr < ch; lr += rpi, ptr += step) {
          const uint32_t skip = cskip | (~bits8(bm + lr * p.wpr, p.wpr, lc0) & 0xFFu);
          if (skip == 0xFFu) continue;
          const uint4 q = ld_stream16(ptr);
          if (kMode >= 2) count8_fast<kMode - 2, true>(hist, q, skip, fb, dum2);
          else count8_generic<kMode == 0>(hist, q, skip, p.bp, dummy);
        }
      }
    } else {
      for (int lr = 0; lr < ch; ++lr) {
        for (int kk = threadIdx.x; kk < nk; kk += blockDim.x) {
          const int64_t cs = (k0 + kk) * 8;
          const uint32_t skip = cols_skip8(cs, c0, w) | (~bits8(bm + lr * p.wpr, p.wpr, (int)(cs - c0)) & 0xFFu);
          if (skip == 0xFFu) continue;
          const uint4 q = ld_stream16(base + (int64_t)lr * pitch + kk * 8);
          if (kMode >= 2) count8_fast<kMode - 2, true>(hist, q, skip, fb, dum2);
          else count8_generic<kMode == 0>(hist, q, skip, p.bp, dummy);
        }
      }
    }
    __syncthreads();
  }
  // ---- flush the pair's histogram
  const int nbins = p.bp.nbins;
  const int64_t orow = (int64_t)k * nbins;
  for (int b = threadIdx.x; b < nbins; b += blockDim.x) {
    const uint32_t v = hist[kOff + b];
    if (v) {
      if (kU64) atomicAdd(reinterpret_cast<unsigned long long*>(p.out) + orow + b, (unsigned long long)v);
      else atomicAdd(reinterpret_cast<uint32_t*>(p.out) + orow + b, v);
    }
  }
}

cudaError_t launch_pip(Ctx& c) { return launch_pip_list(c, c.d_isect.as<int2>(), c.n_isect, nullptr); }

cudaError_t launch_pip_list(Ctx& c, const int2* pairs, int64_t grid, const int64_t* n_dev) {
  if (grid == 0) return cudaSuccess;
  PipP p;
  p.n_dev = n_dev;
  p.rp = c.rp;
  p.g = c.geo;
  p.bp = c.bp;
  p.isect = pairs;
  p.mbb = c.d_mbb.as<int4>();
  p.band_base = c.d_band_base.as<int64_t>();
  p.band_off = c.d_band_off.as<int32_t>();
  p.band_edges = c.d_band_edges.as<int32_t>();
  p.edges = c.d_edges.as<Edge>();
  p.erows = c.d_erows.as<int2>();
  p.out = c.d_out;
  p.B_pad = c.B_pad;
  p.fb = make_fast_bins(c.bp);
  p.wpr = c.rp.T / 32 + 1;
  // up to 32 KB of parity bitmap per CTA, less when the histogram is large (227 KB per CTA)
  const int hist_bytes = hist_words(c.bp.nbins) * 4;
  int bm_budget_words = (227 * 1024 - 2048 - hist_bytes) / 4;
  if (bm_budget_words > 8192) bm_budget_words = 8192;
  p.rc = bm_budget_words / p.wpr;
  if (p.rc < 1) p.rc = 1;
  if (p.rc > c.rp.T) p.rc = c.rp.T;
  const size_t smem = (size_t)hist_words(c.bp.nbins) * 4 + (size_t)p.rc * p.wpr * 4;
  const int threads = 256;
  void (*k)(PipP);
  const int mode = fast_bins_ok(c.bp) ? (p.fb.bias ? 4 : (c.bp.use_nodata ? 3 : 2)) : (c.bp.width == 1 ? 0 : 1);
  switch (mode) {
    case 0: k = c.out_u64 ? k_pip<0, true> : k_pip<0, false>; break;
    case 1: k = c.out_u64 ? k_pip<1, true> : k_pip<1, false>; break;
    case 2: k = c.out_u64 ? k_pip<2, true> : k_pip<2, false>; break;
    case 3: k = c.out_u64 ? k_pip<3, true> : k_pip<3, false>; break;
    default: k = c.out_u64 ? k_pip<4, true> : k_pip<4, false>; break;
  }
  if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  k<<<(unsigned)grid, threads, smem, c.stream>>>(p);
  c.launches += 1;
  return cudaGetLastError();
}

}  // namespace zh
