// k_pip.cu — step 4: cell-in-polygon test and histogram update for intersecting pairs
// (§III.D, Fig. 5, pip_test_kernel).
//
// For each intersecting (tile, polygon k) pair and each cell of the tile whose centre passes the
// even-odd ray-crossing test against all rings of k, out[k][bin(v)] += 1.
//
// Paper design (prior art): one block per polygon, one thread per cell, and for every cell a loop
// over ALL polygon vertices in global memory with float coordinates; the histogram update is a
// non-atomic read-modify-write (a race).  B200 design, bit-identical to the per-cell test, in two
// kernels (k_parity, then k_pip_cells for the four-step path or k_mixed_cells for the fused one):
//   * one CTA per intersecting pair; only the edges of the pair's band (edges that straddle one
//     of the tile's centre rows, built in step 2) are visited;
//   * the crossing test `xc < xi` depends on the cell only through xc, and xc is monotone in the
//     column, so for each (edge, row) the crossed cells form a prefix (gt1 > 0) or suffix
//     (gt1 < 0) of the row: the exact boundary column is found with the SAME xc(c) expression
//     (first_false), and recorded as a flip in a per-row difference bitmap in shared memory;
//     a suffix-XOR turns it into the per-cell parity (inside) bits, stored as the pair's bitmap
//     (k_parity).  Work per pair is O(#(edge,row) crossings + cells) instead of O(cells x edges);
//   * edges entirely left / right of the tile's centres (with half a cell of margin, far above
//     the intercept's rounding) skip the division;
//   * the cells are then streamed exactly like step 1 (16-byte vectors, packed 16x2 bin mapping,
//     one branch-free shared atomic per cell; vectors with no inside cell are not even loaded)
//     into a CTA-private shared histogram, flushed once per pair with one global atomic per
//     non-zero bin (no race).
#include <algorithm>

#include "zh_ctx.h"
#include "zh_pip.cuh"

namespace zh {

#ifndef ZH_PIP_MINB
#define ZH_PIP_MINB 6
#endif
#ifndef ZH_PIP_THREADS
#define ZH_PIP_THREADS 256
#endif
constexpr int kPipThreads = ZH_PIP_THREADS;  // k_pip_cells

// Split form (zh_pip.cuh): parity bitmaps of every pair, then the cells.
#ifndef ZH_PAR_THREADS
#define ZH_PAR_THREADS 128
#endif
#ifndef ZH_PAR_MINB
#define ZH_PAR_MINB 14
#endif
template <bool kRep>
__global__ void __launch_bounds__(ZH_PAR_THREADS, ZH_PAR_MINB) k_parity(PipP p) {
  if (p.n_dev && (int64_t)blockIdx.x >= *p.n_dev) return;
  extern __shared__ __align__(16) uint32_t sh[];
  __shared__ LongQ lq;
  parity_pair_body<kRep>(p, blockIdx.x, sh, &lq);
}

template <int kMode, bool kU64>
__global__ void __launch_bounds__(kPipThreads, ZH_PIP_MINB) k_pip_cells(PipP p) {
  if (p.n_dev && (int64_t)blockIdx.x >= *p.n_dev) return;
  extern __shared__ __align__(16) uint32_t sh[];
  pip_cells_body<kMode, kU64>(p, blockIdx.x, sh);
}

#ifndef ZH_MIX_THREADS
#define ZH_MIX_THREADS 256
#endif
#ifndef ZH_MIX_CODE
#define ZH_MIX_CODE 1  // k_mixed_cells: code-byte routing with B at a power-of-two offset (packed bins)
#endif
#ifndef ZH_MIX_FLAT
#define ZH_MIX_FLAT 1  // k_mixed_cells: flat layout (whole-tile bitmaps, added code bytes) when it fits
#endif
#ifndef ZH_MIX_MINB
#define ZH_MIX_MINB 4
#endif
// Tile groups of <= 2 pairs (fused path): each cell read once per group (zh_pip.cuh).
template <int kMode, bool kU64, int kCode>
__global__ void __launch_bounds__(ZH_MIX_THREADS, ZH_MIX_MINB) k_mixed_cells(PipP p) {
  if (p.n_dev && (int64_t)blockIdx.x >= *p.n_dev) return;
  extern __shared__ __align__(16) uint32_t sh[];
  mixed_cells_body<kMode, kU64, kCode>(p, blockIdx.x, sh);
}

cudaError_t launch_pip(Ctx& c) { return launch_pip_list(c, c.d_isect.as<int2>(), c.n_isect, nullptr); }


PipP pip_params(Ctx& c, const int2* pairs, const int64_t* n_dev) {
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
  p.wpo = (c.rp.T + 31) / 32;
  p.rcc = 8192 / p.wpo;
  if (p.rcc < 1) p.rcc = 1;
  if (p.rcc > c.rp.T) p.rcc = c.rp.T;
  p.pbits = c.d_pbits.as<uint32_t>();
  p.grp = nullptr;
  p.offb = 0;
  p.bmo = 0;
  return p;
}

static int pip_mode(const Ctx& c) {
  const FastBins fb = make_fast_bins(c.bp);
  return fast_bins_ok(c.bp) ? (fb.bias ? 4 : (c.bp.use_nodata ? 3 : 2)) : (c.bp.width == 1 ? 0 : 1);
}

cudaError_t pip_prepare(Ctx& c, int64_t grid) {
  const size_t need = (size_t)grid * (size_t)c.rp.T * (size_t)((c.rp.T + 31) / 32) * 4;
  return c.d_pbits.ensure(need);
}

cudaError_t launch_parity(Ctx& c, const int2* pairs, int64_t grid, const int64_t* n_dev, cudaStream_t s) {
  if (grid == 0) return cudaSuccess;
  PipP p = pip_params(c, pairs, n_dev);
  const size_t smem = ((size_t)p.rc * p.wpr + 3) / 4 * 16;
  const bool rep = !(c.geo.ox == 0.5 && c.geo.oy == 0.5);
  void (*k)(PipP) = rep ? k_parity<true> : k_parity<false>;
  prep_kernel(k, smem);
  k<<<(unsigned)grid, ZH_PAR_THREADS, smem, s>>>(p);
  c.launches += 1;
  return cudaGetLastError();
}

cudaError_t launch_pip_cells(Ctx& c, const int2* pairs, int64_t grid, const int64_t* n_dev) {
  if (grid == 0) return cudaSuccess;
  PipP p = pip_params(c, pairs, n_dev);
  const size_t smem = (size_t)hist_words(c.bp.nbins) * 4 + (size_t)p.rcc * p.wpo * 4;
  void (*k)(PipP);
  switch (pip_mode(c)) {
    case 0: k = c.out_u64 ? k_pip_cells<0, true> : k_pip_cells<0, false>; break;
    case 1: k = c.out_u64 ? k_pip_cells<1, true> : k_pip_cells<1, false>; break;
    case 2: k = c.out_u64 ? k_pip_cells<2, true> : k_pip_cells<2, false>; break;
    case 3: k = c.out_u64 ? k_pip_cells<3, true> : k_pip_cells<3, false>; break;
    default: k = c.out_u64 ? k_pip_cells<4, true> : k_pip_cells<4, false>; break;
  }
  prep_kernel(k, smem);
  k<<<(unsigned)grid, kPipThreads, smem, c.stream>>>(p);
  c.launches += 1;
  return cudaGetLastError();
}

// Rows per staged bitmap chunk of k_mixed_cells: 4 KB per pair (4 CTAs of 48 KB per SM at 5,000 bins).
static int mixed_rows(const Ctx& c) {
  const int wpo = (c.rp.T + 31) / 32;
  return std::max(1, std::min(c.rp.T, 1024 / wpo));
}

// Shared-memory layout of k_mixed_cells: histogram A at word 0, B at word *offb, the two staged
// bitmaps (*rows rows of each pair) at word *bmo; *code = the routing form (mixed_cells_body's kCode).
//  2 (flat, preferred): B right after A at a multiple of 256 words, the whole tile's bitmaps
//    after B (one staging round per group instead of one per 128 rows), code bytes added; only
//    while the CTA stays within 56 KB (4 CTAs per SM) and the 16-bit indices cannot wrap;
//  1: B at a power of two (OR-ed code bytes), 128-row bitmap chunks in the gap below it;
//  0: B right after A, offsets added per cell.
// Returns the bytes, or 0 when the grouped form does not apply (two histograms must fit the CTA,
// and the packed forms need 16-bit byte offsets over both).
static size_t mixed_layout(const Ctx& c, int* offb, int* bmo, int* code, int* rows) {
  const int hw = hist_words(c.bp.nbins);
  const int wpo = (c.rp.T + 31) / 32;
  const bool packed = pip_mode(c) >= 2;
  const FastBins fb = make_fast_bins(c.bp);
  const int nod_idx = 0xFFFF - (int)(fb.Cb2 & 0xFFFFu);
  {
    const int ob = (hw + 255) & ~255;
    const int bo = (ob + hw + 3) & ~3;
    const size_t words = (size_t)bo + 2 * (size_t)c.rp.T * wpo;
    if (ZH_MIX_FLAT && packed && pip_mode(c) != 3 && (ob >> 8) < 0x40 && ob + hw < 0x4000 &&
        (!fb.bias || (nod_idx >= ob + hw && nod_idx + 0x4000 <= 0xFFFF)) && words * 4 <= 56 * 1024) {
      *code = 2;
      *offb = ob;
      *bmo = bo;
      *rows = c.rp.T;
      return words * 4;
    }
  }
  *rows = mixed_rows(c);
  const int bmw = 2 * *rows * wpo;
  int ob = 256;
  while (ob < hw) ob *= 2;
  const bool c1 = ZH_MIX_CODE && packed && (ob + hw) * 4 < 65536 && (!fb.bias || nod_idx >= ob + hw);
  *code = c1 ? 1 : 0;
  if (c1) {
    *offb = ob;
    *bmo = (hw + bmw <= ob) ? hw : ob + hw;
  } else {
    *offb = hw;
    *bmo = 2 * hw;
  }
  const size_t words = std::max<size_t>((size_t)*offb + hw, (size_t)*bmo + bmw);
  if (words * 4 > 200 * 1024) return 0;
  if (packed && !c1 && 2 * (size_t)hw * 4 >= 65536) return 0;
  return words * 4;
}

size_t mixed_smem(Ctx& c) {
  int ob, bo, code, rows;
  return mixed_layout(c, &ob, &bo, &code, &rows);
}

cudaError_t launch_mixed_cells(Ctx& c, const int2* pairs, const int2* grp, int64_t grid, const int64_t* n_dev) {
  if (grid == 0) return cudaSuccess;
  PipP p = pip_params(c, pairs, n_dev);
  p.grp = grp;
  int code = 0;
  const size_t smem = mixed_layout(c, &p.offb, &p.bmo, &code, &p.rcc);
  void (*k)(PipP);
#define ZH_MIX_K1(M, U) (code == 2 ? k_mixed_cells<M, U, 2> : code == 1 ? k_mixed_cells<M, U, 1> : k_mixed_cells<M, U, 0>)
#define ZH_MIX_K(M) (c.out_u64 ? ZH_MIX_K1(M, true) : ZH_MIX_K1(M, false))
  switch (pip_mode(c)) {
    case 0: k = ZH_MIX_K(0); break;
    case 1: k = ZH_MIX_K(1); break;
    case 2: k = ZH_MIX_K(2); break;
    case 3: k = ZH_MIX_K(3); break;
    default: k = ZH_MIX_K(4); break;
  }
#undef ZH_MIX_K
#undef ZH_MIX_K1
  prep_kernel(k, smem);
  k<<<(unsigned)grid, ZH_MIX_THREADS, smem, c.stream>>>(p);
  c.launches += 1;
  return cudaGetLastError();
}

// Four-step step 4 over step 2's intersecting pairs (bitmap slot = isect index).
cudaError_t launch_pip_list(Ctx& c, const int2* pairs, int64_t grid, const int64_t* n_dev) {
  if (grid == 0) return cudaSuccess;
  cudaError_t e = pip_prepare(c, grid);
  if (e != cudaSuccess) return e;
  if ((e = launch_parity(c, pairs, grid, n_dev, c.stream)) != cudaSuccess) return e;
  if (c.cover && pairs == c.d_isect.as<int2>() && (e = launch_touch(c, nullptr, c.stream)) != cudaSuccess) return e;
  return launch_pip_cells(c, pairs, grid, n_dev);
}

}  // namespace zh
