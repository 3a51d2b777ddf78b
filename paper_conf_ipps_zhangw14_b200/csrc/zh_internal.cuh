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
// (ox, oy): the representative point inside the cell, in cell units — (0.5, 0.5) is the centre the
// paper chooses (§III.D); other points (corners, ...) are the alternatives it mentions
// (SURVEY.md §8f-3).  The names below say "centre" for the general representative point.
struct Geo {
  double gt0, gt1, gt3, gt5;
  double ox, oy;
  double igt1;  // 1 / gt1: only for first guesses of a column (every decision is exact, first_false)
  double igt5;  // 1 / gt5: likewise for rows
};

// kRep = false: the centre (0.5 as an immediate — the hot kernels are instantiated for it, the
// runtime offsets cost ~12 % in the round-1 one-kernel step 4); kRep = true: the runtime offsets g.ox, g.oy.  Both give
// identical values when the offsets are 0.5.
template <bool kRep = true>
__device__ __forceinline__ double col_centre(const Geo& g, int64_t c) {
  return __dadd_rn(g.gt0, __dmul_rn(__dadd_rn((double)c, kRep ? g.ox : 0.5), g.gt1));
}
template <bool kRep = true>
__device__ __forceinline__ double row_centre(const Geo& g, int64_t r) {
  return __dadd_rn(g.gt3, __dmul_rn(__dadd_rn((double)r, kRep ? g.oy : 0.5), g.gt5));
}

// Canonical edge (ya <= yb), Fig. 5 predicate in lower-endpoint-first orientation (R8).
struct __align__(32) Edge {
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

// 32-byte streaming load (sm_100: one LDG.256 for 16 cells).
__device__ __forceinline__ void ld_stream32(const void* p, uint4& lo, uint4& hi) {
  asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(lo.x), "=r"(lo.y), "=r"(lo.z), "=r"(lo.w), "=r"(hi.x), "=r"(hi.y), "=r"(hi.z), "=r"(hi.w)
               : "l"(p));
}

__device__ __forceinline__ int cell_of(const uint4& q, int j) {
  const uint32_t w = (j < 2) ? q.x : (j < 4) ? q.y : (j < 6) ? q.z : q.w;
  return (int)(int16_t)(w >> ((j & 1) * 16));
}

// ----------------------------------------------------------------------------------------------
// Shared-memory histogram layout used by steps 1 and 4 (HistLayout):
//   hist[kOff - 1]            "below range" trash (drop mode)
//   hist[kOff + b]            bin b, b in [0, nbins)          (16-byte aligned: kOff = 4)
//   hist[kOff + nbins]        "above range" trash (drop mode)
//   hist[dum + lane]          32 per-lane dummy slots for cells that are not counted (nodata,
//                             outside the tile / polygon): every cell issues exactly one shared
//                             atomic, with no predicate and no branch, and the not-counted
//                             ones never collide across lanes.
// ----------------------------------------------------------------------------------------------
constexpr int kOff = 4;

__host__ __device__ __forceinline__ int hist_dummy(int nbins) { return (kOff + nbins + 1 + 3) & ~3; }
__host__ __device__ __forceinline__ int hist_words(int nbins) { return hist_dummy(nbins) + 32; }

// Packed 16x2 bin mapping (width == 1, lo in int16, nbins <= 16000; see fast_bins_ok).
// Two formulations, both ending with idx in [kOff-1, kOff+nbins] for counted cells and a value
// >= the dummy base for cells that are not counted:
//  kBias (use_nodata and nodata < L, e.g. SRTM voids = -32768 below every bin):
//     a = min_s16(v, H); b = a - (nodata+1) (mod 2^16)   -> nodata becomes 0xFFFF, the rest keep order
//     c = max_u16(b, L - nodata - 1); idx = c - (C - nodata - 1)
//     (nodata stays far above the dummy base; 4 ALU ops per two cells, no compare)
//  plain (no nodata, or nodata inside the range):
//     c = clamp_s16(v, L, H); idx = c - C; nodata halves -> 0xFFFF by a zero-detect of v ^ nodata
// clamp mode: L = lo, H = lo+nbins-1 (capped at 32767)   drop mode: L = lo-1, H = lo+nbins (trash)
// C = lo - kOff.
struct FastBins {
  uint32_t L2, H2, C2, nod2;   // plain
  uint32_t Hb2, Nb2, Lb2, Cb2;  // biased
  uint32_t use_nodata, bias;
  uint32_t nC2, nNb2, nCb2;     // -C2, -Nb2, -Cb2 per half: the kernels add them (VIADD.16x2 of a
                                // kernel parameter, no per-use negation)
};

#ifndef ZH_NEG
#define ZH_NEG 1
#endif

__host__ __device__ inline bool fast_bins_ok(const BinP& b) {
  return b.width == 1 && b.lo >= -32768 && b.lo <= 32767 && b.nbins <= 16000;
}

__host__ __device__ inline FastBins make_fast_bins(const BinP& b) {
  FastBins f;
  const int top = b.lo + b.nbins - 1;  // last value with a bin of its own
  int L = b.lo, H = top < 32767 ? top : 32767;
  if (b.drop) {
    if (b.lo > -32768) L = b.lo - 1;  // below-range trash; nothing is below -32768
    if (top < 32767) H = top + 1;     // above-range trash; nothing is above 32767
  }
  const int C = b.lo - kOff;
  auto pk = [](int v) { return (uint32_t)(uint16_t)v * 0x10001u; };
  f.L2 = pk(L);
  f.H2 = pk(H);
  f.C2 = pk(C);
  f.nod2 = pk(b.nodata);
  f.use_nodata = b.use_nodata ? 1u : 0u;
  // biased form: valid when nodata < L, the nodata index stays above the dummy slots, and no value
  // lies below nodata that would have to be counted: v - (nodata+1) wraps for v < nodata, which
  // sends those cells to the dummy slots.  That is right in drop mode (v < nodata < lo is dropped)
  // and vacuous for nodata = -32768; in clamp mode with a higher nodata they belong in bin 0.
  const int N1 = b.nodata + 1;
  f.Hb2 = pk(H);
  f.Nb2 = pk(N1);
  f.Lb2 = pk(L - N1);
  f.Cb2 = pk(C - N1);
  f.nC2 = pk(-C);
  f.nNb2 = pk(-N1);
  f.nCb2 = pk(N1 - C);
  const int nod_idx = 0xFFFF - ((C - N1) & 0xFFFF);  // where a nodata cell lands
  f.bias = (b.use_nodata && b.nodata < L && (b.drop || b.nodata == -32768) && nod_idx >= hist_dummy(b.nbins) + 32)
               ? 1u : 0u;
  return f;
}

// kNeg: add the pre-negated constants (k_mixed_cells: fewer operations per vector; the pure-tile
// kernel is slower with them, 3.16 -> 3.43 ms at CONUS — its register allocation changes)
template <int kForm, bool kNeg = false>  // 0 plain, 1 plain + nodata zero-detect, 2 biased (nodata below range)
__device__ __forceinline__ uint32_t fast_idx2(uint32_t w, const FastBins& f) {
  if (kForm == 2) {
    uint32_t a = __vmins2(w, f.Hb2);
    a = kNeg ? __vadd2(a, f.nNb2) : __vsub2(a, f.Nb2);
    a = __vmaxu2(a, f.Lb2);
    return kNeg ? __vadd2(a, f.nCb2) : __vsub2(a, f.Cb2);
  }
  uint32_t c = __vmaxs2(w, f.L2);
  c = __vmins2(c, f.H2);
  c = kNeg ? __vadd2(c, f.nC2) : __vsub2(c, f.C2);
  if (kForm == 1) {
    const uint32_t x = w ^ f.nod2;                 // zero halves where v == nodata
    const uint32_t z = __vsub2(x, 0x00010001u) & ~x & 0x80008000u;
    c |= __byte_perm(z, 0, 0xBB99);                // 0xFFFF in those halves
  }
  return c;
}

// Byte j of the result pair (lo: cells 0-3, hi: cells 4-7) is 0xFF when bit j of m is set.
__device__ __forceinline__ void spread_bits8(uint32_t m, uint32_t& lo, uint32_t& hi) {
  lo = (((m & 0xFu) * 0x00204081u) & 0x01010101u) * 0xFFu;
  hi = ((((m >> 4) & 0xFu) * 0x00204081u) & 0x01010101u) * 0xFFu;
}

// Count 8 cells (one 16-byte vector) into the shared histogram.  `skip` has bit j set for cells
// that must not be counted (outside the tile / not inside the polygon).  `dum2` = (dummy slot
// of this lane) in both halves.  Indices are < 2^14, so idx*4 of both halves is one 32-bit
// shift of the packed pair.
template <int kForm, bool kMask>
__device__ __forceinline__ void count8_fast(uint32_t* __restrict__ hist, const uint4& q, uint32_t skip,
                                            const FastBins& f, uint32_t dum2) {
  uint32_t sl = 0, sh = 0;
  if (kMask) spread_bits8(skip, sl, sh);
  const uint32_t ws[4] = {q.x, q.y, q.z, q.w};
  char* hb = reinterpret_cast<char*>(hist);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    uint32_t x = fast_idx2<kForm>(ws[i], f);
    if (kMask) x |= __byte_perm(sl, sh, (uint32_t)((2 * i) | (2 * i) << 4 | (2 * i + 1) << 8 | (2 * i + 1) << 12));
    x = __vminu2(x, dum2) << 2;  // byte offsets of both cells
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x & 0xFFFFu)), 1u);
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x >> 16)), 1u);
  }
}

// Two histograms side by side (words [0, hw) and [hw, 2 hw)): as count8_fast, and cell j goes to
// the second one when bit j of `sel` is set.  `off2` = hw in both halves; the slot offset is added
// after the dummy clamp, so a selected cell that is not counted lands on the second histogram's
// dummy slot (never flushed).  Byte offsets stay 16-bit: the caller guarantees 2 hw * 4 < 2^16.
template <int kForm>
__device__ __forceinline__ void count8_fast_sel(uint32_t* __restrict__ hist, const uint4& q, uint32_t skip,
                                                uint32_t sel, const FastBins& f, uint32_t dum2, uint32_t off2) {
  uint32_t sl, sh, el, eh;
  spread_bits8(skip, sl, sh);
  spread_bits8(sel, el, eh);
  const uint32_t ws[4] = {q.x, q.y, q.z, q.w};
  char* hb = reinterpret_cast<char*>(hist);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint32_t P = (uint32_t)((2 * i) | (2 * i) << 4 | (2 * i + 1) << 8 | (2 * i + 1) << 12);
    uint32_t x = fast_idx2<kForm>(ws[i], f) | __byte_perm(sl, sh, P);
    x = __vminu2(x, dum2);
    x = (x + (__byte_perm(el, eh, P) & off2)) << 2;  // halves < 2 hw: no carry between them
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x & 0xFFFFu)), 1u);
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x >> 16)), 1u);
  }
}

// Two histograms, A at word 0 and B at word `offb`, a power of two (>= 256) above every index of A:
// a cell goes to B by OR-ing offb into its index.  One code byte per cell — 0 (A), offb >> 8 (B),
// 0xFF (not counted) — lands in the high byte of the cell's 16-bit half (one PRMT per two cells);
// the clamp to dumB2 = (offb + this lane's dummy slot) in both halves then sends not-counted cells
// to B's dummy slots (never flushed).  The caller guarantees (offb + hist_words) * 4 < 2^16 and a
// biased nodata index >= offb + hist_words.
template <int kForm>
__device__ __forceinline__ void count8_fast_code(uint32_t* __restrict__ hist, const uint4& q, uint32_t skip,
                                                 uint32_t sel, const FastBins& f, uint32_t dumB2, uint32_t ob) {
  const uint32_t e = sel & ~skip;
  const uint32_t clo = (((skip & 0xFu) * 0x00204081u) & 0x01010101u) * 0xFFu +
                       (((e & 0xFu) * 0x00204081u) & 0x01010101u) * ob;
  const uint32_t chi = ((((skip >> 4) & 0xFu) * 0x00204081u) & 0x01010101u) * 0xFFu +
                       ((((e >> 4) & 0xFu) * 0x00204081u) & 0x01010101u) * ob;
  const uint32_t ws[4] = {q.x, q.y, q.z, q.w};
  char* hb = reinterpret_cast<char*>(hist);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint32_t j = (uint32_t)(i & 1) * 2;  // first of the two cells within its 4-cell code word
    const uint32_t P = 4u | (j << 4) | (4u << 8) | ((j + 1) << 12);
    uint32_t x = fast_idx2<kForm>(ws[i], f) | __byte_perm(i < 2 ? clo : chi, 0u, P);
    x = __vminu2(x, dumB2) << 2;
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x & 0xFFFFu)), 1u);
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x >> 16)), 1u);
  }
}

// count8_fast_code with fewer operations per vector: a not-counted cell's code byte is 0x80
// (its 16-bit index >= 0x8000 > every slot, so the dummy clamp still catches it) and both code
// bytes come straight out of one multiply each — bit j of a nibble times 0x00204081 * k, masked
// with 0x01010101 * k, is byte j = k (k a power of two): 0x80 for skip, ob = offb >> 8 for B.
// mb = 0x00204081 * ob, kb = 0x01010101 * ob (the caller hoists them).
template <int kForm>
__device__ __forceinline__ void count8_fast_code2(uint32_t* __restrict__ hist, const uint4& q, uint32_t skip,
                                                  uint32_t sel, const FastBins& f, uint32_t dumB2, uint32_t mb,
                                                  uint32_t kb) {
  const uint32_t e = sel & ~skip;
  const uint32_t clo = (((skip & 0xFu) * 0x10204080u) & 0x80808080u) | (((e & 0xFu) * mb) & kb);
  const uint32_t chi = (((skip >> 4) * 0x10204080u) & 0x80808080u) | (((e >> 4) * mb) & kb);
  const uint32_t ws[4] = {q.x, q.y, q.z, q.w};
  char* hb = reinterpret_cast<char*>(hist);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint32_t j = (uint32_t)(i & 1) * 2;
    const uint32_t P = 4u | (j << 4) | (4u << 8) | ((j + 1) << 12);
    uint32_t x = fast_idx2<kForm, ZH_NEG>(ws[i], f) | __byte_perm(i < 2 ? clo : chi, 0u, P);
    x = __vminu2(x, dumB2) << 2;
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x & 0xFFFFu)), 1u);
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x >> 16)), 1u);
  }
}

// Flat layout of k_mixed_cells (B right after A, at a multiple of 256 words, so that a group's
// whole-tile bitmaps fit beside both histograms): the code byte is ADDED to the cell's 16-bit
// index — 0 (A), kB = offb >> 8 (B), 0x40 (not counted: index >= 0x4000, above every slot, the
// dummy clamp catches it).  kForm 0 or 2 only; the caller guarantees offb + hist_words < 0x4000
// and that a biased nodata index plus 0x40 << 8 stays below 2^16 (no half wraps, so the add of
// both halves is one 32-bit add).
template <int kForm>
__device__ __forceinline__ void count8_fast_code3(uint32_t* __restrict__ hist, const uint4& q, uint32_t skip,
                                                  uint32_t sel, const FastBins& f, uint32_t dumB2, uint32_t kB) {
  const uint32_t e = sel & ~skip;
  const uint32_t clo = (((skip & 0xFu) * 0x08102040u) & 0x40404040u) | ((((e & 0xFu) * 0x00204081u) & 0x01010101u) * kB);
  const uint32_t chi = (((skip >> 4) * 0x08102040u) & 0x40404040u) | ((((e >> 4) * 0x00204081u) & 0x01010101u) * kB);
  const uint32_t ws[4] = {q.x, q.y, q.z, q.w};
  char* hb = reinterpret_cast<char*>(hist);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint32_t j = (uint32_t)(i & 1) * 2;
    const uint32_t P = 4u | (j << 4) | (4u << 8) | ((j + 1) << 12);
    // per-half add of the code, then the dummy clamp: one VIADDMNMX
    uint32_t x = __vminu2(__vadd2(fast_idx2<kForm, ZH_NEG>(ws[i], f), __byte_perm(i < 2 ? clo : chi, 0u, P)), dumB2) << 2;
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x & 0xFFFFu)), 1u);
    atomicAdd(reinterpret_cast<uint32_t*>(hb + (x >> 16)), 1u);
  }
}

// Generic path (any width / lo / nbins): same layout, scalar mapping, per-cell atomics.
template <bool kW1>
__device__ __forceinline__ void count8_generic(uint32_t* __restrict__ hist, const uint4& q, uint32_t skip,
                                               const BinP& bp, uint32_t dummy) {
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    int b = ((skip >> j) & 1u) ? -1 : bin_of<kW1>(cell_of(q, j), bp);
    atomicAdd(&hist[b >= 0 ? kOff + b : (int)dummy], 1u);
  }
}

// Generic path of count8_fast_sel: cell j goes to hist + hw when bit j of `sel` is set.
template <bool kW1>
__device__ __forceinline__ void count8_generic_sel(uint32_t* __restrict__ hist, const uint4& q, uint32_t skip,
                                                   uint32_t sel, const BinP& bp, uint32_t dummy, int hw) {
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    int b = ((skip >> j) & 1u) ? -1 : bin_of<kW1>(cell_of(q, j), bp);
    atomicAdd(&hist[(b >= 0 ? kOff + b : (int)dummy) + (((sel >> j) & 1u) ? hw : 0)], 1u);
  }
}

// Validity of the 8 cells starting at column cs within the tile columns [c0, c0 + w): bit j set
// when column cs + j is OUTSIDE (to be skipped).
__device__ __forceinline__ uint32_t cols_skip8(int64_t cs, int64_t c0, int w) {
  uint32_t valid = 0xFFu;
  if (cs < c0) valid &= (0xFFu << (int)(c0 - cs)) & 0xFFu;
  if (cs + 8 > c0 + w) valid &= 0xFFu >> (int)(cs + 8 - (c0 + w));
  return ~valid & 0xFFu;
}

// ----------------------------------------------------------------------------------------------
// Kernel parameter blocks
// ----------------------------------------------------------------------------------------------
struct RasterP {
  const int16_t* data;  // points at row `row0` of the full raster (device)
  int64_t rows, cols, pitch, row0, nrows;
  int32_t T, TC, tr0, TRn;  // tile size, tile columns, first tile row, tile rows in shard
  uint32_t tc_mul, tc_sh;   // tile / TC by multiply-high (set_tc_div; Granlund-Montgomery round-up)
  int32_t wide;             // 32-byte loads apply: data and pitch keep every 16-cell segment 32-byte aligned
  uint32_t t_mul, t_sh;     // cell / T likewise
};

// (mul, sh) for an exact n / d, 0 <= n < 2^31, with one multiply-high instead of a division loop
// (Granlund-Montgomery round-up): t = umulhi(mul, n), q = (t + ((n - t) >> 1)) >> (sh - 1); sh = 0: d = 1.
__host__ inline void magic_div(uint32_t d, uint32_t& mul, uint32_t& sh) {
  uint32_t l = 0;
  while ((1ull << l) < d) ++l;  // ceil(log2 d)
  sh = l;
  mul = l == 0 ? 0u : (uint32_t)(((1ull << 32) * ((1ull << l) - d)) / d + 1);
}
__host__ inline void set_tc_div(RasterP& rp) {
  magic_div((uint32_t)rp.TC, rp.tc_mul, rp.tc_sh);
  magic_div((uint32_t)rp.T, rp.t_mul, rp.t_sh);
}
__device__ __forceinline__ int magic_q(uint32_t n, uint32_t mul, uint32_t sh) {
  if (sh == 0) return (int)n;
  const uint32_t t = __umulhi(mul, n);
  return (int)((t + ((n - t) >> 1)) >> (sh - 1));
}

// (tile row, tile column) of a shard-local tile index
__device__ __forceinline__ int tile_row(const RasterP& rp, int tile) { return magic_q((uint32_t)tile, rp.tc_mul, rp.tc_sh); }
// tile row / column of a (non-negative) cell row / column
__device__ __forceinline__ int cell_tile(const RasterP& rp, int64_t cell) { return magic_q((uint32_t)cell, rp.t_mul, rp.t_sh); }

}  // namespace zh
