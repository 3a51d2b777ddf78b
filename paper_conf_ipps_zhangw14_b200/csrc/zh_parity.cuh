// zh_parity.cuh — the per-(tile, polygon) inside mask of step 4 (k_parity, one pair per CTA).
//
// For a chunk of the tile's rows [rlo, rhi) and columns [c0, c0 + w), the ray-crossing parity of
// every cell centre (Fig. 5, canonical orientation R8, half-open rule R10) is built as
//   1. crossings: every band edge straddling a row r (exact row interval from step 2) has the
//      intercept xi = intercept(e, yc(r)) (the same left-to-right double expression as the oracle);
//      the cells it crosses, {c : xc(c) < xi}, are a prefix (gt1 > 0) or suffix (gt1 < 0) of the
//      row, whose boundary column is found exactly with the SAME xc(c) expression (first_false);
//      the prefix [0, j) is recorded as a flip of bit j of a per-row difference bitmap D
//      (bit w = "all cells"), a suffix as flips of bits j and w;
//   2. suffix XOR: parity(lc) = XOR_{j > lc} D[j], computed word by word from the high end.
// Edges entirely left / right of the tile's centres (half a cell of margin, far above the
// intercept's rounding, zh_create enforces it) skip the division.
#pragma once
#include "zh_internal.cuh"

namespace zh {

struct TileGeom {
  int64_t r0, c0;  // first global row / column of the tile
  int h, w;        // rows / columns of the tile (edge tiles are partial)
  double xlo_t, xhi_t, half;
  bool s;          // gt1 > 0: xc increases with the column
};

template <bool kRep = true>
__device__ __forceinline__ TileGeom tile_geom(const RasterP& rp, const Geo& g, int tile) {
  TileGeom t;
  const int trl = tile_row(rp, tile), tc = tile - trl * rp.TC;
  t.r0 = (int64_t)(rp.tr0 + trl) * rp.T;
  t.h = (int)min((int64_t)rp.T, rp.row0 + rp.nrows - t.r0);
  t.c0 = (int64_t)tc * rp.T;
  t.w = (int)min((int64_t)rp.T, rp.cols - t.c0);
  const double xa = col_centre<kRep>(g, t.c0), xb = col_centre<kRep>(g, t.c0 + t.w - 1);
  t.xlo_t = fmin(xa, xb);
  t.xhi_t = fmax(xa, xb);
  t.half = 0.5 * fabs(g.gt1);
  t.s = g.gt1 > 0;
  return t;
}

// One (edge, row) crossing: flip the bits of D that record {c : xc(c) < xi}.
template <bool kRep>
__device__ __forceinline__ void crossing_row(uint32_t* __restrict__ bm, int wpr, const Edge& e, int64_t r,
                                             int64_t rlo, const Geo& g, const TileGeom& t) {
  const int w = t.w;
  const double yc = row_centre<kRep>(g, r);
  const double xi = intercept(e, yc);
  const double est = (xi - g.gt0) * g.igt1 - g.ox - (double)t.c0;
  int64_t ei;
  if (!(est > 0.0)) ei = 0;
  else if (est > (double)w) ei = w;
  else ei = (int64_t)ceil(est);
  const int64_t jb =
      first_false(0, w, ei, [&](int64_t j) { return (col_centre<kRep>(g, t.c0 + j) < xi) == t.s; });
  const int lr = (int)(r - rlo);
  if (jb > 0) atomicXor(&bm[lr * wpr + (int)(jb >> 5)], 1u << (jb & 31));
  if (!t.s) atomicXor(&bm[lr * wpr + (w >> 5)], 1u << (w & 31));
}

// Shared-memory queue of long edges (more than kLongRows straddled rows in the chunk): they are
// processed afterwards by whole warps, one row per lane, so that no thread serialises hundreds of
// rows while the others wait at the barrier.
#ifndef ZH_PAR_ST32
#define ZH_PAR_ST32 1  // k_parity: 32-byte streaming stores of the parity rows
#endif
#ifndef ZH_PAR_DYN
#define ZH_PAR_DYN 1  // k_parity: band edges claimed dynamically (atomic counter) after the first
#endif
#ifndef ZH_PAR_SPEC
#define ZH_PAR_SPEC 1
#endif
#ifndef ZH_LONG_ROWS
#define ZH_LONG_ROWS 8
#endif
constexpr int kLongRows = ZH_LONG_ROWS;
constexpr int kLongQ = 128;
struct LongQ {
  int n;
  int next;  // ZH_PAR_DYN: band edges claimed beyond the first blockDim.x
  int4 e[kLongQ];  // (edge, ra, rb, kind: 0 compute, 1 crosses every cell)
};

// Step 1 of the header comment for band edges [e0, e1) into bm (rows [rlo, rhi), wpr words per
// row, zeroed by the caller).  Block-strided over the band's edges; `q` must hold q->n = 0, made
// visible by a barrier, before the first call; the function leaves it so and ends with a barrier.
template <bool kRep>
__device__ __forceinline__ void crossings_to_bitmap(uint32_t* __restrict__ bm, int wpr, int e0, int e1,
                                                    const int32_t* __restrict__ band_edges,
                                                    const Edge* __restrict__ edges, const int2* __restrict__ erows,
                                                    const Geo& g, const TileGeom& t, int64_t rlo, int64_t rhi,
                                                    LongQ* q) {
  const int w = t.w;
#if ZH_PAR_DYN
  // the first edge of each thread by index, the rest claimed one at a time (threads whose edges
  // straddle few rows or miss the tile take more of them: no tail at the barrier below)
  for (int i = e0 + threadIdx.x; i < e1; i = e0 + (int)blockDim.x + atomicAdd(&q->next, 1)) {
#else
  for (int i = e0 + threadIdx.x; i < e1; i += blockDim.x) {
#endif
    const int v = band_edges[i];
#if ZH_PAR_SPEC  // the edge's rows and coordinates loaded together: two dependent loads, not three
    const int2 rr = erows[v];
    const Edge e = edges[v];
    const int64_t ra = max((int64_t)rr.x, rlo), rb = min((int64_t)rr.y, rhi);
    if (ra >= rb) continue;
#else
    const int2 rr = erows[v];
    const int64_t ra = max((int64_t)rr.x, rlo), rb = min((int64_t)rr.y, rhi);
    if (ra >= rb) continue;
    const Edge e = edges[v];
#endif
    const double exl = fmin(e.xa, e.xb), exh = fmax(e.xa, e.xb);
    if (exh + t.half < t.xlo_t) continue;  // xi < every xc: crosses no cell of the tile
    const int all = exl - t.half > t.xhi_t;  // xi > every xc: crosses every cell
    if (rb - ra > kLongRows) {
      const int pos = atomicAdd(&q->n, 1);
      if (pos < kLongQ) {
        q->e[pos] = make_int4(v, (int)ra, (int)rb, all);
        continue;
      }
    }
    if (all) {
      for (int64_t r = ra; r < rb; ++r) atomicXor(&bm[(int)(r - rlo) * wpr + (w >> 5)], 1u << (w & 31));
    } else {
      for (int64_t r = ra; r < rb; ++r) crossing_row<kRep>(bm, wpr, e, r, rlo, g, t);
    }
  }
  __syncthreads();
  const int nq = min(q->n, kLongQ);
  __syncthreads();                 // every thread has read the count ...
  if (threadIdx.x == 0) {  // ... so it can be reset for the next call
    q->n = 0;
    q->next = 0;
  }
  const int lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  for (int qi = threadIdx.x >> 5; qi < nq; qi += nw) {
    const int4 it = q->e[qi];
    if (it.w) {
      for (int r = it.y + lane; r < it.z; r += 32) atomicXor(&bm[(int)(r - rlo) * wpr + (w >> 5)], 1u << (w & 31));
    } else {
      const Edge e = edges[it.x];
      for (int r = it.y + lane; r < it.z; r += 32) crossing_row<kRep>(bm, wpr, e, r, rlo, g, t);
    }
  }
  __syncthreads();
}

// Step 2 for the split form: rows [0, ch) of bm become parity bits written straight to `out`
// (row stride wpo = ceil(w / 32) words, the word wpr - 1 = wpo only carries the "all cells" flips).
// Thread per row; with wpo % 4 == 0 the row is produced 4 words at a time and stored as 16 bytes.
__device__ __forceinline__ void suffix_xor_store(const uint32_t* __restrict__ bm, int wpr, int ch,
                                                 uint32_t* __restrict__ out, int wpo) {
  for (int lr = threadIdx.x; lr < ch; lr += blockDim.x) {
    const uint32_t* row = bm + lr * wpr;
    uint32_t* orow = out + (int64_t)lr * wpo;
    uint32_t carry = 0;
    // A row has one or two crossings, and neighbouring rows (the lanes of a warp) have theirs in the
    // same word: words with no flip in any lane of the warp take the 1-op path (uniform branch).
    const uint32_t lanes = __activemask();
    auto step = [&](uint32_t t) -> uint32_t {
      if (!__any_sync(lanes, t != 0u)) return 0u - carry;
      t ^= t >> 1; t ^= t >> 2; t ^= t >> 4; t ^= t >> 8; t ^= t >> 16;
      const uint32_t v = (t >> 1) ^ (0u - carry);
      carry ^= (t & 1u);
      return v;
    };
    for (int wi = wpr - 1; wi >= wpo; --wi) carry ^= __popc(row[wi]) & 1u;  // "all cells" flips: parity only
#if ZH_PAR_ST32
    if ((wpo & 7) == 0) {  // 8 words per 32-byte streaming store (sm_100)
      for (int g = wpo - 8; g >= 0; g -= 8) {
        uint32_t v[8];
#pragma unroll
        for (int k = 7; k >= 0; --k) v[k] = step(row[g + k]);
        asm volatile("st.global.cs.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(orow + g), "r"(v[0]), "r"(v[1]),
                     "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
                     : "memory");
      }
    } else
#endif
    if ((wpo & 3) == 0) {
      for (int g = wpo - 4; g >= 0; g -= 4) {
        uint4 v;
        v.w = step(row[g + 3]);
        v.z = step(row[g + 2]);
        v.y = step(row[g + 1]);
        v.x = step(row[g]);
        __stcs(reinterpret_cast<uint4*>(orow + g), v);
      }
    } else {
      for (int wi = wpo - 1; wi >= 0; --wi) orow[wi] = step(row[wi]);
    }
  }
}

// Parity bits of local columns lc0 .. lc0+7 of one bitmap row (lc0 may be negative when the tile
// is not 8-aligned; missing bits read as 0).
__device__ __forceinline__ uint32_t bits8(const uint32_t* __restrict__ row, int wpr, int lc0) {
  if (lc0 >= 0) {
    const int wi = lc0 >> 5, sh = lc0 & 31;
    uint64_t v = row[wi];
    if (sh > 24 && wi + 1 < wpr) v |= (uint64_t)row[wi + 1] << 32;
    return (uint32_t)(v >> sh) & 0xFFu;
  }
  return (row[0] << (-lc0)) & 0xFFu;
}

}  // namespace zh
