// k_touch.cu — the "geometrically intersect" variant of step 4 (reading R15, §III ¶1:
// "the raster cells that geometrically intersect with P_k"; the paper itself then tests the cell
// centre, §III.D).  A cell counts in P_k when its CLOSED rectangle meets the CLOSED
// polygon: its centre is inside (the parity bits k_parity already stored), or some edge of P_k
// meets the rectangle.  This kernel ORs the second set into the per-pair parity bitmaps before
// k_pip_cells streams the cells, so the cell pass is unchanged.
//
// Why only the intersecting pairs: a cell an edge reaches lies in a tile whose rectangle the edge's
// bounding box meets, and step 2 marks every such (tile, polygon) pair INTERSECT (k_mark); inside
// tiles have no edge within a cell, so there cover == centre (all cells).
//
// Work: one CTA per polygon, its edges walked along their MAJOR axis (rows for steep edges, columns
// for flat ones): per slab of the major axis the segment covers a short run of the minor axis
// (<= slope + 1 cells), found with a guess of +-1 cell and decided EXACTLY per candidate cell by the
// separating-axis test below — the same binary64 expression, operand order and no-FMA rule as the
// oracle (oracle/zh_oracle.c zho_seg_touches; the two share no code).  Short edges: thread per
// edge; long ones: a warp per edge, lane per slab.
#include "zh_ctx.h"

namespace zh {

// Grid lines X(c) = gt0 + c*gt1, Y(r) = gt3 + r*gt5 (two IEEE ops each).
__device__ __forceinline__ double grid_x(const Geo& g, int64_t c) { return __dadd_rn(g.gt0, __dmul_rn((double)c, g.gt1)); }
__device__ __forceinline__ double grid_y(const Geo& g, int64_t r) { return __dadd_rn(g.gt3, __dmul_rn((double)r, g.gt5)); }

// Segment vs closed rectangle [X0,X1] x [Y0,Y1] (either order): bounding boxes overlap and the
// four corners are not all strictly on one side of the segment's line; endpoints ordered by (y, x).
__device__ __forceinline__ bool seg_touches(double x0, double y0, double x1, double y1, double X0, double X1,
                                            double Y0, double Y1) {
  const double xlo = fmin(X0, X1), xhi = fmax(X0, X1), ylo = fmin(Y0, Y1), yhi = fmax(Y0, Y1);
  if (fmax(x0, x1) < xlo || fmin(x0, x1) > xhi || fmax(y0, y1) < ylo || fmin(y0, y1) > yhi) return false;
  double xa = x0, ya = y0, xb = x1, yb = y1;
  if (ya > yb || (ya == yb && xa > xb)) { xa = x1; ya = y1; xb = x0; yb = y0; }
  const double dx = __dsub_rn(xb, xa), dy = __dsub_rn(yb, ya);
  const double cx[4] = {xlo, xhi, xlo, xhi}, cy[4] = {ylo, ylo, yhi, yhi};
  int pos = 0, neg = 0;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const double o = __dsub_rn(__dmul_rn(dx, __dsub_rn(cy[i], ya)), __dmul_rn(dy, __dsub_rn(cx[i], xa)));
    pos += o > 0.0;
    neg += o < 0.0;
  }
  return !(pos == 4 || neg == 4);
}

struct TouchP {
  RasterP rp;
  Geo g;
  const int32_t* pro;
  const int32_t* rvo;
  const Edge* edges;
  const int4* mbb;
  const int64_t* cand_off;
  const uint8_t* cls;
  const uint64_t* flag_pos;  // isect index of a candidate = flag_pos >> 32
  const int32_t* remap;      // isect index -> index in the pair list of k_parity (nullptr: identity)
  uint32_t* pbits;           // [pair][T][wpo]
  int wpo;
  double igt1, igt5;         // 1/gt1, 1/gt5 (candidate ranges only)
};

// Mark cell (r, c) of polygon k as covered in its pair's bitmap.
__device__ __forceinline__ void mark_cell(const TouchP& p, int k, const int4& m, int64_t r, int64_t c) {
  const int T = p.rp.T;
  const int tr = (int)(r / T), tc = (int)(c / T);
  if (tr < m.z || tr > m.w || tc < m.x || tc > m.y) return;  // cannot happen (1-cell MBB margin)
  const int64_t ci = p.cand_off[k] + (int64_t)(tr - m.z) * (m.y - m.x + 1) + (tc - m.x);
  if (p.cls[ci] != 2) return;  // cannot happen (k_mark marks every tile an edge box reaches)
  int64_t pi = (int64_t)(p.flag_pos[ci] >> 32);
  if (p.remap) pi = p.remap[pi];
  const int lr = (int)(r - (int64_t)tr * T), lc = (int)(c - (int64_t)tc * T);
  atomicOr(&p.pbits[pi * (int64_t)T * p.wpo + (int64_t)lr * p.wpo + (lc >> 5)], 1u << (lc & 31));
}

// Candidate cell indices [ceil(q0 - d) - 1, floor(q1 + d)] along an axis for a real-valued index
// interval [q0, q1]: cell j spans [j, j + 1] in index units, and it can meet the interval only if
// j <= q1 and j + 1 >= q0.  d = 1e-3 cell absorbs the rounding of the (approximate) guesses; the
// exact test decides every candidate.
constexpr double kSlack = 1e-3;

// Cells of slab i (a row when `rows`, else a column) that the segment meets: the minor-axis range
// of the segment clipped to the slab (approximate: reciprocals, no exact arithmetic needed for a
// candidate range), then the exact test for each candidate cell.
__device__ __forceinline__ void touch_slab(const TouchP& p, int k, const int4& m, const Edge& e, bool rows,
                                           int64_t i, int64_t lo2, int64_t hi2, double inv_da) {
  const Geo& g = p.g;
  const double s0 = rows ? grid_y(g, i) : grid_x(g, i), s1 = rows ? grid_y(g, i + 1) : grid_x(g, i + 1);
  const double slo = fmin(s0, s1), shi = fmax(s0, s1);
  const double a0 = rows ? e.ya : e.xa, a1 = rows ? e.yb : e.xb;  // major coordinates of the ends
  const double b0 = rows ? e.xa : e.ya, b1 = rows ? e.xb : e.yb;  // minor coordinates
  double bmin, bmax;
  if (a0 == a1) {
    bmin = fmin(b0, b1);
    bmax = fmax(b0, b1);
  } else {
    const double t0 = fmin(fmax((slo - a0) * inv_da, 0.0), 1.0), t1 = fmin(fmax((shi - a0) * inv_da, 0.0), 1.0);
    const double u0 = b0 + t0 * (b1 - b0), u1 = b0 + t1 * (b1 - b0);
    bmin = fmin(u0, u1);
    bmax = fmax(u0, u1);
  }
  double q0 = rows ? (bmin - g.gt0) * p.igt1 : (bmin - g.gt3) * p.igt5;
  double q1 = rows ? (bmax - g.gt0) * p.igt1 : (bmax - g.gt3) * p.igt5;
  if (q0 > q1) { const double t = q0; q0 = q1; q1 = t; }
  const double jlo = fmax(ceil(q0 - kSlack) - 1.0, (double)lo2), jhi = fmin(floor(q1 + kSlack), (double)hi2);
  if (!(jlo <= jhi)) return;
  for (int64_t j = (int64_t)jlo; j <= (int64_t)jhi; ++j) {
    const int64_t r = rows ? i : j, c = rows ? j : i;
    if (seg_touches(e.xa, e.ya, e.xb, e.yb, grid_x(g, c), grid_x(g, c + 1), grid_y(g, r), grid_y(g, r + 1)))
      mark_cell(p, k, m, r, c);
  }
}

// Major axis and slab range of an edge (clipped to the shard rows / raster columns); false if empty.
__device__ __forceinline__ bool edge_slabs(const TouchP& p, const Edge& e, bool& rows, int64_t& i0, int64_t& i1,
                                           int64_t& lo2, int64_t& hi2, double& inv_da) {
  const Geo& g = p.g;
  const RasterP& rp = p.rp;
  double ca = (fmin(e.xa, e.xb) - g.gt0) * p.igt1, cb = (fmax(e.xa, e.xb) - g.gt0) * p.igt1;
  if (ca > cb) { const double t = ca; ca = cb; cb = t; }
  double ra = (e.ya - g.gt3) * p.igt5, rb = (e.yb - g.gt3) * p.igt5;
  if (ra > rb) { const double t = ra; ra = rb; rb = t; }
  const double R0 = (double)rp.row0, R1 = (double)(rp.row0 + rp.nrows - 1), C1 = (double)(rp.cols - 1);
  const double rlo = fmax(ceil(ra - kSlack) - 1.0, R0), rhi = fmin(floor(rb + kSlack), R1);
  const double clo = fmax(ceil(ca - kSlack) - 1.0, 0.0), chi = fmin(floor(cb + kSlack), C1);
  if (!(rlo <= rhi) || !(clo <= chi)) return false;
  rows = (rb - ra) >= (cb - ca);
  if (rows) { i0 = (int64_t)rlo; i1 = (int64_t)rhi; lo2 = 0; hi2 = rp.cols - 1; }
  else      { i0 = (int64_t)clo; i1 = (int64_t)chi; lo2 = rp.row0; hi2 = rp.row0 + rp.nrows - 1; }
  const double da = rows ? e.yb - e.ya : e.xb - e.xa;
  inv_da = da != 0.0 ? 1.0 / da : 0.0;
  return true;
}

constexpr int kTouchLong = 16;   // slabs above which an edge goes to the warp queue
constexpr int kTouchQ = 256;

__global__ void __launch_bounds__(256) k_touch(TouchP p) {
  const int k = blockIdx.x;
  const int4 m = p.mbb[k];
  if (m.x > m.y) return;
  __shared__ int qn;
  __shared__ int q[kTouchQ];
  if (threadIdx.x == 0) qn = 0;
  __syncthreads();
  const int vb = p.rvo[p.pro[k]], ve = p.rvo[p.pro[k + 1]];
  for (int v = vb + threadIdx.x; v < ve; v += blockDim.x) {
    const Edge e = p.edges[v];
    bool rows;
    int64_t i0, i1, lo2, hi2;
    double ida;
    if (!edge_slabs(p, e, rows, i0, i1, lo2, hi2, ida)) continue;
    if (i1 - i0 + 1 > kTouchLong) {
      const int pos = atomicAdd(&qn, 1);
      if (pos < kTouchQ) {
        q[pos] = v;
        continue;
      }
    }
    for (int64_t i = i0; i <= i1; ++i) touch_slab(p, k, m, e, rows, i, lo2, hi2, ida);
  }
  __syncthreads();
  const int nq = min(qn, kTouchQ);
  const int lane = threadIdx.x & 31;
  for (int qi = threadIdx.x >> 5; qi < nq; qi += blockDim.x >> 5) {
    const Edge e = p.edges[q[qi]];
    bool rows;
    int64_t i0, i1, lo2, hi2;
    double ida;
    edge_slabs(p, e, rows, i0, i1, lo2, hi2, ida);
    for (int64_t i = i0 + lane; i <= i1; i += 32) touch_slab(p, k, m, e, rows, i, lo2, hi2, ida);
  }
}

cudaError_t launch_touch(Ctx& c, const int32_t* remap, cudaStream_t s) {
  if (c.P == 0 || c.n_isect == 0) return cudaSuccess;
  TouchP p;
  p.rp = c.rp;
  p.g = c.geo;
  p.pro = c.d_pro.as<int32_t>();
  p.rvo = c.d_rvo.as<int32_t>();
  p.edges = c.d_edges.as<Edge>();
  p.mbb = c.d_mbb.as<int4>();
  p.cand_off = c.d_cand_off.as<int64_t>();
  p.cls = c.d_class.as<uint8_t>();
  p.flag_pos = c.d_flag_pos.as<uint64_t>();
  p.remap = remap;
  p.pbits = c.d_pbits.as<uint32_t>();
  p.wpo = (c.rp.T + 31) / 32;
  p.igt1 = 1.0 / c.geo.gt1;
  p.igt5 = 1.0 / c.geo.gt5;
  k_touch<<<(unsigned)c.P, 256, 0, s>>>(p);
  c.launches += 1;
  return cudaGetLastError();
}

}  // namespace zh
