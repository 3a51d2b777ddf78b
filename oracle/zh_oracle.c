/* zh_oracle.c — CPU ORACLE for zonal histogramming.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  The product path (libzh.so, paper_conf_ipps_zhangw14_b200)
 * never does; the two share no code, headers or constants.
 *
 * What it computes is the plain definition of the method's result (§III ¶1):
 *   for every polygon P_k and bin b,  H_k[b] = #{ cells (i,j) : centre(i,j) in P_k and bin(v_ij) = b }
 * with the cell-centre choice of PAPER.md:18 §III.D ("we choose the center of a raster cell
 * for point-in-polygon test") and the ray-crossing (even-odd) test of PAPER.md:20 Fig. 5
 * (Franklin's PNPOLY, the italic code), applied over all rings of a polygon (PAPER.md:20,
 * the multi-ring paragraph after Fig. 5).  The four-step tiling of the paper only skips work
 * (§II end), so the definition is the oracle.
 *
 * Readings (DESIGN.md §3 lists them all):
 *   R1 cell centre inside (":18") rather than "geometrically intersect" (":12");
 *   R2 0 <= i < M, 0 <= j < N;
 *   R3 bin = (v - lo) / width, clamped to [0, nbins-1] (default) or dropped (oor_drop);
 *   R4 nodata cells are never counted;
 *   R5 int16 input, bins in int32;
 *   R7 double precision, each operation a separate IEEE-754 binary64 op (built with
 *      -ffp-contract=off: no FMA contraction);
 *   R8 canonical edge orientation: endpoints ordered so that ya <= yb before evaluating
 *      Franklin's expression xi = (xb - xa) * (yc - ya) / (yb - ya) + xa, left to right;
 *   R9 rings given by offsets, closed implicitly (edge v_{n-1} -> v_0);
 *   R10 half-open crossing rule: edge straddles iff ya <= yc < yb; crossing iff xc < xi;
 *   R15 (cover variant only) "geometrically intersect": closed cell rectangle meets the closed
 *       polygon (see zho_cover_o0 at the end of this file).
 *
 * Functions:
 *   zho_bin            R3/R4 value -> bin (or -1)
 *   zho_centre         cell centre from the GDAL geotransform
 *   zho_crossings      number of crossings of the ray from (xc,yc) toward +x (Fig. 5 counts)
 *   zho_o0             O0: literally the definition, every cell x every polygon x every edge
 *                      (optional exact bounding-box prefilter, see below)
 *   zho_o1             O1: the same comparisons hoisted per row: for each row and polygon
 *                      whose y-range holds the row, the intercepts xi of the straddling edges
 *                      are computed with the same expression, sorted, and the cells are walked
 *                      in increasing xc; a cell is inside iff #{xi > xc} is odd.  It evaluates
 *                      exactly the same (xc < xi) comparisons as O0, only once per
 *                      (edge,row) instead of once per (edge,cell).  Pinned O0 == O1.
 *   zho_seg_touches    R15: does a segment meet a closed cell rectangle (separating-axis test)
 *   zho_cover_o0       the "geometrically intersect" variant: a cell counts in P_k
 *                      when its closed rectangle meets the closed polygon — its centre is inside
 *                      (the test above) or some edge of P_k meets the rectangle (end of file)
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#if defined(__FP_FAST_FMA) && !defined(ZHO_ALLOW_FMA)
/* a hint only: the build uses -ffp-contract=off, which is what matters */
#endif

typedef struct {
  int32_t lo, width, nbins, use_nodata, nodata, oor_drop;
} zho_bins;

/* R3/R4: value -> bin, or -1 when the cell is not counted. */
int zho_bin(int32_t v, const zho_bins* b) {
  if (b->use_nodata && v == b->nodata) return -1;
  int32_t d = v - b->lo;
  if (d < 0) return b->oor_drop ? -1 : 0;
  int32_t q = d / b->width;
  if (q >= b->nbins) return b->oor_drop ? -1 : b->nbins - 1;
  return q;
}

/* Cell centre (GDAL convention, north-up: gt2 = gt4 = 0).  gt has 8 entries: gt[6], gt[7] are the
 * representative point's offsets inside the cell in cell units — 0.5, 0.5 for the centre the paper
 * chooses (§III.D); other points are its alternatives (e.g. 0, 0: a corner). */
void zho_centre(const double* gt, int64_t r, int64_t c, double* xc, double* yc) {
  double cc = (double)c + gt[6];
  double rr = (double)r + gt[7];
  double tx = cc * gt[1];
  double ty = rr * gt[5];
  *xc = gt[0] + tx;
  *yc = gt[3] + ty;
}

/* One edge, Franklin's predicate in canonical orientation (R8, R10).
 * Returns 1 if the edge is crossed by the ray from (xc, yc) toward +x. */
static inline int edge_crossed(double x0, double y0, double x1, double y1, double xc, double yc) {
  double xa, ya, xb, yb;
  if (y0 <= y1) { xa = x0; ya = y0; xb = x1; yb = y1; }
  else          { xa = x1; ya = y1; xb = x0; yb = y0; }
  if (!(ya <= yc && yc < yb)) return 0;
  double t1 = xb - xa;
  double t2 = yc - ya;
  double t3 = t1 * t2;
  double t4 = yb - ya;
  double t5 = t3 / t4;
  double xi = t5 + xa;
  return xc < xi;
}

/* Intercept of a straddling edge with the row y = yc (same expression as edge_crossed). */
static inline int edge_intercept(double x0, double y0, double x1, double y1, double yc, double* xi) {
  double xa, ya, xb, yb;
  if (y0 <= y1) { xa = x0; ya = y0; xb = x1; yb = y1; }
  else          { xa = x1; ya = y1; xb = x0; yb = y0; }
  if (!(ya <= yc && yc < yb)) return 0;
  double t1 = xb - xa;
  double t2 = yc - ya;
  double t3 = t1 * t2;
  double t4 = yb - ya;
  double t5 = t3 / t4;
  *xi = t5 + xa;
  return 1;
}

/* Number of crossings of the +x ray from (xc, yc) with all rings of polygon k. */
int64_t zho_crossings(double xc, double yc, int64_t k, const int64_t* pro, const int64_t* rvo,
                      const double* x, const double* y) {
  int64_t n = 0;
  for (int64_t r = pro[k]; r < pro[k + 1]; ++r) {
    int64_t a = rvo[r], b = rvo[r + 1];
    int64_t m = b - a;
    for (int64_t i = 0; i < m; ++i) {
      int64_t j = (i + 1 == m) ? 0 : i + 1;
      n += edge_crossed(x[a + i], y[a + i], x[a + j], y[a + j], xc, yc);
    }
  }
  return n;
}

typedef struct { double xmin, xmax, ymin, ymax; int empty; } bbox_t;

static void poly_bbox(int64_t k, const int64_t* pro, const int64_t* rvo, const double* x, const double* y,
                      bbox_t* bb) {
  bb->empty = 1;
  bb->xmin = bb->ymin = INFINITY;
  bb->xmax = bb->ymax = -INFINITY;
  for (int64_t i = rvo[pro[k]]; i < rvo[pro[k + 1]]; ++i) {
    bb->empty = 0;
    if (x[i] < bb->xmin) bb->xmin = x[i];
    if (x[i] > bb->xmax) bb->xmax = x[i];
    if (y[i] < bb->ymin) bb->ymin = y[i];
    if (y[i] > bb->ymax) bb->ymax = y[i];
  }
}

/* O0 — the definition.  The raster window `win` holds rows [row0, row0+nrows) and columns
 * [col0, col0+ncols) of the full raster (`pitch` elements between rows); geotransform `gt`
 * refers to the full raster.  out[k*nbins + b] is ACCUMULATED (uint64).
 * prefilter = 0: every polygon tested at every cell (literal).
 * prefilter = 1: polygon k is skipped at a cell when yc < ymin_k or yc >= ymax_k (then no edge
 *   straddles, exact) or when xc < xmin_k - |gt1| or xc > xmax_k + |gt1| (then every intercept
 *   lies on one side of xc: the computed xi of a straddling edge lies within a few ulp of the
 *   edge's x-range, far less than one cell, and a closed ring is straddled an even number of
 *   times) — pinned against prefilter = 0 in tests/test_oracle_pins.py. */
void zho_o0(const int16_t* win, int64_t row0, int64_t col0, int64_t nrows, int64_t ncols, int64_t pitch,
            const double* gt, int64_t n_poly, const int64_t* pro, const int64_t* rvo, const double* x,
            const double* y, const zho_bins* bins, uint64_t* out, int prefilter, int nthreads) {
  bbox_t* bb = (bbox_t*)malloc(sizeof(bbox_t) * (size_t)(n_poly > 0 ? n_poly : 1));
  for (int64_t k = 0; k < n_poly; ++k) poly_bbox(k, pro, rvo, x, y, &bb[k]);
  const double mx = fabs(gt[1]);
  if (nthreads < 1) nthreads = 1;
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
  for (int64_t i = 0; i < nrows; ++i) {
    for (int64_t j = 0; j < ncols; ++j) {
      int32_t v = win[i * pitch + j];
      int b = zho_bin(v, bins);
      if (b < 0) continue;
      double xc, yc;
      zho_centre(gt, row0 + i, col0 + j, &xc, &yc);
      for (int64_t k = 0; k < n_poly; ++k) {
        if (prefilter) {
          if (bb[k].empty) continue;
          if (yc < bb[k].ymin || yc >= bb[k].ymax) continue;
          if (xc < bb[k].xmin - mx || xc > bb[k].xmax + mx) continue;
        }
        int64_t n = zho_crossings(xc, yc, k, pro, rvo, x, y);
        if (n & 1) __atomic_fetch_add(&out[k * bins->nbins + b], (uint64_t)1, __ATOMIC_RELAXED);
      }
    }
  }
  free(bb);
}

static int cmp_double(const void* a, const void* b) {
  double da = *(const double*)a, db = *(const double*)b;
  return (da > db) - (da < db);
}

/* O1 — row-hoisted, same comparisons as O0 (see the header comment). */
void zho_o1(const int16_t* win, int64_t row0, int64_t col0, int64_t nrows, int64_t ncols, int64_t pitch,
            const double* gt, int64_t n_poly, const int64_t* pro, const int64_t* rvo, const double* x,
            const double* y, const zho_bins* bins, uint64_t* out, int nthreads) {
  bbox_t* bb = (bbox_t*)malloc(sizeof(bbox_t) * (size_t)(n_poly > 0 ? n_poly : 1));
  int64_t maxv = 1;
  for (int64_t k = 0; k < n_poly; ++k) {
    poly_bbox(k, pro, rvo, x, y, &bb[k]);
    int64_t nv = rvo[pro[k + 1]] - rvo[pro[k]];
    if (nv > maxv) maxv = nv;
  }
  if (nthreads < 1) nthreads = 1;
  const int increasing = gt[1] > 0; /* xc increases with c */
#pragma omp parallel num_threads(nthreads)
  {
    double* xs = (double*)malloc(sizeof(double) * (size_t)maxv);
#pragma omp for schedule(dynamic, 1)
    for (int64_t i = 0; i < nrows; ++i) {
      const int64_t r = row0 + i;
      double xc0, yc;
      zho_centre(gt, r, col0, &xc0, &yc);
      for (int64_t k = 0; k < n_poly; ++k) {
        if (bb[k].empty || yc < bb[k].ymin || yc >= bb[k].ymax) continue; /* no edge straddles */
        int64_t n = 0;
        for (int64_t rg = pro[k]; rg < pro[k + 1]; ++rg) {
          int64_t a = rvo[rg], m = rvo[rg + 1] - a;
          for (int64_t e = 0; e < m; ++e) {
            int64_t f = (e + 1 == m) ? 0 : e + 1;
            double xi;
            if (edge_intercept(x[a + e], y[a + e], x[a + f], y[a + f], yc, &xi)) xs[n++] = xi;
          }
        }
        if (n == 0) continue;
        qsort(xs, (size_t)n, sizeof(double), cmp_double);
        /* cells whose xc lies outside [xs[0], xs[n-1]) have #{xi > xc} in {0, n}; with n even
         * (a closed ring is straddled an even number of times) they are outside.  Visit a
         * conservative column range around it (2 cells of margin) and evaluate each visited
         * cell exactly; when n is odd (cannot happen for closed rings) visit the whole row. */
        int64_t jlo = 0, jhi = ncols; /* window-relative, half-open */
        if ((n & 1) == 0) {
          double clo = (xs[0] - gt[0]) / gt[1] - gt[6];
          double chi = (xs[n - 1] - gt[0]) / gt[1] - gt[6];
          if (clo > chi) { double t = clo; clo = chi; chi = t; }
          double a0 = floor(clo) - 2 - (double)col0, a1 = ceil(chi) + 3 - (double)col0;
          if (a0 > (double)jlo) jlo = a0 > (double)ncols ? ncols : (int64_t)a0;
          if (a1 < (double)jhi) jhi = a1 < 0 ? 0 : (int64_t)a1;
        }
        if (jlo >= jhi) continue;
        /* walk in increasing xc; p = #{xi <= xc} via a pointer, inside iff (n - p) odd */
        int64_t p = 0;
        for (int64_t s = 0; s < jhi - jlo; ++s) {
          int64_t j = increasing ? jlo + s : jhi - 1 - s;
          double xc, ycc;
          zho_centre(gt, r, col0 + j, &xc, &ycc);
          while (p < n && !(xc < xs[p])) ++p; /* xs[p] <= xc  <=>  not (xc < xs[p]) */
          if (((n - p) & 1) == 0) continue;
          int b = zho_bin(win[i * pitch + j], bins);
          if (b < 0) continue;
          __atomic_fetch_add(&out[k * bins->nbins + b], (uint64_t)1, __ATOMIC_RELAXED);
        }
      }
    }
    free(xs);
  }
  free(bb);
}

/* Per-cell membership for a list of cells (sampled checks): writes inside[q*n_poly + k] in {0,1}. */
void zho_membership(const int64_t* rows, const int64_t* cols, int64_t nq, const double* gt, int64_t n_poly,
                    const int64_t* pro, const int64_t* rvo, const double* x, const double* y, uint8_t* inside,
                    int nthreads) {
  if (nthreads < 1) nthreads = 1;
#pragma omp parallel for schedule(dynamic, 16) num_threads(nthreads)
  for (int64_t q = 0; q < nq; ++q) {
    double xc, yc;
    zho_centre(gt, rows[q], cols[q], &xc, &yc);
    for (int64_t k = 0; k < n_poly; ++k)
      inside[q * n_poly + k] = (uint8_t)(zho_crossings(xc, yc, k, pro, rvo, x, y) & 1);
  }
}

/* ---------------------------------------------------------------------------------------------
 * Reading R15 — the literal "cells that geometrically intersect with P_k" (§III ¶1;
 * the paper then picks the cell centre, §III.D).  A cell (r, c) is the CLOSED
 * rectangle between the grid lines X(c), X(c+1) and Y(r), Y(r+1), with
 *     X(c) = gt0 + (double)c * gt1,   Y(r) = gt3 + (double)r * gt5   (two IEEE ops each, no FMA).
 * It meets the closed region of P_k iff its centre is inside P_k (the crossing test above, which
 * decides the cells no edge reaches) or some edge of P_k meets the rectangle.  Segment vs closed
 * rectangle is the separating-axis test: the bounding boxes overlap (closed comparisons) and the
 * four corners are not all strictly on one side of the segment's line, with the orientation
 *     o(P) = dx * (Py - ya) - dy * (Px - xa),   dx = xb - xa,  dy = yb - ya,
 * each product and difference one binary64 op, the endpoints ordered lexicographically by (y, x)
 * so that the result depends on the undirected segment only.  A segment that only touches the
 * rectangle (a corner or a side) meets it: the sets are closed (ST_Intersects semantics).
 * --------------------------------------------------------------------------------------------- */
static inline double grid_x(const double* gt, int64_t c) { double t = (double)c * gt[1]; return gt[0] + t; }
static inline double grid_y(const double* gt, int64_t r) { double t = (double)r * gt[5]; return gt[3] + t; }

int zho_seg_touches(double x0, double y0, double x1, double y1, double X0, double X1, double Y0, double Y1) {
  const double xlo = X0 < X1 ? X0 : X1, xhi = X0 < X1 ? X1 : X0;
  const double ylo = Y0 < Y1 ? Y0 : Y1, yhi = Y0 < Y1 ? Y1 : Y0;
  if ((x0 > x1 ? x0 : x1) < xlo || (x0 < x1 ? x0 : x1) > xhi) return 0;
  if ((y0 > y1 ? y0 : y1) < ylo || (y0 < y1 ? y0 : y1) > yhi) return 0;
  double xa = x0, ya = y0, xb = x1, yb = y1;
  if (ya > yb || (ya == yb && xa > xb)) { xa = x1; ya = y1; xb = x0; yb = y0; }
  const double dx = xb - xa, dy = yb - ya;
  const double cx[4] = {xlo, xhi, xlo, xhi}, cy[4] = {ylo, ylo, yhi, yhi};
  int pos = 0, neg = 0;
  for (int i = 0; i < 4; ++i) {
    double u = cy[i] - ya;
    double v = cx[i] - xa;
    double p = dx * u;
    double q = dy * v;
    double o = p - q;
    pos += o > 0;
    neg += o < 0;
  }
  return !(pos == 4 || neg == 4);
}

/* Does polygon k meet the closed rectangle of cell (r, c)? */
static int cell_covered(const double* gt, int64_t r, int64_t c, int64_t k, const int64_t* pro, const int64_t* rvo,
                        const double* x, const double* y) {
  double xc, yc;
  zho_centre(gt, r, c, &xc, &yc);
  if (zho_crossings(xc, yc, k, pro, rvo, x, y) & 1) return 1;
  const double X0 = grid_x(gt, c), X1 = grid_x(gt, c + 1), Y0 = grid_y(gt, r), Y1 = grid_y(gt, r + 1);
  for (int64_t rg = pro[k]; rg < pro[k + 1]; ++rg) {
    int64_t a = rvo[rg], m = rvo[rg + 1] - a;
    for (int64_t e = 0; e < m; ++e) {
      int64_t f = (e + 1 == m) ? 0 : e + 1;
      if (zho_seg_touches(x[a + e], y[a + e], x[a + f], y[a + f], X0, X1, Y0, Y1)) return 1;
    }
  }
  return 0;
}

/* The cover variant of O0 (gt[6], gt[7] must be 0.5: the centre decides the cells no edge reaches).
 * prefilter = 1 skips polygon k at a cell whose closed rectangle misses k's closed vertex bounding
 * box: then no edge meets it, and the centre, half a cell outside the box, is outside (the O0
 * prefilter argument) — pinned against prefilter = 0. */
void zho_cover_o0(const int16_t* win, int64_t row0, int64_t col0, int64_t nrows, int64_t ncols, int64_t pitch,
                  const double* gt, int64_t n_poly, const int64_t* pro, const int64_t* rvo, const double* x,
                  const double* y, const zho_bins* bins, uint64_t* out, int prefilter, int nthreads) {
  bbox_t* bb = (bbox_t*)malloc(sizeof(bbox_t) * (size_t)(n_poly > 0 ? n_poly : 1));
  for (int64_t k = 0; k < n_poly; ++k) poly_bbox(k, pro, rvo, x, y, &bb[k]);
  if (nthreads < 1) nthreads = 1;
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
  for (int64_t i = 0; i < nrows; ++i) {
    for (int64_t j = 0; j < ncols; ++j) {
      int b = zho_bin(win[i * pitch + j], bins);
      if (b < 0) continue;
      const int64_t r = row0 + i, c = col0 + j;
      const double X0 = grid_x(gt, c), X1 = grid_x(gt, c + 1), Y0 = grid_y(gt, r), Y1 = grid_y(gt, r + 1);
      const double xlo = X0 < X1 ? X0 : X1, xhi = X0 < X1 ? X1 : X0;
      const double ylo = Y0 < Y1 ? Y0 : Y1, yhi = Y0 < Y1 ? Y1 : Y0;
      for (int64_t k = 0; k < n_poly; ++k) {
        if (prefilter) {
          if (bb[k].empty) continue;
          if (xhi < bb[k].xmin || xlo > bb[k].xmax || yhi < bb[k].ymin || ylo > bb[k].ymax) continue;
        }
        if (cell_covered(gt, r, c, k, pro, rvo, x, y))
          __atomic_fetch_add(&out[k * bins->nbins + b], (uint64_t)1, __ATOMIC_RELAXED);
      }
    }
  }
  free(bb);
}

/* Per-cell cover membership for a list of cells: covered[q*n_poly + k] in {0,1}. */
void zho_cover_membership(const int64_t* rows, const int64_t* cols, int64_t nq, const double* gt, int64_t n_poly,
                          const int64_t* pro, const int64_t* rvo, const double* x, const double* y,
                          uint8_t* covered, int nthreads) {
  if (nthreads < 1) nthreads = 1;
#pragma omp parallel for schedule(dynamic, 16) num_threads(nthreads)
  for (int64_t q = 0; q < nq; ++q)
    for (int64_t k = 0; k < n_poly; ++k)
      covered[q * n_poly + k] = (uint8_t)cell_covered(gt, rows[q], cols[q], k, pro, rvo, x, y);
}
