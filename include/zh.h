/* zh.h — C ABI of libzh, the B200-native (sm_100a) zonal-histogramming library.
 *
 * Operation (§III ¶1): given a raster R (M rows x N columns, integer values) and
 * polygons P_k, compute for every polygon the histogram
 *     H_k[b] = #{ cells (i, j) : centre of (i, j) inside P_k  and  bin(R[i][j]) = b }.
 * The cell CENTRE is the representative point (§III.D); "inside" is the even-odd
 * ray-crossing test of Franklin's PNPOLY over all rings of the polygon (Fig. 5 and
 * the multi-ring paragraph after it), evaluated in IEEE double with canonical edge orientation
 * and no FMA contraction (readings R7/R8/R10).
 *
 * The paper's four steps (§I, §III ¶1 and Fig. 1) are exposed one call
 * per step so each can be timed and tested:
 *   step 1 zh_tile_hist   per-tile histograms of T x T tiles           (PAPER.md:14 §III.A, :16 Fig. 2)
 *   step 2 zh_pair_tiles  MBB rasterisation pairing + inside/outside/intersect classification
 *                                                                        (§III.B, Fig. 3)
 *   step 3 zh_aggregate   add inside tiles' histograms to the polygons  (§III.C, Fig. 4)
 *   step 4 zh_pip_update  cell-in-polygon test for the cells of intersecting tiles
 *                                                                        (§III.D, Fig. 5)
 *   zh_run                steps 2, 1, 3, 4 (or 2 + fused) and the copy of the result to the host.
 *   zh_fused_update       steps 1 + 3 + 4 fused, tile by tile, each raster cell read at most once
 *                         (outside-only tiles are never read; tiles with only
 *                         inside pairs are histogrammed straight into their polygons; tiles with an
 *                         intersecting pair go through the step-4 kernel).  Bit-identical result.
 *
 * Conventions
 *  - Every call returns zh_status; nothing throws, exits or prints.  On failure
 *    zh_last_error() returns a thread-local message.  A failed call leaves the context usable;
 *    after ZH_ERR_CUDA the device state (and the output) is unspecified.
 *  - All device work is enqueued on options.stream (a cudaStream_t, NULL = legacy default
 *    stream).  Calls documented "syncs" block the host until the stream has drained.
 *  - Ownership: the raster is BORROWED (caller keeps it alive for the context's lifetime);
 *    polygons and bin parameters are COPIED by zh_create; tile histograms, pair lists and the
 *    output are OWNED by the context unless zh_set_output supplied a borrowed output buffer.
 *  - Index widths: offsets are int64 at the ABI; kernels use int32 internally, so n_vert,
 *    n_ring, the number of tiles and the number of tile/polygon pairs must stay < 2^31
 *    (else ZH_ERR_UNSUPPORTED).
 *  - Threading: a context is used by one host thread at a time.
 */
#ifndef ZH_H
#define ZH_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ZH_ABI_VERSION 8

typedef struct zh_ctx_s* zh_ctx;

typedef enum {
  ZH_OK = 0,
  ZH_ERR_INVALID_ARG = 1,  /* malformed input (see zh_create)                                 */
  ZH_ERR_UNSUPPORTED = 2,  /* valid but outside what the kernels support (rotated gt, >2^31)  */
  ZH_ERR_OOM = 3,          /* device allocation failed                                        */
  ZH_ERR_CUDA = 4,         /* a CUDA runtime error; message has the CUDA error string         */
  ZH_ERR_OVERFLOW = 5,     /* out_u64 = 0 requested but a count could exceed 2^32 - 1         */
  ZH_ERR_STATE = 6         /* call order violated (e.g. zh_aggregate before steps 1 and 2)     */
} zh_status;

/* Raster shard.  `data` points at the first element of row `row0` of the full raster.
 * Layout: row-major int16, `pitch` elements between consecutive rows (pitch >= cols).
 * on_host = 0: `data` is DEVICE memory (borrowed).  The fast paths need data % 16 == 0 and
 *   pitch % 8 == 0 (16-byte vector loads); other alignments are rejected (INVALID_ARG).
 * on_host = 1: `data` is HOST memory (borrowed; pin it for full PCIe speed); the context owns a
 *   device copy.  zh_upload_raster copies the whole shard host->device; zh_run does too, except
 *   with options.fused = 1, where it runs step 2 first and copies only the tiles that some
 *   (tile, polygon) pair needs (the fused kernels never read the others; zh_stats.h2d_bytes).
 * Geotransform (GDAL): x = gt[0] + col*gt[1] + row*gt[2], y = gt[3] + col*gt[4] + row*gt[5];
 *   the cell (r, c) has centre x = gt[0] + (c + 0.5)*gt[1], y = gt[3] + (r + 0.5)*gt[5]
 *   (with options.rep_custom: (c + rep_x), (r + rep_y) instead of the 0.5s).
 *   gt[2] and gt[4] must be 0 (north-up; rotated -> UNSUPPORTED); gt[1], gt[5] nonzero, finite.
 * Sharding (multi-GPU): a rank holds rows [row0, row0 + nrows) of an M x N raster; row0 must be
 *   a multiple of the tile size so that shards consist of whole tile rows. */
typedef struct {
  const int16_t* data;
  int64_t rows, cols;     /* full raster M, N                                                   */
  int64_t pitch;          /* elements between rows of `data`                                    */
  int64_t row0, nrows;    /* this shard's rows                                                  */
  double gt[6];
  int32_t on_host;
  int32_t reserved;
} zh_raster;

/* Polygons, HOST arrays, copied by zh_create (the caller may free them afterwards).
 * Polygon k owns rings poly_ring_off[k] .. poly_ring_off[k+1]-1; ring r owns vertices
 * ring_vert_off[r] .. ring_vert_off[r+1]-1.  Rings are closed implicitly (edge from the last
 * vertex back to the first); an explicit closing vertex is allowed and adds a zero-length edge.
 * Holes and multi-part polygons are just more rings (even-odd rule over all rings of a polygon,
 * the semantics of the paper's origin-sentinel trick).  Degenerate input is valid:
 * polygons with no rings, rings with 0-2 vertices, zero-area rings, polygons off the raster all
 * contribute nothing.  Offsets must be non-decreasing with [0] = 0 and the last = n_ring /
 * n_vert; coordinates finite (else INVALID_ARG). */
typedef struct {
  int64_t n_poly, n_ring, n_vert;
  const int64_t* poly_ring_off; /* n_poly + 1 */
  const int64_t* ring_vert_off; /* n_ring + 1 */
  const double* x;              /* n_vert     */
  const double* y;              /* n_vert     */
} zh_polygons;

/* Bin mapping (DESIGN.md §3 R3/R4; the paper assumes 0 <= v < B, and Fig. 2 does
 * no check):  a cell with use_nodata && v == nodata is never counted; otherwise
 * d = v - lo; d < 0 -> bin 0 (clamp) or not counted (oor_drop); b = d / width;
 * b >= nbins -> nbins-1 (clamp) or not counted (oor_drop).
 * Requires 1 <= nbins <= 49152 (shared-memory histograms), 1 <= width, |lo| <= 1<<30, and, with
 * use_nodata, -32768 <= nodata <= 32767 (an int16 value; else INVALID_ARG). */
typedef struct {
  int32_t lo, width, nbins;
  int32_t use_nodata, nodata;
  int32_t oor_drop;
} zh_bins;

typedef struct {
  int32_t tile;        /* 1 <= T <= 46340, arbitrary ("allow users to set it
                          arbitrarily"); partial edge tiles hold only real cells; T > 46340 ->
                          UNSUPPORTED (per-tile counts are uint32: T^2 < 2^31)                   */
  int32_t out_u64;     /* 1: uint64 output (default); 0: uint32 (ZH_ERR_OVERFLOW at zh_create if
                          some polygon's MBB could hold >= 2^32 cells)                           */
  int32_t force_isect; /* 1: classify every non-outside pair as intersecting (skips step 3's
                          work; a validation mode — the result must not change)                  */
  int32_t fused;       /* 1: zh_run uses zh_fused_update instead of steps 1, 3, 4               */
  void* stream;        /* cudaStream_t                                                          */
  int32_t rep_custom;  /* 0: the cell CENTRE is the representative point (§III.D);
                          1: the point (c + rep_x, r + rep_y) in cell units, rep_x, rep_y in
                          [0, 1] — e.g. (0, 0) the cell corner at the origin of the cell
                          (the alternatives of PAPER.md:18)                   */
  int32_t cover;       /* 0: a cell counts in P_k when its representative point is inside (the
                          paper's choice, §III.D); 1: when its CLOSED rectangle meets
                          the CLOSED polygon — the literal "cells that geometrically intersect
                          with P_k" of PAPER.md:12 §III ¶1 (R15; touching counts).
                          Requires rep_custom = 0 (ZH_ERR_UNSUPPORTED otherwise)               */
  double rep_x, rep_y;
} zh_options;

typedef struct {
  int64_t n_tiles;        /* tiles of this shard                                                */
  int64_t n_candidates;   /* (tile, polygon) pairs from MBB rasterisation                      */
  int64_t n_inside;       /* pairs classified inside (step 3 work)                              */
  int64_t n_isect;        /* pairs classified intersecting (step 4 work)                        */
  int64_t n_band_entries; /* (edge, tile-row) entries of the step-4 edge lists                  */
  int64_t n_edges;        /* polygon edges                                                      */
  int64_t device_bytes;   /* device memory owned by the context                                 */
  int64_t n_pure_tiles;   /* after zh_fused_update: tiles histogrammed straight into polygons     */
  int64_t n_pip_pairs;    /* after zh_fused_update: pairs sent to the cell-in-polygon kernel      */
  int64_t n_pure_cells;   /* cells of those pure tiles                                          */
  int64_t n_pip_cells;    /* cells of the tiles of those pairs (counted once per pair)           */
  int64_t h2d_bytes;      /* on_host rasters: bytes copied host->device by the last zh_run /
                             zh_upload_raster                                                   */
  int64_t n_mixed_groups; /* after zh_fused_update: tile groups (<= 2 pairs of one tile) of the
                             grouped cell kernel (0 when it does not apply)                      */
  int64_t n_group_cells;  /* cells those groups read (a mixed tile once per group)              */
  int64_t n_mixed_cells;  /* cells of the mixed tiles, each once (the HBM bytes the grouped cell
                             kernel must read: a tile's later groups find it in L2)              */
} zh_stats;

/* Validate, copy polygons to the device (H2D on options->stream), allocate per-tile histograms
 * and the output.  *out is set only on ZH_OK. */
zh_status zh_create(zh_ctx* out, const zh_raster* raster, const zh_polygons* polys, const zh_bins* bins,
                    const zh_options* options);

/* on_host rasters: enqueue the host->device copy of the shard (zh_run does this itself). */
zh_status zh_upload_raster(zh_ctx ctx);

/* Step 1 (async): tile_hist[t][b] for every tile t of the shard (the first call allocates the
 * n_tiles x B_pad uint32 array). */
zh_status zh_tile_hist(zh_ctx ctx);

/* Step 2: edge preparation, MBB pairing, classification, pair lists; zeroes the output.
 * Syncs the stream (twice) to size its lists.  n_inside / n_isect may be NULL. */
zh_status zh_pair_tiles(zh_ctx ctx, int64_t* n_inside, int64_t* n_isect);

/* Step 3 (async): out[k][b] += sum of tile_hist[t][b] over inside tiles t of k.
 * Needs steps 1 and 2 since the last zh_pair_tiles, else ZH_ERR_STATE. */
zh_status zh_aggregate(zh_ctx ctx);

/* Step 4 (async): for every intersecting (tile, polygon) pair and every cell of the tile whose
 * centre is inside the polygon, out[k][bin(v)] += 1.  Needs step 2, else ZH_ERR_STATE. */
zh_status zh_pip_update(zh_ctx ctx);

/* Steps 1 + 3 + 4 fused (async).  Needs step 2; exclusive with zh_aggregate / zh_pip_update for the
 * same zh_pair_tiles (ZH_ERR_STATE).  Does not need (or fill) the per-tile histograms. */
zh_status zh_fused_update(zh_ctx ctx);

/* Upload (on_host), steps 2, 1, 3, 4 (or 2 + fused when options.fused), then copy n_poly * nbins elements (uint64 or uint32 per
 * out_u64, row-major [n_poly][nbins]) to host_out (may be NULL to skip the copy).  Syncs.
 * on_host with options.fused: the upload follows step 2 and covers only the needed tiles (see
 * zh_raster). */
zh_status zh_run(zh_ctx ctx, void* host_out);

/* One whole step — zh_pair_tiles + zh_fused_update (options.fused = 1), else zh_pair_tiles +
 * zh_tile_hist + zh_aggregate + zh_pip_update — replayed from a CUDA graph.  The step's list sizes
 * are a function of the context's fixed geometry: the first call runs the step directly and learns
 * them (host syncs); the next call captures the step (on a context-owned stream) and every later
 * call launches the captured graph: one launch, no host round trip.  A device check compares each
 * replay's counts with the learnt sizes and any mismatch is reported (ZH_ERR_STATE) by the next
 * syncing call.  Enqueued on options.stream, asynchronous; afterwards the histogram is complete
 * as after the individual calls.  zh_set_output / zh_set_timing drop the captured graph.  Host
 * rasters need zh_upload_raster (or a zh_run) first. */
zh_status zh_step_graph(zh_ctx ctx);

/* Device memory of destroyed contexts is kept in a process-wide cache and reused by later
 * contexts of the same device (no cudaMalloc / cudaFree of the raster copy per zh_create /
 * zh_destroy cycle); allocations that fail return the cache to the driver and retry.  The
 * contexts' small pinned host buffers are cached the same way (cudaFreeHost can stall for
 * hundreds of ms while a large host raster is pinned).
 * zh_trim_cache frees every cached block; keep_caching = 0 also disables caching from then on.
 * zh_cache_bytes: bytes currently cached. */
void zh_trim_cache(int32_t keep_caching);
int64_t zh_cache_bytes(void);

/* Zonal statistics from the histograms (the classic per-zone min, max, average,
 * count and standard deviation of PAPER.md:10 §I ¶1), exact integers in units of bin indices b
 * (value of bin b = lo + b * width).  Per polygon ZH_NSTATS int64:
 *   [0] count  [1] min_bin  [2] max_bin  [3] lower-median bin  (bins -1 for an empty polygon)
 *   [4] sum of b  [5],[6] sum of b^2 as (low, high) 64-bit words of a 128-bit integer
 *   [7] number of non-zero bins
 * Needs a completed histogram since the last zh_pair_tiles (zh_run, steps 3+4, or the fused
 * update).  host_stats (n_poly * ZH_NSTATS, may be NULL) receives a copy (syncs); *dptr (may be
 * NULL) a BORROWED device pointer. */
#define ZH_NSTATS 8
zh_status zh_zonal_stats(zh_ctx ctx, int64_t* host_stats, int64_t** dptr);

/* Zonal summary in value units (the "min, max, average, count and standard deviation" of
 * PAPER.md:10 §I ¶1), derived on the device from zh_zonal_stats' exact integers n = count,
 * S1 = sum_b b*H[b], S2 = sum_b b^2*H[b].  A bin stands for the value lo + b*width (its lower
 * edge: the cell value itself for width = 1 and unclamped cells; R16).  Per polygon
 * ZH_NSUMMARY doubles, every step ONE correctly rounded binary64 operation (bit-reproducible):
 *   [0] count = n
 *   [1] min, [2] max, [3] lower median = lo + b*width for the bins of zh_zonal_stats (exact)
 *   [4] mean = lo + width * (S1 / n)                         (RN of: S1 -> double, /, *, +)
 *   [5] std  = width * (sqrt(D) / n), D = n*S2 - S1^2         (population standard deviation;
 *            D exact in 128 bits, then RN of: D -> double, sqrt, /, *)
 * [1]..[5] are NaN for an empty polygon.  Requires every count < 2^40.  Needs a completed
 * histogram (as zh_zonal_stats).  host_out (n_poly * ZH_NSUMMARY, may be NULL) receives a copy
 * (syncs); *dptr (may be NULL) a BORROWED device pointer. */
#define ZH_NSUMMARY 6
zh_status zh_zonal_summary(zh_ctx ctx, double* host_out, double** dptr);

/* Histogram feature distances (§I ¶1: the per-zone histograms "can further be used
 * as feature vectors for ... computing various distance measurements which can be used for
 * subsequent clustering").  Between the NORMALISED histograms p = H_a / n_a, q = H_b / n_b of
 * polygons a and b (n = count):
 *   ZH_DIST_L1   sum_b |p_b - q_b|                       = RN(RN(RN(N) / n_1) / n_2),
 *                N = sum_b |H_a[b]*n_b - H_b[b]*n_a|  (an exact 128-bit integer: bit-exact)
 *   ZH_DIST_EMD  sum_b |P_b - Q_b|, P, Q the cumulative distributions (1-D earth mover's
 *                distance in bin units; times width for value units); same form with the
 *                cumulative counts C_a[b] = sum_{b' <= b} H_a[b'] in place of H (bit-exact)
 *   ZH_DIST_CHI2 1/2 sum_{b: p_b + q_b > 0} (p_b - q_b)^2 / (p_b + q_b), evaluated as
 *                0.5 * RN(RN(sum_b RN(RN(d^2) / s)) / n_1) / n_2) with d = RN(|H_a[b] n_b - H_b[b] n_a|),
 *                s = RN(H_a[b] n_b + H_b[b] n_a), the sum in an unspecified order: relative
 *                error <= (nbins + 8) * 2^-53
 * (n_1 = min(n_a, n_b), n_2 = max(n_a, n_b): the result is symmetric in a and b.)
 * NaN when either polygon is empty.  a_ids, b_ids: HOST int32 arrays of n polygon ids (each in
 * [0, n_poly), else INVALID_ARG); host_out[i] = d(a_ids[i], b_ids[i]).  a_ids = b_ids = NULL:
 * ALL pairs, host_out is [n_poly][n_poly] row-major (n ignored), symmetric, zero diagonal for
 * non-empty polygons.  Needs a completed histogram (as zh_zonal_stats).  Syncs. */
#define ZH_DIST_L1 0
#define ZH_DIST_EMD 1
#define ZH_DIST_CHI2 2
zh_status zh_hist_distance(zh_ctx ctx, int32_t kind, const int32_t* a_ids, const int32_t* b_ids, int64_t n,
                           double* host_out);

/* Work-balanced multi-GPU decomposition (the paper's future work on load
 * balancing across nodes, §IV.C): split the raster's rows into n_shards contiguous
 * ranges of WHOLE tile rows with about equal estimated work, from step 2's pair lists over the
 * full raster (geometry only: raster values are not read; raster->data, row0, nrows and on_host
 * are ignored).  row_bounds receives n_shards + 1 row indices (0 = first, rows = last); shard s
 * holds rows [row_bounds[s], row_bounds[s+1]) (possibly empty).  shard_cost (may be NULL)
 * receives the estimated cost of each shard (arbitrary units).  Runs on options->stream; syncs. */
zh_status zh_plan_rows(const zh_raster* raster, const zh_polygons* polys, const zh_options* options,
                       int32_t n_shards, int64_t* row_bounds, double* shard_cost);

/* BORROWED device pointer to the output ([n_poly][nbins], uint64 or uint32) — e.g. for an
 * NCCL reduce across shards.  *n = n_poly * nbins elements. */
zh_status zh_output_device(zh_ctx ctx, void** dptr, int64_t* n);

/* Use a caller-owned device buffer (n_poly * nbins elements, 8-byte aligned) as the output
 * from now on (BORROWED, must outlive the context).  NULL reverts to the context's own. */
zh_status zh_set_output(zh_ctx ctx, void* dptr);

/* Copy the per-tile histograms of the shard ([n_tiles][nbins] uint32, tile id = local tile row *
 * tile columns + tile column) to host memory (testing/inspection).  Syncs. */
zh_status zh_copy_tile_hist(zh_ctx ctx, uint32_t* host, int64_t n_elems);

/* Copy step 2's pair lists to host memory (testing).  inside: n_inside (tile, poly) int32 pairs;
 * isect: n_isect (tile, poly) int32 pairs; either may be NULL.  Syncs. */
zh_status zh_copy_pairs(zh_ctx ctx, int32_t* inside, int32_t* isect);

zh_status zh_get_stats(zh_ctx ctx, zh_stats* stats);

/* Device time (ms) of the last call of each step, measured with CUDA events on the context stream
 * when timing is enabled (zh_set_timing).  Up to n values: [0..3] steps 1..4, [4] zh_fused_update,
 * [5] its pure-tile kernel, [6] its cell-in-polygon kernel; -1 for a call not made since timing
 * was enabled.  Syncs. */
zh_status zh_set_timing(zh_ctx ctx, int32_t enable);
zh_status zh_get_step_ms(zh_ctx ctx, float* ms, int32_t n);

/* Number of kernel launches the context has enqueued since creation (self-reported). */
int64_t zh_launch_count(zh_ctx ctx);

const char* zh_last_error(void);
int32_t zh_abi_version(void);

/* Frees the context's device memory (after synchronising its stream). NULL is a no-op. */
void zh_destroy(zh_ctx ctx);

#ifdef __cplusplus
}
#endif
#endif /* ZH_H */
