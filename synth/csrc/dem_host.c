/* dem_host.c — host evaluation of the counter-based DEM generator (INPUT GENERATION ONLY).
 * Same function as synth/csrc/dem_dev.cu evaluates on the GPU (see dem_core.h). */
#include "dem_core.h"
#include <stddef.h>

/* Fill a window [row0, row0+nrows) x [col0, col0+ncols) of the global raster into
 * out (row-major, `pitch` elements between rows).  kind 0 = DEM, 1..3 = patterns. */
void zhs_fill_host(const zhs_dem_params* p, int kind, int32_t pm, int32_t poff, int64_t gcols,
                   int16_t* out, int64_t row0, int64_t col0, int64_t nrows, int64_t ncols,
                   int64_t pitch, int nthreads) {
  if (nthreads < 1) nthreads = 1;
#pragma omp parallel for schedule(dynamic, 4) num_threads(nthreads)
  for (int64_t i = 0; i < nrows; ++i) {
    int16_t* row = out + (size_t)i * (size_t)pitch;
    const int64_t r = row0 + i;
    if (kind == 0) {
      for (int64_t j = 0; j < ncols; ++j) row[j] = zhs_dem_cell(p, r, col0 + j);
    } else {
      for (int64_t j = 0; j < ncols; ++j) row[j] = zhs_pattern_cell(kind, r, col0 + j, gcols, pm, poff);
    }
  }
}
