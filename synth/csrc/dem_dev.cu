/* dem_dev.cu — device evaluation of the counter-based DEM generator (INPUT GENERATION ONLY).
 * Bit-identical to dem_host.c (same dem_core.h).  Not part of the zonal-histogram path:
 * it only fills the synthetic raster that bench.py / tests hand to libzh. */
#include <cuda_runtime.h>
#include "dem_core.h"

__global__ void zhs_fill_kernel(zhs_dem_params p, int kind, int32_t pm, int32_t poff, int64_t gcols,
                                int16_t* __restrict__ out, int64_t row0, int64_t col0,
                                int64_t nrows, int64_t ncols, int64_t pitch) {
  const int64_t n = nrows * ncols;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t rr = i / ncols, cc = i - rr * ncols;
    int16_t v = (kind == 0) ? zhs_dem_cell(&p, row0 + rr, col0 + cc)
                            : zhs_pattern_cell(kind, row0 + rr, col0 + cc, gcols, pm, poff);
    out[rr * pitch + cc] = v;
  }
}

extern "C" int zhs_fill_device(const zhs_dem_params* p, int kind, int32_t pm, int32_t poff, int64_t gcols,
                               int16_t* out, int64_t row0, int64_t col0, int64_t nrows, int64_t ncols,
                               int64_t pitch, void* stream) {
  if (nrows <= 0 || ncols <= 0) return 0;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  zhs_fill_kernel<<<sms * 16, 256, 0, (cudaStream_t)stream>>>(*p, kind, pm, poff, gcols, out, row0, col0,
                                                              nrows, ncols, pitch);
  return (int)cudaGetLastError();
}
