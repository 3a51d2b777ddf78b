/* dem_core.h — counter-based synthetic SRTM-like DEM generator (INPUT GENERATION ONLY).
 *
 * This header holds no arithmetic of the zonal-histogramming method.  It is the one
 * piece shared by the CPU oracle side (compiled by gcc into libsynth_host.so) and the
 * GPU side (compiled by nvcc into libsynth_cuda.so): both evaluate the SAME pure
 * integer function of (seed, row, col), so a raster generated on the device is
 * bit-identical to one generated on the host (tests/test_synth.py checks that).
 *
 * Recipe (SURVEY.md §8d "DEM recipe"):
 *   - lowbias32 lattice hash of (ix, iy, key) -> lattice value in [-16384, 16383];
 *   - exact fixed-point bilinear value noise at lattice spacing 2^s (int64 math);
 *   - macro relief: octaves s = 14..10; a "mountainness" field at s = 13 scales
 *     fine fBm octaves s = 8..2 (so plains are smooth and runs of equal values are
 *     common, as in SRTM — the paper notes values are "mostly < 5000");
 *   - clustered voids: nodata (-32768) where a s = 7 noise field exceeds a threshold.
 */
#ifndef ZH_SYNTH_DEM_CORE_H
#define ZH_SYNTH_DEM_CORE_H
#include <stdint.h>

#if defined(__CUDACC__)
#define ZHS_HD __host__ __device__ __forceinline__
#else
#define ZHS_HD static inline
#endif

#define ZHS_NODATA (-32768)

typedef struct {
  uint32_t seed;
  int32_t base;        /* metres added to the relief                                  */
  int32_t macro_amp;   /* amplitude of the s=14 octave (halved per finer octave)        */
  int32_t fine_amp;    /* amplitude of the s=8 fine octave (halved per finer octave)    */
  int32_t void_thresh; /* lattice-noise threshold for voids, > 16383 disables voids     */
  int32_t lo_clip, hi_clip; /* clamp of the final elevation                              */
} zhs_dem_params;

ZHS_HD uint32_t zhs_lowbias32(uint32_t h) {
  h ^= h >> 16; h *= 0x7feb352du;
  h ^= h >> 15; h *= 0x846ca68bu;
  h ^= h >> 16;
  return h;
}

ZHS_HD int64_t zhs_lattice(uint32_t ix, uint32_t iy, uint32_t key) {
  uint32_t h = zhs_lowbias32(ix * 0x9E3779B1u + iy * 0x85EBCA77u + key * 0xC2B2AE3Du);
  return (int64_t)(h >> 17) - 16384; /* [-16384, 16383] */
}

/* Bilinear value noise, lattice spacing 2^s (s in 1..20), result in [-16384, 16383]. */
ZHS_HD int32_t zhs_vnoise(int64_t r, int64_t c, int s, uint32_t key) {
  const int64_t S = (int64_t)1 << s, m = S - 1;
  const uint32_t ix = (uint32_t)(c >> s), iy = (uint32_t)(r >> s);
  const int64_t fx = c & m, fy = r & m;
  const int64_t a = zhs_lattice(ix, iy, key), b = zhs_lattice(ix + 1u, iy, key);
  const int64_t d = zhs_lattice(ix, iy + 1u, key), e = zhs_lattice(ix + 1u, iy + 1u, key);
  const int64_t top = a * (S - fx) + b * fx;
  const int64_t bot = d * (S - fx) + e * fx;
  const int64_t v = top * (S - fy) + bot * fy; /* |v| < 2^14 * 2^(2s) */
  return (int32_t)(v >> (2 * s));              /* arithmetic shift = floor */
}

/* Elevation of cell (r, c) of the global raster; int16 with ZHS_NODATA voids. */
ZHS_HD int16_t zhs_dem_cell(const zhs_dem_params* p, int64_t r, int64_t c) {
  const uint32_t k = p->seed * 0x27d4eb2fu;
  /* clustered voids */
  if (p->void_thresh <= 16383) {
    if (zhs_vnoise(r, c, 7, k + 101u) > p->void_thresh) return (int16_t)ZHS_NODATA;
  }
  /* macro relief, skewed: positive relief is stretched (mountains), negative compressed */
  int64_t macro = 0;
  int64_t amp = p->macro_amp;
  for (int s = 14; s >= 10; --s) {
    macro += ((int64_t)zhs_vnoise(r, c, s, k + (uint32_t)s) * amp) >> 14;
    amp >>= 1;
  }
  if (macro > 0) macro = macro + (macro * macro) / 2048;
  else macro = macro / 4;
  /* mountainness in [0, 1024) */
  const int64_t mount = ((int64_t)zhs_vnoise(r, c, 13, k + 77u) + 16384) >> 5;
  const int64_t mount2 = (mount * mount) >> 10;
  int64_t fine = 0;
  amp = p->fine_amp;
  for (int s = 8; s >= 2; --s) {
    fine += ((int64_t)zhs_vnoise(r, c, s, k + 50u + (uint32_t)s) * amp) >> 14;
    amp = (amp * 5) >> 3;
  }
  int64_t e = (int64_t)p->base + macro + ((fine * mount2) >> 10);
  if (e < p->lo_clip) e = p->lo_clip;
  if (e > p->hi_clip) e = p->hi_clip;
  return (int16_t)e;
}

/* Alternative closed-form rasters used by the oracle pins (tests/test_oracle_pins.py):
 * kind 1: v = (c mod m) + off ; kind 2: v = (r mod m) + off ; kind 3: v = ((r*cols + c) mod m) + off */
ZHS_HD int16_t zhs_pattern_cell(int kind, int64_t r, int64_t c, int64_t cols, int32_t m, int32_t off) {
  int64_t v;
  if (kind == 1) v = c % m;
  else if (kind == 2) v = r % m;
  else v = (r * cols + c) % m;
  return (int16_t)(v + off);
}

#endif
