// Read-only bandwidth of the TILE access pattern of the pure-tile kernel: the CONUS raster
// (93,600 x 216,000 int16, row pitch 432,000 B), 256 x 256 tiles, one 512-thread CTA per run of
// consecutive tiles of a tile row, 16-byte loads, ROWS rows in flight per thread, XOR only (no
// histogram) — the ceiling of k_fused_pure's memory stream, against the linear read of read_bw.cu.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 tile_read_bw.cu -o tile_read_bw && ./tile_read_bw
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint4 ld_stream16(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

constexpr int T = 256;
template <int ROWS>
__global__ void __launch_bounds__(512, 3) k_tiles(const int16_t* __restrict__ a, int64_t pitch, int TC, int ntiles,
                                                 int run, uint32_t* __restrict__ out) {
  uint32_t acc = 0;
  const int nk = T / 8, rpi = 512 / nk;  // 32 vectors per row, 16 rows per pass
  const int kk = threadIdx.x % nk, rs = threadIdx.x / nk;
  for (int j = 0; j < run; ++j) {
    const int tile = blockIdx.x * run + j;
    if (tile >= ntiles) break;
    const int tr = tile / TC, tc = tile - tr * TC;
    const int16_t* p = a + ((int64_t)tr * T + rs) * pitch + (int64_t)tc * T + kk * 8;
    const int64_t step = (int64_t)rpi * pitch;
    for (int r = rs; r < T; r += ROWS * rpi, p += ROWS * step) {
      uint4 q[ROWS];
#pragma unroll
      for (int u = 0; u < ROWS; ++u) q[u] = ld_stream16(p + u * step);
#pragma unroll
      for (int u = 0; u < ROWS; ++u) acc ^= q[u].x ^ q[u].y ^ q[u].z ^ q[u].w;
    }
  }
  if (acc == 0x12345678u) out[0] = acc;
}

__device__ __forceinline__ void ld_stream32(const void* p, uint4& lo, uint4& hi) {
  asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(lo.x), "=r"(lo.y), "=r"(lo.z), "=r"(lo.w), "=r"(hi.x), "=r"(hi.y), "=r"(hi.z), "=r"(hi.w)
               : "l"(p));
}

// the same with one 32-byte load per thread and row (16-cell segments: 16 per row, 32 rows per pass)
template <int ROWS>
__global__ void __launch_bounds__(512, 3) k_tiles32(const int16_t* __restrict__ a, int64_t pitch, int TC, int ntiles,
                                                   int run, uint32_t* __restrict__ out) {
  uint32_t acc = 0;
  const int nk = T / 16, rpi = 512 / nk;
  const int kk = threadIdx.x % nk, rs = threadIdx.x / nk;
  for (int j = 0; j < run; ++j) {
    const int tile = blockIdx.x * run + j;
    if (tile >= ntiles) break;
    const int tr = tile / TC, tc = tile - tr * TC;
    const int16_t* p = a + ((int64_t)tr * T + rs) * pitch + (int64_t)tc * T + kk * 16;
    const int64_t step = (int64_t)rpi * pitch;
    for (int r = rs; r < T; r += ROWS * rpi, p += ROWS * step) {
      uint4 q[ROWS], h[ROWS];
#pragma unroll
      for (int u = 0; u < ROWS; ++u) ld_stream32(p + u * step, q[u], h[u]);
#pragma unroll
      for (int u = 0; u < ROWS; ++u) acc ^= q[u].x ^ q[u].y ^ q[u].z ^ q[u].w ^ h[u].x ^ h[u].y ^ h[u].z ^ h[u].w;
    }
  }
  if (acc == 0x12345678u) out[0] = acc;
}

int main() {
  const int64_t rows = 93600, cols = 216000, pitch = cols;
  const size_t bytes = (size_t)rows * pitch * 2;
  int16_t* a;
  uint32_t* out;
  cudaMalloc(&a, bytes);
  cudaMalloc(&out, 4);
  cudaMemset(a, 1, bytes);
  const int TC = (int)(cols / T), TR = (int)(rows / T);
  const int ntiles = TC * TR;
  const double tb = (double)ntiles * T * T * 2;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int run : {1, 8}) {
    for (int rows_in_flight : {2, 4, 8}) {
      float best = 1e30f;
      const int grid = (ntiles + run - 1) / run;
      for (int rep = 0; rep < 5; ++rep) {
        cudaEventRecord(e0);
        if (rows_in_flight == 2) k_tiles<2><<<grid, 512>>>(a, pitch, TC, ntiles, run, out);
        else if (rows_in_flight == 4) k_tiles<4><<<grid, 512>>>(a, pitch, TC, ntiles, run, out);
        else k_tiles<8><<<grid, 512>>>(a, pitch, TC, ntiles, run, out);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
      }
      printf("tiles %dx%d run %d rows_in_flight %d: %.3f ms for %.2f GB = %.1f GB/s\n", T, T, run, rows_in_flight,
             best, tb / 1e9, tb / best / 1e6);
    }
  }
  for (int run : {1, 8}) {
    for (int rows_in_flight : {2, 4}) {
      float best = 1e30f;
      const int grid = (ntiles + run - 1) / run;
      for (int rep = 0; rep < 5; ++rep) {
        cudaEventRecord(e0);
        if (rows_in_flight == 2) k_tiles32<2><<<grid, 512>>>(a, pitch, TC, ntiles, run, out);
        else k_tiles32<4><<<grid, 512>>>(a, pitch, TC, ntiles, run, out);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
      }
      printf("tiles %dx%d 32-byte loads run %d rows_in_flight %d: %.3f ms for %.2f GB = %.1f GB/s\n", T, T, run,
             rows_in_flight, best, tb / 1e9, tb / best / 1e6);
    }
  }
  return 0;
}
