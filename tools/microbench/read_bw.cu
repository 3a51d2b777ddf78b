// Read-only HBM bandwidth on B200: how fast can a kernel stream bytes it only reads (the pure-tile
// kernel's situation), against the copy peak of MEASURED_PEAKS.json (read + write).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 read_bw.cu -o read_bw && ./read_bw
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint4 ld_stream16(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

template <int U>
__global__ void __launch_bounds__(512) k_read(const uint4* __restrict__ a, size_t n, uint32_t* __restrict__ out) {
  uint32_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    uint4 q[U];
#pragma unroll
    for (int u = 0; u < U; ++u) q[u] = ld_stream16(a + i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= q[u].x ^ q[u].y ^ q[u].z ^ q[u].w;
  }
  for (; i < n; i += stride) {
    const uint4 q = ld_stream16(a + i);
    acc ^= q.x ^ q.y ^ q.z ^ q.w;
  }
  if (acc == 0x12345678u) out[0] = acc;
}

int main() {
  const size_t bytes = 40ull << 30;
  const size_t n = bytes / 16;
  uint4* a;
  uint32_t* out;
  cudaMalloc(&a, bytes);
  cudaMalloc(&out, 4);
  cudaMemset(a, 1, bytes);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int blocks_per_sm : {2, 3, 4}) {
    for (int u : {2, 4, 8}) {
      const int grid = 148 * blocks_per_sm;
      float best = 1e30f;
      for (int rep = 0; rep < 5; ++rep) {
        cudaEventRecord(e0);
        if (u == 2) k_read<2><<<grid, 512>>>(a, n, out);
        if (u == 4) k_read<4><<<grid, 512>>>(a, n, out);
        if (u == 8) k_read<8><<<grid, 512>>>(a, n, out);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 0 && ms < best) best = ms;
      }
      printf("read-only: %d CTAs/SM x 512 thr, %d x 16 B in flight per thread: %.3f ms, %.1f GB/s\n", blocks_per_sm, u,
             best, bytes / (best * 1e-3) / 1e9);
    }
  }
  return 0;
}
