// Microbenchmark: achievable bandwidth of random 128-byte row gathers on B200, as a
// function of rows in flight per warp (MLP) and occupancy.  Table = 4 GiB (>> 126 MB L2),
// rows chosen by a hash (uniform).  Each group of 4 lanes loads one 128-B row with one
// 256-bit load per lane (the frag_kernel pattern); a warp keeps K rows/group in flight.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

template <int K>
__global__ void gather(const float4* __restrict__ tab, uint64_t rows, int iters, float* out) {
  const int lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const uint64_t wid = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  float acc = 0.f;
  for (int it = 0; it < iters; ++it) {
    float4 a[K], b[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint64_t r = mix(wid * 1000003ULL + (uint64_t)(it * K + k) * 8 + g) % rows;
      const float4* p = tab + r * 8 + 2 * t;
      asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                   : "=f"(a[k].x), "=f"(a[k].y), "=f"(a[k].z), "=f"(a[k].w), "=f"(b[k].x), "=f"(b[k].y),
                     "=f"(b[k].z), "=f"(b[k].w)
                   : "l"(p));
    }
#pragma unroll
    for (int k = 0; k < K; ++k) acc += a[k].x + a[k].y + a[k].z + a[k].w + b[k].x + b[k].y + b[k].z + b[k].w;
  }
  if (acc == 123.456f) out[0] = acc;
}

int main() {
  const uint64_t bytes = 4ull << 30, rows = bytes / 128;
  float4* tab;
  cudaMalloc(&tab, bytes);
  cudaMemset(tab, 0, bytes);
  float* out;
  cudaMalloc(&out, 64);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto run = [&](auto kern, int K, int threads, int blocks_per_sm) {
    const int blocks = 148 * blocks_per_sm;
    const int iters = 256 / K;
    kern<<<blocks, threads>>>(tab, rows, iters, out);
    cudaEventRecord(e0);
    kern<<<blocks, threads>>>(tab, rows, iters, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double nrows = (double)blocks * threads / 32 * 8 * iters * K;
    printf("K=%2d threads=%4d blocks/SM=%d warps/SM=%2d : %7.1f GB/s (%.3f ms) %s\n", K, threads, blocks_per_sm,
           threads / 32 * blocks_per_sm, nrows * 128 / (ms * 1e-3) / 1e9, ms, cudaGetErrorString(cudaGetLastError()));
  };
  for (int occ : {1, 2}) {
    run(gather<1>, 1, 512, occ);
    run(gather<2>, 2, 512, occ);
    run(gather<4>, 4, 512, occ);
    run(gather<8>, 8, 512, occ);
  }
  run(gather<2>, 2, 1024, 2);
  run(gather<4>, 4, 1024, 2);
  run(gather<8>, 8, 256, 4);
  return 0;
}
