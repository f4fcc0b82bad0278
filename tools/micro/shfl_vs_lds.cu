// Microbenchmark: does SHFL share the L1TEX/shared-memory data path with LDS on sm_100a?
// Each thread issues ITERS conflict-free LDS.128; variant 1 adds K SHFLs per LDS.
#include <cstdio>
#include <cuda_runtime.h>

template <int K>
__global__ void k(float* out, int iters) {
  __shared__ __align__(16) float s[8192];
  for (int i = threadIdx.x; i < 8192; i += blockDim.x) s[i] = i * 0.5f;
  __syncthreads();
  float4 acc = make_float4(0, 0, 0, 0);
  float x = threadIdx.x;
  int base = (threadIdx.x * 4) & 8191;
  for (int it = 0; it < iters; ++it) {
    float4 v = *reinterpret_cast<float4*>(&s[(base + it * 128) & 8188]);
    acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
#pragma unroll
    for (int q = 0; q < K; ++q) x += __shfl_sync(0xffffffff, x, (threadIdx.x + q + it) & 31);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc.x + acc.y + acc.z + acc.w + x;
}

int main() {
  float* out;
  cudaMalloc(&out, 148 * 8 * 1024 * 4);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 20000;
  auto run = [&](auto kern, const char* name, int nshfl) {
    kern<<<148 * 2, 1024>>>(out, iters);
    cudaEventRecord(a);
    kern<<<148 * 2, 1024>>>(out, iters);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    double lds_wf = 148.0 * 2 * 32 * iters * 4;  // 4 wavefronts per warp LDS.128
    printf("%s: %.3f ms  LDS wavefronts/clk/SM(@1.965GHz)=%.3f  shfl/LDS=%d\n", name, ms,
           lds_wf / (ms * 1e-3) / 148 / 1.965e9, nshfl);
  };
  run(k<0>, "LDS only   ", 0);
  run(k<1>, "LDS+1 SHFL ", 1);
  run(k<2>, "LDS+2 SHFL ", 2);
  run(k<4>, "LDS+4 SHFL ", 4);
  return 0;
}
