// Microbenchmark: which on-chip paths can feed random 128-byte factor-row gathers into
// registers on B200 (sm_100a) when the factors are L2-resident (the nell-2 regime, where
// frag3_kernel is bound by the LSU data pipe / writeback: profiles/r01_frag3/).
// One "nonzero" = two 128-B rows (two gathered modes) multiplied and accumulated, 4 lanes
// per nonzero (8 floats per lane), U nonzeros per lane group in flight.  Row sources:
//   G = global, ld.global.nc.L1::no_allocate.v8.f32 (LSU pipe)
//   S = shared memory (two LDS.128 per lane, parity order; 64 KB block)
//   T = texture, tex1Dfetch<float4> x2 per lane (TEX pipe, separate writeback path?)
// Variants: GG, SG (= frag3 today), TG, TS, TT.  Table: 4 MB of rows (L2-resident).
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t mix32(uint32_t z) {
  z ^= z >> 16; z *= 0x7feb352dU; z ^= z >> 15; z *= 0x846ca68bU; z ^= z >> 16;
  return z;
}

struct F8 { float4 a, b; };

__device__ __forceinline__ F8 ldg_row(const float4* tab, uint32_t r, int t) {
  F8 x;
  asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(x.a.x), "=f"(x.a.y), "=f"(x.a.z), "=f"(x.a.w), "=f"(x.b.x), "=f"(x.b.y), "=f"(x.b.z),
                 "=f"(x.b.w)
               : "l"(tab + (size_t)r * 8 + 2 * t));
  return x;
}
__device__ __forceinline__ F8 lds_row(const float4* s, uint32_t r, int t, int par) {
  const float4 x = s[r * 8 + 2 * t + par], y = s[r * 8 + 2 * t + 1 - par];
  F8 o;
  o.a = par ? y : x;
  o.b = par ? x : y;
  return o;
}
__device__ __forceinline__ F8 tex_row(cudaTextureObject_t tx, uint32_t r, int t) {
  F8 o;
  o.a = tex1Dfetch<float4>(tx, (int)(r * 8 + 2 * t));
  o.b = tex1Dfetch<float4>(tx, (int)(r * 8 + 2 * t + 1));
  return o;
}

template <int A, int B, int U>  // sources of row 1 / row 2: 0 = G, 1 = S, 2 = T
__global__ void __launch_bounds__(512) bench(const float4* __restrict__ tab, cudaTextureObject_t tx, uint32_t rows,
                                             int iters, float* out) {
  extern __shared__ float4 sm[];
  const uint32_t srows = 512;  // 64 KB block
  for (uint32_t i = threadIdx.x; i < srows * 8; i += blockDim.x) sm[i] = tab[i];
  __syncthreads();
  const int lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3, par = (lane >> 2) & 1;
  const uint32_t wid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  float4 acc0 = make_float4(0, 0, 0, 0), acc1 = acc0;
  auto fetch = [&](int src, uint32_t h, uint32_t nrows) -> F8 {
    const uint32_t r = h % nrows;
    if (src == 0) return ldg_row(tab, r, t);
    if (src == 1) return lds_row(sm, r % srows, t, par);
    return tex_row(tx, r, t);
  };
  for (int it = 0; it < iters; ++it) {
    F8 x[U], y[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t h = mix32(wid * 7919u + (uint32_t)(it * U + u) * 8u + g);
      x[u] = fetch(A, h, rows);
      y[u] = fetch(B, mix32(h), rows);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      acc0.x += x[u].a.x * y[u].a.x; acc0.y += x[u].a.y * y[u].a.y;
      acc0.z += x[u].a.z * y[u].a.z; acc0.w += x[u].a.w * y[u].a.w;
      acc1.x += x[u].b.x * y[u].b.x; acc1.y += x[u].b.y * y[u].b.y;
      acc1.z += x[u].b.z * y[u].b.z; acc1.w += x[u].b.w * y[u].b.w;
    }
  }
  const float s = acc0.x + acc0.y + acc0.z + acc0.w + acc1.x + acc1.y + acc1.z + acc1.w;
  if (s == 123.456f) out[0] = s;
}

int main() {
  const uint32_t rows = (4u << 20) / 128;  // 4 MB table
  float4* tab;
  cudaMalloc(&tab, (size_t)rows * 128);
  cudaMemset(tab, 0, (size_t)rows * 128);
  float* out;
  cudaMalloc(&out, 64);
  cudaResourceDesc rd{};
  rd.resType = cudaResourceTypeLinear;
  rd.res.linear.devPtr = tab;
  rd.res.linear.desc = cudaCreateChannelDesc<float4>();
  rd.res.linear.sizeInBytes = (size_t)rows * 128;
  cudaTextureDesc td{};
  td.readMode = cudaReadModeElementType;
  cudaTextureObject_t tx = 0;
  cudaCreateTextureObject(&tx, &rd, &td, nullptr);
  int maxw = 0;
  cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxTexture1DLinearWidth, 0);
  printf("max 1D linear texture width: %d texels\n", maxw);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const size_t smem = 512 * 128;
  auto run = [&](const char* name, auto kern) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const int blocks = 148 * 2, threads = 512, iters = 512;
    kern<<<blocks, threads, smem>>>(tab, tx, rows, iters, out);
    cudaEventRecord(e0);
    kern<<<blocks, threads, smem>>>(tab, tx, rows, iters, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double nnz = (double)blocks * threads / 4 * iters * 2;  // U = 2
    printf("%s: %.3f ms  %.2f Gnnz/s  %.2f nnz/clk/SM (at 1.965 GHz)  %s\n", name, ms, nnz / (ms * 1e-3) / 1e9,
           nnz / (ms * 1e-3) / 1.965e9 / 148, cudaGetErrorString(cudaGetLastError()));
  };
  run("GG (global+global)", bench<0, 0, 2>);
  run("SG (smem+global)  ", bench<1, 0, 2>);
  run("TG (tex+global)   ", bench<2, 0, 2>);
  run("TS (tex+smem)     ", bench<2, 1, 2>);
  run("TT (tex+tex)      ", bench<2, 2, 2>);
  run("SS (smem+smem)    ", bench<1, 1, 2>);
  return 0;
}
