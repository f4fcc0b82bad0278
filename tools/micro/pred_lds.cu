// Microbenchmark: what does a shared-memory / L2 row gather cost when only some lane
// groups of the warp take it (fiber reuse keeps a row in registers for the others)?
// And what does the record broadcast cost for 16-B vs 8-B records?
//
//   rows   : every lane group (G lanes, G*32 B = one 128-B fp32 R=32 row at 8 floats per
//            lane for G = 4, 4 floats per lane for G = 8) reads a random row of a
//            256-row block in smem with probability p (per group, per iteration).
//   ldg    : same from a 4 MB global table (L2-resident), 256-bit loads (G = 4).
//   rec16 / rec8 : broadcast loads of a 16-B / 8-B record per 4-lane group.
// Prints ns per warp-iteration and the implied wavefronts/clk at 1.965 GHz.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <algorithm>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

// MODE 0: smem rows, G lanes per group; MODE 1: ldg rows (G = 4); MODE 2: rec16; MODE 3: rec8
template <int MODE, int G>
__global__ void __launch_bounds__(512) k(const float4* __restrict__ gtab, float* out, int iters, uint32_t pthr) {
  __shared__ __align__(16) float4 s[256 * 8 + 64];
  for (int i = threadIdx.x; i < 256 * 8 + 64; i += blockDim.x) s[i] = make_float4(i, i + 1, i + 2, i + 3);
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int group = lane / G, lig = lane % G;
  const uint32_t gid = (blockIdx.x * blockDim.x + threadIdx.x) / G;
  float4 acc = make_float4(0, 0, 0, 0), acc2 = acc;
  uint32_t x = hsh(gid);
  const int par = (lane >> 2) & 1;  // parity issue order (as frag3): conflict-free quarter-warps
  for (int it = 0; it < iters; ++it) {
    x = x * 1664525u + 1013904223u;  // per-group LCG: 1 IMAD (light ALU so the LSU cost shows)
    const uint32_t h = x;
    const bool take = (h & 0xFFFFu) < pthr;
    const uint32_t row = h >> 24;
    if (MODE == 0) {
      if (take) {
        if (G == 4) {
          const float4 u = s[row * 8 + 2 * lig + par], w = s[row * 8 + 2 * lig + 1 - par];
          acc.x += u.x; acc.y += u.y; acc.z += u.z; acc.w += u.w;
          acc2.x += w.x; acc2.y += w.y; acc2.z += w.z; acc2.w += w.w;
        } else {
          const float4 u = s[row * 8 + lig];
          acc.x += u.x; acc.y += u.y; acc.z += u.z; acc.w += u.w;
        }
      }
    } else if (MODE == 1) {
      if (take) {
        const uint32_t grow = (h >> 9) & 32767u;  // 32768 rows x 128 B = 4 MB
        const float4* p = gtab + (size_t)grow * 8 + 2 * lig;
        float4 u, w;
        asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=f"(u.x), "=f"(u.y), "=f"(u.z), "=f"(u.w), "=f"(w.x), "=f"(w.y), "=f"(w.z), "=f"(w.w)
                     : "l"(p));
        acc.x += u.x; acc.y += u.y; acc.z += u.z; acc.w += u.w;
        acc2.x += w.x; acc2.y += w.y; acc2.z += w.z; acc2.w += w.w;
      }
    } else if (MODE == 4) {  // L1-resident 16 KB table, default (L1-allocating) caching
      if (take) {
        const float4* p = gtab + (size_t)(row & 127u) * 8 + 2 * lig;
        float4 u, w;
        asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=f"(u.x), "=f"(u.y), "=f"(u.z), "=f"(u.w), "=f"(w.x), "=f"(w.y), "=f"(w.z), "=f"(w.w)
                     : "l"(p));
        acc.x += u.x; acc.y += u.y; acc.z += u.z; acc.w += u.w;
        acc2.x += w.x; acc2.y += w.y; acc2.z += w.z; acc2.w += w.w;
      }
    } else if (MODE >= 10) {  // L2 row, load variants (p applies)
      if (take) {
        const uint32_t grow = (h >> 9) & 32767u;
        const float4* p = gtab + (size_t)grow * 8 + 2 * lig;
        float4 u, w;
        if (MODE == 10)
          asm volatile("ld.global.cg.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                       : "=f"(u.x), "=f"(u.y), "=f"(u.z), "=f"(u.w), "=f"(w.x), "=f"(w.y), "=f"(w.z), "=f"(w.w) : "l"(p));
        else if (MODE == 11)
          asm volatile("ld.global.nc.L1::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                       : "=f"(u.x), "=f"(u.y), "=f"(u.z), "=f"(u.w), "=f"(w.x), "=f"(w.y), "=f"(w.z), "=f"(w.w) : "l"(p));
        else if (MODE == 12)
          asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                       : "=f"(u.x), "=f"(u.y), "=f"(u.z), "=f"(u.w), "=f"(w.x), "=f"(w.y), "=f"(w.z), "=f"(w.w) : "l"(p));
        else {  // 13: two 128-bit no_allocate loads
          asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                       : "=f"(u.x), "=f"(u.y), "=f"(u.z), "=f"(u.w) : "l"(p));
          asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                       : "=f"(w.x), "=f"(w.y), "=f"(w.z), "=f"(w.w) : "l"(p + 1));
        }
        acc.x += u.x; acc.y += u.y; acc.z += u.z; acc.w += u.w;
        acc2.x += w.x; acc2.y += w.y; acc2.z += w.z; acc2.w += w.w;
      }
    } else if (MODE == 2) {
      const uint32_t r = (it * 8 + group) & 2047u;
      const float4 u = s[r];
      acc.x += u.x; acc.y += u.y; acc.z += u.z; acc.w += u.w;
    } else {
      const uint32_t r = (it * 8 + group) & 4095u;
      const float2 u = reinterpret_cast<const float2*>(s)[r];
      acc.x += u.x; acc.y += u.y;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc.x + acc.y + acc.z + acc.w + acc2.x + acc2.y + acc2.z + acc2.w;
}

int main() {
  float* out;
  float4* gtab;
  cudaMalloc(&out, 148 * 4 * 512 * 4);
  cudaMalloc(&gtab, 32768 * 128 + 4096);
  cudaMemset(gtab, 0, 32768 * 128 + 4096);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 4096;
  const int thr = 512;
  int ctas = 148 * 4;
  auto run = [&](auto kern, const char* name, double p, double wf_per_warp_it) {
    const uint32_t pthr = (uint32_t)(p * 65536.0);
    kern<<<ctas, thr>>>(gtab, out, iters, pthr);
    cudaEventRecord(a);
    kern<<<ctas, thr>>>(gtab, out, iters, pthr);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double warp_its = (double)ctas * (thr / 32) * iters;
    const double clk_per_warp_it_sm = (ms * 1e-3) * 1.965e9 * std::min(148, ctas / 4) / warp_its;
    printf("%-28s p=%.2f  %.3f ms  SM-clk per warp-iteration=%.3f  (full-take wavefronts %.1f)\n", name, p, ms,
           clk_per_warp_it_sm, wf_per_warp_it);
  };
  for (double p : {1.0, 0.75, 0.58, 0.5, 0.25, 0.0}) run(k<0, 4>, "smem row G=4 (2xLDS.128)", p, 8);
  for (double p : {1.0, 0.75, 0.58, 0.5, 0.25, 0.0}) run(k<0, 8>, "smem row G=8 (1xLDS.128)", p, 4);
  for (double p : {1.0, 0.75, 0.58, 0.5, 0.25, 0.0}) run(k<1, 4>, "L2 row G=4 (LDG.256)", p, 8);
  run(k<4, 4>, "L1 row G=4 (LDG.256 L1 hit)", 1.0, 8);
  run(k<1, 4>, "L2 row .nc.L1::no_allocate", 1.0, 8);
  run(k<10, 4>, "L2 row .cg v8", 1.0, 8);
  run(k<11, 4>, "L2 row .nc.L1::evict_first", 1.0, 8);
  run(k<12, 4>, "L2 row .nc (default)", 1.0, 8);
  run(k<13, 4>, "L2 row 2x v4 no_allocate", 1.0, 8);
  ctas = 37 * 4;
  run(k<1, 4>, "L2 row G=4, 37 SMs", 1.0, 8);
  ctas = 74 * 4;
  run(k<1, 4>, "L2 row G=4, 74 SMs", 1.0, 8);
  ctas = 148 * 4;
  run(k<2, 4>, "rec16 bcast LDS.128", 1.0, 0);
  run(k<3, 4>, "rec8 bcast LDS.64", 1.0, 0);
  return 0;
}
