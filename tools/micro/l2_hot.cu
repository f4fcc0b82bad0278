// l2_hot.cu - microbenchmark: can L2 eviction-priority hints keep the hot rows of Zipf-skewed
// factor gathers resident (nell-1 mode 2: rows gathered from A0 2.9M x 128 B and A1 2.1M x 128 B,
// 143.6 M nonzeros, 16-byte records streamed, Y rows written)?
//
// Variants (per gather, a lane group of 4 lanes loads one 128-B row as 4 x 32 B):
//   0  ld.global.nc.L1::no_allocate                      (frag3 today)
//   1  hot rows: L2::cache_hint evict_last, cold rows: evict_first
//   2  hot rows: evict_last, cold rows: plain (evict_normal)
//   3  hot rows: evict_unchanged... (fraction policy 1.0 evict_last on hot only, cold evict_unchanged)
//   4  hot rows copied into a dense block (records point into it), plain loads
//   5  every row renumbered by frequency (no scatter)
//   6  dense hot block + evict_last on hot rows, evict_first on cold rows
//   7  dense hot block + evict_last on hot rows, plain cold rows
// hot = Zipf rank below k_A / k_B with k chosen so the hot rows of both factors take H bytes and
// have equal expected counts at the cut (the optimal static cache for independent references).
//
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o l2_hot l2_hot.cu
// run:   ./l2_hot [nnz] [IA] [IB] [s]
#include <cuda_runtime.h>
#include <stdint.h>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
// inverse CDF of the bucket-free power law F(x) = ((x+1)^(1-s) - 1) / ((I+1)^(1-s) - 1)
__device__ __forceinline__ uint32_t zipf_rank(uint64_t h, uint32_t I, double s) {
  const double u = (double)(h >> 11) * (1.0 / 9007199254740992.0);
  const double a = 1.0 - s;
  const double x = pow(1.0 + u * (pow((double)I + 1.0, a) - 1.0), 1.0 / a) - 1.0;
  uint32_t r = (uint32_t)x;
  return r >= I ? I - 1 : r;
}
// scatter ranks over the rows: r * P mod I (P prime, not dividing I)
__device__ __forceinline__ uint32_t scatter(uint32_t r, uint32_t I) { return (uint32_t)(((uint64_t)r * 2654435761ull) % I); }

// record = [row_of_Y, gA | hot<<31, gB | hot<<31, v]
__global__ void gen(uint4* rec, uint64_t nnz, uint32_t IA, uint32_t IB, double s, uint32_t kA, uint32_t kB, int compact) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < nnz; e += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t ra = zipf_rank(mix(e * 2 + 1), IA, s), rb = zipf_rank(mix(e * 2 + 2 + (1ull << 40)), IB, s);
    uint4 r;
    r.x = (uint32_t)(e / 6);  // runs of ~6 like nell-1 mode 2
    // compact: hot rows index the dense hot copy (rank order), cold rows the scattered table
    // compact == 2: every row renumbered by frequency rank (no scatter at all) in the main table
    r.y = compact == 2 ? ra : (compact && ra < kA) ? (ra | 0x80000000u) : (scatter(ra, IA) | (ra < kA ? 0x80000000u : 0u));
    r.z = compact == 2 ? rb : (compact && rb < kB) ? (rb | 0x80000000u) : (scatter(rb, IB) | (rb < kB ? 0x80000000u : 0u));
    r.w = __float_as_uint(1.0f);
    rec[e] = r;
  }
}

__device__ __forceinline__ void ld_na(const float* p, float4& a, float4& b) {
  asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w), "=f"(b.x), "=f"(b.y), "=f"(b.z), "=f"(b.w) : "l"(p));
}
__device__ __forceinline__ void ld_pol(const float* p, float4& a, float4& b, uint64_t pol) {
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
               : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w), "=f"(b.x), "=f"(b.y), "=f"(b.z), "=f"(b.w)
               : "l"(p), "l"(pol));
}

template <int V>
__global__ void __launch_bounds__(512) gather(const uint4* __restrict__ rec, uint64_t nnz, const float* __restrict__ A,
                                              const float* __restrict__ B, float* __restrict__ Y,
                                              const float* __restrict__ HA, const float* __restrict__ HB) {
  uint64_t p_last, p_first, p_unch;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p_last));
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p_first));
  asm volatile("createpolicy.fractional.L2::evict_unchanged.b64 %0, 1.0;" : "=l"(p_unch));
  const int lig = threadIdx.x & 3;
  const uint64_t g = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 2;
  const uint64_t G = ((uint64_t)gridDim.x * blockDim.x) >> 2;
  // each group walks a contiguous range (like a frag3 sub-range)
  const uint64_t e0 = g * nnz / G, e1 = (g + 1) * nnz / G;
  float4 acc0 = make_float4(0, 0, 0, 0), acc1 = acc0;
  uint32_t cur = 0xFFFFFFFFu;
  auto load = [&](const float* base, const float* hbase, uint32_t idx, float4& a, float4& b) {
    const bool hot = idx >> 31;
    const float* p = ((V == 4 || V >= 6) && hot ? hbase : base) + (size_t)(idx & 0x7FFFFFFFu) * 32 + 8 * lig;
    if (V == 0 || V == 4) ld_na(p, a, b);
    else if (V == 6) { if (hot) ld_pol(p, a, b, p_last); else ld_pol(p, a, b, p_first); }
    else if (V == 7) { if (hot) ld_pol(p, a, b, p_last); else ld_na(p, a, b); }
    else if (V == 1) { if (hot) ld_pol(p, a, b, p_last); else ld_pol(p, a, b, p_first); }
    else if (V == 2) { if (hot) ld_pol(p, a, b, p_last); else ld_na(p, a, b); }
    else { if (hot) ld_pol(p, a, b, p_last); else ld_pol(p, a, b, p_unch); }
  };
  for (uint64_t e = e0; e < e1; e += 2) {
    uint4 r[2];
    float4 a[2][2], b[2][2];
#pragma unroll
    for (int u = 0; u < 2; ++u) r[u] = (e + u < e1) ? __ldg(rec + e + u) : make_uint4(cur, 0, 0, 0);
#pragma unroll
    for (int u = 0; u < 2; ++u) { load(A, HA, r[u].y, a[u][0], a[u][1]); load(B, HB, r[u].z, b[u][0], b[u][1]); }
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      if (r[u].x != cur) {
        if (cur != 0xFFFFFFFFu) {
          float4* y = reinterpret_cast<float4*>(Y + (size_t)cur * 32 + 8 * lig);
          y[0] = acc0; y[1] = acc1;
        }
        cur = r[u].x; acc0 = make_float4(0, 0, 0, 0); acc1 = acc0;
      }
      const float v = __uint_as_float(r[u].w);
      acc0.x += v * a[u][0].x * b[u][0].x; acc0.y += v * a[u][0].y * b[u][0].y;
      acc0.z += v * a[u][0].z * b[u][0].z; acc0.w += v * a[u][0].w * b[u][0].w;
      acc1.x += v * a[u][1].x * b[u][1].x; acc1.y += v * a[u][1].y * b[u][1].y;
      acc1.z += v * a[u][1].z * b[u][1].z; acc1.w += v * a[u][1].w * b[u][1].w;
    }
  }
  if (cur != 0xFFFFFFFFu) {
    float4* y = reinterpret_cast<float4*>(Y + (size_t)cur * 32 + 8 * lig);
    y[0] = acc0; y[1] = acc1;
  }
}

int main(int argc, char** argv) {
  const uint64_t nnz = argc > 1 ? strtoull(argv[1], 0, 10) : 143599552ull;
  const uint32_t IA = argc > 2 ? atoi(argv[2]) : 2902330, IB = argc > 3 ? atoi(argv[3]) : 2143368;
  const double s = argc > 4 ? atof(argv[4]) : 0.8;
  uint4* rec;
  float *A, *B, *Y;
  CK(cudaMalloc(&rec, nnz * 16));
  CK(cudaMalloc(&A, (size_t)IA * 128));
  CK(cudaMalloc(&B, (size_t)IB * 128));
  CK(cudaMalloc(&Y, (nnz / 6 + 2) * 128));
  CK(cudaMemset(A, 0, (size_t)IA * 128));
  CK(cudaMemset(B, 0, (size_t)IB * 128));
  float *HA, *HB;  // dense hot copies (up to 128 MB of rows each)
  CK(cudaMalloc(&HA, (size_t)1 << 27));
  CK(cudaMalloc(&HB, (size_t)1 << 27));
  CK(cudaMemset(HA, 0, (size_t)1 << 27));
  CK(cudaMemset(HB, 0, (size_t)1 << 27));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  cudaEvent_t t0, t1;
  CK(cudaEventCreate(&t0));
  CK(cudaEventCreate(&t1));
  // expected count of rank x: nnz * a (x+1)^-s / ((I+1)^a - 1); equal-count cut: kB+1 = (kA+1) * (cB/cA)^(1/s)
  const double a = 1.0 - s, cA = 1.0 / (pow(IA + 1.0, a) - 1.0), cB = 1.0 / (pow(IB + 1.0, a) - 1.0);
  const double ratio = pow(cB / cA, 1.0 / s);
  for (double HMB : {0.0, 32.0, 64.0, 96.0, 128.0}) {
    const double rows = HMB * 1048576.0 / 128.0;
    const uint32_t kA = (uint32_t)(rows / (1.0 + ratio)), kB = (uint32_t)(rows - kA);
    for (int V = 0; V < 8; ++V) {
      if (HMB == 0.0 && V > 0 && V != 5) continue;
      if (HMB > 0.0 && V == 5) continue;
      if (V == 0 || V == 4 || V == 5) {  // V 6, 7 reuse V 4's dense-hot records
        gen<<<sms * 8, 256>>>(rec, nnz, IA, IB, s, kA, kB, V == 4 ? 1 : (V == 5 ? 2 : 0));
        CK(cudaDeviceSynchronize());
      }
      auto run = [&]() {
        switch (V) {
          case 0: gather<0><<<sms * 2, 512>>>(rec, nnz, A, B, Y, HA, HB); break;
          case 1: gather<1><<<sms * 2, 512>>>(rec, nnz, A, B, Y, HA, HB); break;
          case 2: gather<2><<<sms * 2, 512>>>(rec, nnz, A, B, Y, HA, HB); break;
          case 3: gather<3><<<sms * 2, 512>>>(rec, nnz, A, B, Y, HA, HB); break;
          case 4: gather<4><<<sms * 2, 512>>>(rec, nnz, A, B, Y, HA, HB); break;
          case 6: gather<6><<<sms * 2, 512>>>(rec, nnz, A, B, Y, HA, HB); break;
          case 7: gather<7><<<sms * 2, 512>>>(rec, nnz, A, B, Y, HA, HB); break;
          default: gather<0><<<sms * 2, 512>>>(rec, nnz, A, B, Y, HA, HB); break;
        }
      };
      run(); run();
      CK(cudaEventRecord(t0));
      for (int it = 0; it < 5; ++it) run();
      CK(cudaEventRecord(t1));
      CK(cudaEventSynchronize(t1));
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, t0, t1));
      ms /= 5;
      printf("{\"hot_MB\": %.0f, \"kA\": %u, \"kB\": %u, \"variant\": %d, \"ms\": %.3f, \"gathers_GBs\": %.0f}\n", HMB, kA,
             kB, V, ms, nnz * 256.0 / (ms * 1e-3) / 1e9);
    }
  }
  return 0;
}
