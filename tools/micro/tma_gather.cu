// tma_gather.cu - microbenchmark for round-1 VERDICT item 4: do TMA tile::gather4 copies
// (sm_100a: 4 table rows per instruction, landed in shared memory without registers) gather
// random 128-byte factor rows faster than frag3's 256-bit register loads?
//
//   ldg   : a 4-lane group loads one 128-B row as 4 x 32 B (ld.global.nc.L1::no_allocate.v8),
//           K rows in flight per group (frag3's pattern), 256-thread CTAs, 8 per SM
//   g4    : a producer warp per CTA draws 32 rows per stage and 8 of its lanes each issue one
//           cp.async.bulk.tensor.2d ... tile::gather4 into a ring of STAGES x 4 KB (one mbarrier
//           per stage with complete_tx); 3 consumer warps read every landed row from shared
//           memory and release the stage through an "empty" mbarrier
//
// Result on B200 (profiles/r02/micro_tma_gather.txt): LDG 15.5 / 8.0 / 5.3 / 5.4 TB/s for
// 32 MB / 256 MB / 1 GB / 4 GB tables, gather4 at most 5.7 / 5.7 / 5.3 / 4.6 TB/s: never faster;
// 2.7x slower on L2-resident rows (~45 G rows/s: the TMA unit's issue rate), equal at best when
// DRAM-bound.
//
// Rows are drawn by the same hash in both (uniform over the table).  Tables from L2-resident
// (32 MB) to >> L2 (4 GB).  Prints rows/s and the row bytes moved per second.
//
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tma_gather tma_gather.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <cstdio>
#include <cstdlib>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

// ---- ldg: frag3's register gather ----
template <int K>
__global__ void ldg_gather(const float4* __restrict__ tab, uint64_t rows, int iters, float* out) {
  const int lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const uint64_t wid = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  float acc = 0.f;
  for (int it = 0; it < iters; ++it) {
    float4 a[K], b[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint64_t r = mix(wid * 1000003ULL + (uint64_t)(it * K + k) * 8 + g) & (rows - 1);
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

// ---- g4: TMA gather4 into a shared-memory ring ----
constexpr int STAGES = 8, G4_PER_STAGE = 8, ROW_BYTES = 128;
constexpr int STAGE_BYTES = G4_PER_STAGE * 4 * ROW_BYTES;  // 4 KB = 32 rows
constexpr int CONSUMERS = 3;                               // consumer warps

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(n));
}
__device__ __forceinline__ void mbar_expect(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  uint32_t done = 0;
  while (!done)
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                 : "=r"(done) : "r"(su32(b)), "r"(parity) : "memory");
}
__device__ __forceinline__ void gather4(void* dst, const CUtensorMap* tm, int r0, int r1, int r2, int r3, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
      ::"r"(su32(dst)), "l"(tm), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(su32(bar))
      : "memory");
}

__global__ void __launch_bounds__(32 * (1 + CONSUMERS)) g4_gather(const __grid_constant__ CUtensorMap tm, uint64_t rows,
                                                                   int stages_per_cta, float* out) {
  extern __shared__ __align__(128) uint8_t ring[];
  __shared__ uint64_t full[STAGES], empty[STAGES];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], CONSUMERS);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == 0) {
    // the producer warp: 32 lanes draw 32 rows, lanes 0..7 issue one gather4 each
    for (int it = 0; it < stages_per_cta; ++it) {
      const int s = it % STAGES;
      if (it >= STAGES) mbar_wait(&empty[s], ((it / STAGES) - 1) & 1);
      if (lane == 0) mbar_expect(&full[s], STAGE_BYTES);
      __syncwarp();
      const uint64_t base = ((uint64_t)blockIdx.x * stages_per_cta + it) * 32;
      const int r = (int)(mix(base + lane) & (rows - 1));
      const int r0 = __shfl_sync(0xffffffffu, r, 4 * (lane & 7) + 0), r1 = __shfl_sync(0xffffffffu, r, 4 * (lane & 7) + 1),
                r2 = __shfl_sync(0xffffffffu, r, 4 * (lane & 7) + 2), r3 = __shfl_sync(0xffffffffu, r, 4 * (lane & 7) + 3);
      if (lane < G4_PER_STAGE) gather4(ring + s * STAGE_BYTES + lane * 4 * ROW_BYTES, &tm, r0, r1, r2, r3, &full[s]);
    }
  } else {
    float acc = 0.f;
    const int c = warp - 1;
    for (int it = 0; it < stages_per_cta; ++it) {
      const int s = it % STAGES;
      mbar_wait(&full[s], (it / STAGES) & 1);
      const float4* v = reinterpret_cast<const float4*>(ring + s * STAGE_BYTES);
      for (int i = c * 32 + lane; i < STAGE_BYTES / 16; i += CONSUMERS * 32) {
        const float4 x = v[i];
        acc += x.x + x.y + x.z + x.w;
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);
    }
    if (acc == 123.456f) out[0] = acc;
  }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  EncodeFn encode = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&encode, cudaEnableDefault, &q));
  if (!encode) { printf("no cuTensorMapEncodeTiled\n"); return 1; }
  float* out;
  CK(cudaMalloc(&out, 16));
  const uint64_t sizes[] = {32ull << 20, 256ull << 20, 1ull << 30, 4ull << 30};
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  CK(cudaFuncSetAttribute(g4_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, STAGES * STAGE_BYTES));
  for (uint64_t bytes : sizes) {
    const uint64_t rows = bytes / ROW_BYTES;
    float* tab;
    CK(cudaMalloc(&tab, bytes));
    CK(cudaMemset(tab, 0, bytes));
    // ldg, K = 2 and 4 rows in flight per 4-lane group
    const int blocks = 148 * 8, iters = 64;
    for (int K : {2, 4}) {
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(e0);
        if (K == 2) ldg_gather<2><<<blocks, 256>>>((const float4*)tab, rows, iters, out);
        else ldg_gather<4><<<blocks, 256>>>((const float4*)tab, rows, iters, out);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        const double nrows = (double)blocks * 256 / 4 * iters * K;
        if (rep) printf("table %6.0f MB  ldg K=%d      : %8.2f Grows/s  %7.0f GB/s\n", bytes / 1048576.0, K,
                        nrows / ms / 1e6, nrows * 128 / ms / 1e6);
      }
    }
    CUtensorMap tm;
    cuuint64_t gdim[2] = {32, rows}, gstride[1] = {128};
    cuuint32_t box[2] = {32, 1}, estr[2] = {1, 1};
    CUresult r = encode(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, tab, gdim, gstride, box, estr,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
      printf("cuTensorMapEncodeTiled failed: %d\n", (int)r);
      return 1;
    }
    for (int ctas_per_sm : {2, 4, 8}) {
      const int grid = 148 * ctas_per_sm, spc = 256;
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(e0);
        g4_gather<<<grid, 32 * (1 + CONSUMERS), STAGES * STAGE_BYTES>>>(tm, rows, spc, out);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        CK(cudaGetLastError());
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        const double nrows = (double)grid * spc * 32;
        if (rep) printf("table %6.0f MB  g4 %d CTA/SM : %8.2f Grows/s  %7.0f GB/s\n", bytes / 1048576.0, ctas_per_sm,
                        nrows / ms / 1e6, nrows * 128 / ms / 1e6);
      }
    }
    CK(cudaFree(tab));
  }
  return 0;
}
