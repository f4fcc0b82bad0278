// sf_mttkrp.cu - the MTTKRP kernels (§8(a) A5-A7, A8 (ii)).
//
// Computes mode-n MTTKRP, PAPER.md L124-127 (Eq. (4)), elementwise
//   Y(i_n(e), :) += v_e * prod_{m != n} A_m(i_m(e), :)
// No tensor cores: this is a bandwidth-bound gather/scatter, not a dense
// contraction.
//
// Lane mapping (both kernels): a "lane group" of LPN = R/4 lanes owns one
// nonzero at a time; lane `sub` of the group owns rank slice [4*sub, 4*sub+4)
// as one float4, so every factor-row gather is one 128-bit access per lane and a
// whole row (R*4 bytes) is one contiguous request per group.
//
// coo_kernel  (SF_KERNEL_COO): raw input order, one vector atomic
//   (red.global.add.v4.f32) per nonzero per group.  Baseline + streamed path.
// frag_kernel (SF_KERNEL_FRAG): persistent CTAs walk chunks of the planned order
//   (tile, i_n, i_s).  Each chunk's N+1 SoA fields are staged into shared memory by
//   1-D TMA bulk copies (cp.async.bulk + mbarrier, double buffered).  Factors of
//   "staged" modes are copied block-wise into shared memory once per tile (the
//   paper's "times_mat in shared memory") and gathered from there;
//   other modes are gathered from global memory (L2).  Each lane group walks a
//   contiguous stretch of the chunk, accumulating in registers while i_n is
//   unchanged (segmented reduction over sorted runs) and flushing one vector
//   atomic per run edge -- global atomics fire only at run / fragment boundaries
//   (north_star; "requirement for atomic operations").
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>

#include "sf_internal.h"

namespace sf {

// ---------------------------------------------------------------------------
// PTX helpers
// ---------------------------------------------------------------------------
__device__ __forceinline__ void red_add_v4(float* addr, const float4& v) {
  asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(addr), "f"(v.x), "f"(v.y),
               "f"(v.z), "f"(v.w)
               : "memory");
}

__device__ __forceinline__ float4 ldg_f4(const float* p) {
  return __ldg(reinterpret_cast<const float4*>(p));
}

__device__ __forceinline__ float4 lds_f4(const float* p) {
  return *reinterpret_cast<const float4*>(p);
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  const uint32_t a = smem_u32(bar);
  do {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  } while (!done);
}

__device__ __forceinline__ float4 f4mul(const float4& a, const float4& b) {
  return make_float4(a.x * b.x, a.y * b.y, a.z * b.z, a.w * b.w);
}

// ---------------------------------------------------------------------------
// Index validation (A1): flag = 1 if any inds[m][e] >= dims[m].
// ---------------------------------------------------------------------------
struct ValidateParams {
  const uint32_t* ind[SF_MAX_MODES];
  uint64_t dims[SF_MAX_MODES];
  int nmodes;
  uint64_t nnz;
};

__global__ void validate_kernel(ValidateParams p, int* flag) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  int bad = 0;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < p.nnz; e += stride)
    for (int m = 0; m < p.nmodes; ++m) bad |= ((uint64_t)p.ind[m][e] >= p.dims[m]);
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicOr(flag, 1);
}

void validate_indices(int nmodes, const uint64_t* dims, uint64_t nnz, uint32_t* const* inds,
                      int* d_flag, cudaStream_t s) {
  if (nnz == 0) return;
  ValidateParams p{};
  for (int m = 0; m < nmodes; ++m) { p.ind[m] = inds[m]; p.dims[m] = dims[m]; }
  p.nmodes = nmodes;
  p.nnz = nnz;
  int blocks = (int)std::min<uint64_t>((nnz + 255) / 256, 148 * 8);
  validate_kernel<<<blocks, 256, 0, s>>>(p, d_flag);
  count_launch();
  SF_CUDA(cudaGetLastError());
}

// ---------------------------------------------------------------------------
// COO kernel (nnz-parallel, raw order)
// ---------------------------------------------------------------------------
struct CooParams {
  const uint32_t* ind[SF_MAX_MODES];
  const float* val;
  const float* fac[SF_MAX_MODES];
  float* out;
  uint64_t nnz;
  int nmodes, mode, rank;
};

template <int R>
__global__ void __launch_bounds__(256) coo_kernel(CooParams p) {
  constexpr int LPN = R / 4;
  const int sub = threadIdx.x % LPN;
  const uint64_t group = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) / LPN;
  const uint64_t ngroups = ((uint64_t)gridDim.x * blockDim.x) / LPN;
  for (uint64_t e = group; e < p.nnz; e += ngroups) {
    const float v = __ldg(p.val + e);
    float4 acc = make_float4(v, v, v, v);
#pragma unroll
    for (int m = 0; m < SF_MAX_MODES; ++m) {
      if (m >= p.nmodes) break;
      if (m == p.mode) continue;
      const uint32_t im = __ldg(p.ind[m] + e);
      acc = f4mul(acc, ldg_f4(p.fac[m] + (size_t)im * R + 4 * sub));
    }
    const uint32_t in = __ldg(p.ind[p.mode] + e);
    red_add_v4(p.out + (size_t)in * R + 4 * sub, acc);
  }
}

// Any rank: one thread per (nonzero, rank column), scalar atomics.
__global__ void coo_generic_kernel(CooParams p) {
  const uint64_t total = p.nnz * (uint64_t)p.rank;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
    const uint64_t e = t / p.rank;
    const int r = (int)(t - e * p.rank);
    float acc = __ldg(p.val + e);
    for (int m = 0; m < p.nmodes; ++m) {
      if (m == p.mode) continue;
      acc *= __ldg(p.fac[m] + (size_t)__ldg(p.ind[m] + e) * p.rank + r);
    }
    atomicAdd(p.out + (size_t)__ldg(p.ind[p.mode] + e) * p.rank + r, acc);
  }
}

void launch_coo(int nmodes, const uint64_t* dims, uint64_t nnz, const uint32_t* const* inds,
                const float* vals, const float* const* factors, int rank, int mode, float* out,
                cudaStream_t s) {
  (void)dims;
  if (nnz == 0) return;
  CooParams p{};
  for (int m = 0; m < nmodes; ++m) { p.ind[m] = inds[m]; p.fac[m] = factors[m]; }
  p.val = vals;
  p.out = out;
  p.nnz = nnz;
  p.nmodes = nmodes;
  p.mode = mode;
  p.rank = rank;
  const int threads = 256;
  auto grid_for = [&](uint64_t work_items) {
    return (int)std::max<uint64_t>(1, std::min<uint64_t>((work_items + threads - 1) / threads,
                                                         (uint64_t)148 * 16));
  };
  switch (rank) {
    case 16: coo_kernel<16><<<grid_for(nnz * 4), threads, 0, s>>>(p); break;
    case 32: coo_kernel<32><<<grid_for(nnz * 8), threads, 0, s>>>(p); break;
    case 64: coo_kernel<64><<<grid_for(nnz * 16), threads, 0, s>>>(p); break;
    default: coo_generic_kernel<<<grid_for(nnz * rank), threads, 0, s>>>(p); break;
  }
  count_launch();
  SF_CUDA(cudaGetLastError());
}

// ---------------------------------------------------------------------------
// Fragment kernel
// ---------------------------------------------------------------------------
struct FragParams {
  const uint32_t* ind[SF_MAX_MODES];  // kernel-order indices, every mode
  const float* val;
  const float* fac[SF_MAX_MODES];
  float* out;
  const uint32_t* chunk_begin;  // num_chunks + 1
  const uint64_t* chunk_tile;   // num_chunks
  uint32_t num_chunks;
  uint32_t nnz;
  int mode;
  uint32_t staged_mask;
  uint32_t block_rows[SF_MAX_MODES];
  uint32_t ntiles[SF_MAX_MODES];   // ceil(I_m / block_rows[m]) for staged modes
  uint32_t dims[SF_MAX_MODES];
  uint32_t fac_off[SF_MAX_MODES];  // float offset of the staged block of mode m in smem
  uint32_t stage_words;            // words per field per pipeline stage
};

constexpr int kStages = 2;

template <int N, int R>
__global__ void __launch_bounds__(1024) frag_kernel(FragParams p) {
  constexpr int LPN = R / 4;  // lanes per nonzero
  extern __shared__ __align__(128) unsigned char smem_raw[];
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw);  // [kStages] stream + [1] factors
  float* stage_base = reinterpret_cast<float*>(smem_raw + 128);
  float* fac_smem = stage_base + (size_t)kStages * (N + 1) * p.stage_words;

  const int tid = threadIdx.x;
  const int sub = tid % LPN;
  const int group = tid / LPN;
  const int ngroups = blockDim.x / LPN;

  // This CTA's chunk range: chunks whose begin lies in [c*nnz/G, (c+1)*nnz/G).
  const uint64_t G = gridDim.x;
  auto lower = [&](uint64_t target) {
    uint32_t lo = 0, hi = p.num_chunks;
    while (lo < hi) {
      uint32_t mid = (lo + hi) >> 1;
      if ((uint64_t)p.chunk_begin[mid] < target) lo = mid + 1; else hi = mid;
    }
    return lo;
  };
  const uint32_t j0 = lower(((uint64_t)blockIdx.x * p.nnz) / G);
  const uint32_t j1 = lower(((uint64_t)(blockIdx.x + 1) * p.nnz) / G);
  if (j0 >= j1) return;

  if (tid == 0) {
    for (int s = 0; s <= kStages; ++s) mbar_init(&bars[s], 1);
    fence_barrier_init();
  }
  __syncthreads();

  // Producer: issue the N+1 bulk copies of chunk j into stage s (aligned superset).
  auto issue = [&](uint32_t j, int s) {
    const uint32_t b = p.chunk_begin[j], e = p.chunk_begin[j + 1];
    const uint32_t start = b & ~3u;
    const uint32_t bytes = (((e - start) + 3u) & ~3u) * 4u;
    float* dst = stage_base + (size_t)s * (N + 1) * p.stage_words;
    mbar_expect_tx(&bars[s], bytes * (N + 1));
#pragma unroll
    for (int m = 0; m < N; ++m) bulk_g2s(dst + (size_t)m * p.stage_words, p.ind[m] + start, bytes, &bars[s]);
    bulk_g2s(dst + (size_t)N * p.stage_words, p.val + start, bytes, &bars[s]);
  };

  if (tid == 0) {
    for (int s = 0; s < kStages && j0 + s < j1; ++s) issue(j0 + s, s);
  }

  uint64_t cur_tile = ~0ull;
  uint32_t base[N];
#pragma unroll
  for (int m = 0; m < N; ++m) base[m] = 0;
  uint32_t fac_phase = 0;

  for (uint32_t j = j0; j < j1; ++j) {
    const int s = (int)((j - j0) % kStages);
    const uint32_t parity = ((j - j0) / kStages) & 1u;

    // (Re)stage factor blocks when the tile changes.
    if (p.staged_mask) {
      const uint64_t tile = p.chunk_tile[j];
      if (tile != cur_tile) {
        cur_tile = tile;
        uint64_t t = tile;
#pragma unroll
        for (int m = N - 1; m >= 0; --m) {
          if (p.staged_mask & (1u << m)) {
            const uint32_t q = (uint32_t)(t % p.ntiles[m]);
            t /= p.ntiles[m];
            base[m] = q * p.block_rows[m];
          }
        }
        __syncthreads();  // everyone is done with the previous block
        if (tid == 0) {
          uint32_t total = 0;
#pragma unroll
          for (int m = 0; m < N; ++m)
            if (p.staged_mask & (1u << m)) {
              const uint32_t rows = min(p.block_rows[m], p.dims[m] - base[m]);
              total += rows * R * 4u;
            }
          mbar_expect_tx(&bars[kStages], total);
#pragma unroll
          for (int m = 0; m < N; ++m)
            if (p.staged_mask & (1u << m)) {
              const uint32_t rows = min(p.block_rows[m], p.dims[m] - base[m]);
              bulk_g2s(fac_smem + p.fac_off[m], p.fac[m] + (size_t)base[m] * R, rows * R * 4u,
                       &bars[kStages]);
            }
        }
        mbar_wait(&bars[kStages], fac_phase);
        fac_phase ^= 1u;
      }
    }

    mbar_wait(&bars[s], parity);

    const uint32_t b = p.chunk_begin[j], e = p.chunk_begin[j + 1];
    const uint32_t off = b - (b & ~3u);
    const uint32_t n = e - b;
    const float* sb = stage_base + (size_t)s * (N + 1) * p.stage_words + off;
    // stretch length per group, bumped so the groups of one warp hit distinct banks
    uint32_t L = (n + ngroups - 1) / ngroups;
    // (the 32/LPN groups of a warp read word g*L + k: distinct banks iff gcd(L,32) <= LPN)
    if (LPN < 32)
      while (L % (2u * LPN) == 0u) ++L;
    const uint32_t k0 = group * L;
    const uint32_t k1 = min(n, k0 + L);
    if (k0 < k1) {
      const uint32_t* sI = reinterpret_cast<const uint32_t*>(sb);
      const float* sV = sb + (size_t)N * p.stage_words;
      uint32_t cur = sI[(size_t)p.mode * p.stage_words + k0];
      float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
      for (uint32_t k = k0; k < k1; ++k) {
        const float v = sV[k];
        float4 prod = make_float4(v, v, v, v);
#pragma unroll
        for (int m = 0; m < N; ++m) {
          if (m == p.mode) continue;
          const uint32_t im = sI[(size_t)m * p.stage_words + k];
          float4 a;
          if (p.staged_mask & (1u << m))
            a = lds_f4(fac_smem + p.fac_off[m] + (im - base[m]) * R + 4 * sub);
          else
            a = ldg_f4(p.fac[m] + (size_t)im * R + 4 * sub);
          prod = f4mul(prod, a);
        }
        const uint32_t i = sI[(size_t)p.mode * p.stage_words + k];
        if (i != cur) {
          red_add_v4(p.out + (size_t)cur * R + 4 * sub, acc);
          acc = make_float4(0.f, 0.f, 0.f, 0.f);
          cur = i;
        }
        acc.x += prod.x;
        acc.y += prod.y;
        acc.z += prod.z;
        acc.w += prod.w;
      }
      red_add_v4(p.out + (size_t)cur * R + 4 * sub, acc);
    }
    __syncthreads();  // stage s fully consumed
    if (tid == 0 && j + kStages < j1) issue(j + kStages, s);
  }
}

template <int N, int R>
static void frag_launch_t(const FragParams& fp, int grid, int threads, size_t smem, cudaStream_t s) {
  auto k = frag_kernel<N, R>;
  SF_CUDA(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  k<<<grid, threads, smem, s>>>(fp);
}

template <int N, int R>
static int frag_occ_t(int threads, size_t smem) {
  auto k = frag_kernel<N, R>;
  SF_CUDA(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int nb = 0;
  SF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k, threads, smem));
  return nb;
}

#define SF_FRAG_DISPATCH(FN, ...)                                        \
  switch (nmodes * 1000 + rank) {                                        \
    case 2016: return FN<2, 16>(__VA_ARGS__);                            \
    case 2032: return FN<2, 32>(__VA_ARGS__);                            \
    case 2064: return FN<2, 64>(__VA_ARGS__);                            \
    case 3016: return FN<3, 16>(__VA_ARGS__);                            \
    case 3032: return FN<3, 32>(__VA_ARGS__);                            \
    case 3064: return FN<3, 64>(__VA_ARGS__);                            \
    case 4016: return FN<4, 16>(__VA_ARGS__);                            \
    case 4032: return FN<4, 32>(__VA_ARGS__);                            \
    case 4064: return FN<4, 64>(__VA_ARGS__);                            \
    case 5016: return FN<5, 16>(__VA_ARGS__);                            \
    case 5032: return FN<5, 32>(__VA_ARGS__);                            \
    case 5064: return FN<5, 64>(__VA_ARGS__);                            \
    default: break;                                                      \
  }

bool frag_supported(int nmodes, int rank) {
  return nmodes >= 2 && nmodes <= 5 && (rank == 16 || rank == 32 || rank == 64);
}

int frag_max_ctas_per_sm(int nmodes, int rank, int threads, size_t smem) {
  SF_FRAG_DISPATCH(frag_occ_t, threads, smem);
  return 0;
}

static void frag_launch(int nmodes, int rank, const FragParams& fp, int grid, int threads,
                        size_t smem, cudaStream_t s) {
  SF_FRAG_DISPATCH(frag_launch_t, fp, grid, threads, smem, s);
  throw StatusError{SF_ERR_UNSUPPORTED, "frag kernel: unsupported (nmodes, rank)"};
}

void launch_mttkrp(const Tensor& t, const Plan& p, const float* const* factors, float* out,
                   cudaStream_t s) {
  const int N = t.nmodes, R = p.rank, n = p.mode;
  // A5 (v1): zero the output, then every flush is an atomic add.
  SF_CUDA(cudaMemsetAsync(out, 0, sizeof(float) * t.dims[n] * (size_t)R, s));
  if (p.nnz_local == 0) return;
  if (p.launch.kernel == SF_KERNEL_COO || !frag_supported(N, R)) {
    uint32_t* ind[SF_MAX_MODES];
    for (int m = 0; m < N; ++m) ind[m] = p.ind[m].as<uint32_t>();
    launch_coo(N, t.dims, p.nnz_local, ind, p.val.as<float>(), factors, R, n, out, s);
    return;
  }
  FragParams fp{};
  for (int m = 0; m < N; ++m) {
    fp.ind[m] = p.ind[m].as<uint32_t>();
    fp.fac[m] = factors[m];
    fp.dims[m] = (uint32_t)t.dims[m];
  }
  fp.val = p.val.as<float>();
  fp.out = out;
  fp.chunk_begin = p.chunk_begin.as<uint32_t>();
  fp.chunk_tile = p.chunk_tile.as<uint64_t>();
  fp.num_chunks = (uint32_t)p.num_chunks;
  fp.nnz = (uint32_t)p.nnz_local;
  fp.mode = n;
  fp.staged_mask = p.launch.staged_mask;
  fp.stage_words = (uint32_t)p.launch.chunk_nnz + 8;
  uint32_t off = 0;
  for (int m = 0; m < N; ++m) {
    if (p.launch.staged_mask & (1u << m)) {
      fp.block_rows[m] = p.launch.block_rows[m];
      fp.ntiles[m] = (uint32_t)((t.dims[m] + fp.block_rows[m] - 1) / fp.block_rows[m]);
      fp.fac_off[m] = off;
      off += fp.block_rows[m] * (uint32_t)R;
    } else {
      fp.block_rows[m] = 1;
      fp.ntiles[m] = 1;
    }
  }
  const size_t smem = frag_smem_bytes(t, n, R, p.launch);
  const int threads = p.launch.block_threads;
  int per_sm = p.launch.ctas_per_sm;
  const int occ = frag_max_ctas_per_sm(N, R, threads, smem);
  if (occ <= 0) throw StatusError{SF_ERR_UNSUPPORTED, "frag kernel: launch does not fit an SM"};
  if (per_sm <= 0 || per_sm > occ) per_sm = occ;
  int grid = (int)std::min<uint64_t>((uint64_t)per_sm * t.num_sms, p.num_chunks);
  grid = std::max(grid, 1);
  frag_launch(N, R, fp, grid, threads, smem, s);
  count_launch();
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    char msg[256];
    snprintf(msg, sizeof msg, "frag_kernel<%d,%d> launch grid=%d threads=%d smem=%zu occ=%d: %s", N, R, grid,
             threads, smem, occ, cudaGetErrorString(e));
    throw StatusError{SF_ERR_CUDA, msg};
  }
}

}  // namespace sf
