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
// frag3_kernel (SF_KERNEL_FRAG, sf_frag3.cuh): persistent CTAs walk the planned order
//   (tile, i_n, i_s) of packed records; each lane group owns a contiguous sub-range,
//   stages its records into shared memory by 1-D TMA bulk copies (cp.async.bulk +
//   mbarrier, double buffered), gathers "staged" factor blocks from shared memory (the
//   paper's "times_mat in shared memory") and the others from L2, and
//   accumulates in registers while i_n is unchanged, flushing once per run -- global
//   atomics fire only at run / sub-range boundaries (north_star).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>

#include "sf_frag3.cuh"
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
  uint64_t dims[SF_MAX_MODES];  // a nonzero with some index >= dims[m] is skipped (the streamed
                                // path range-checks segments concurrently with this kernel)
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
    bool ok = true;
#pragma unroll
    for (int m = 0; m < SF_MAX_MODES; ++m) {
      if (m >= p.nmodes) break;
      if (m == p.mode) continue;
      const uint32_t im = __ldg(p.ind[m] + e);
      ok = ok && im < p.dims[m];
      if (ok) acc = f4mul(acc, ldg_f4(p.fac[m] + (size_t)im * R + 4 * sub));
    }
    const uint32_t in = __ldg(p.ind[p.mode] + e);
    if (ok && in < p.dims[p.mode]) red_add_v4(p.out + (size_t)in * R + 4 * sub, acc);
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
    bool ok = true;
    for (int m = 0; m < p.nmodes && ok; ++m) {
      const uint32_t im = __ldg(p.ind[m] + e);
      ok = im < p.dims[m];
      if (ok && m != p.mode) acc *= __ldg(p.fac[m] + (size_t)im * p.rank + r);
    }
    if (ok) atomicAdd(p.out + (size_t)__ldg(p.ind[p.mode] + e) * p.rank + r, acc);
  }
}

void launch_coo(int nmodes, const uint64_t* dims, uint64_t nnz, const uint32_t* const* inds,
                const float* vals, const float* const* factors, int rank, int mode, float* out,
                cudaStream_t s) {
  if (nnz == 0) return;
  CooParams p{};
  for (int m = 0; m < nmodes; ++m) { p.ind[m] = inds[m]; p.fac[m] = factors[m]; p.dims[m] = dims[m]; }
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
// Sorted-segment kernel (the one-shot streamed paths, §8(a) A8 (ii)).  A segment of the raw
// COO, once on the device, is copied into W-word AoS records [i_0 .. i_{N-1}, 0.., v]
// (one coalesced pass, shared by every mode computed from the segment) and sorted by i_n
// (keys = i_n, payload = position in the segment); each lane group then walks a contiguous
// range of the sorted positions, reading each nonzero as one 16/32-byte record, accumulating
// in registers while i_n is unchanged and adding one vector atomic per run piece -- a heavy
// row gets one atomic per (segment, group) instead of one per nonzero, which keeps the fp32
// chain short (SURVEY C-2: amazon's 1.2e8-nonzero row).  SEG_U nonzeros per group are in
// flight (their records and factor rows are loaded before any is accumulated).
// Out-of-range nonzeros are skipped (the segment's range check runs before and is reported
// at the end).
// ---------------------------------------------------------------------------
struct SegParams {
  const uint32_t* aos;                // segment records (input order), W words each
  const uint32_t* skey;               // sorted i_n
  const uint32_t* spos;               // position of the sorted slot in the segment
  const float* fac[SF_MAX_MODES];
  float* out;
  uint64_t dims[SF_MAX_MODES];
  uint64_t len;
  uint32_t dn;                        // min(dims[mode], 2^32 - 1): i_n >= dn is skipped
  int nmodes, mode;
};

constexpr int SEG_U = 4;

template <int R, int W>
__global__ void __launch_bounds__(256) seg_sorted_kernel(SegParams p) {
  constexpr int LPN = R / 4;
  const int sub = threadIdx.x % LPN;
  const uint64_t g = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) / LPN;
  const uint64_t G = ((uint64_t)gridDim.x * blockDim.x) / LPN;
  const uint64_t k0 = g * p.len / G, k1 = (g + 1) * p.len / G;
  const uint32_t dn = p.dn;
  uint32_t cur = 0xFFFFFFFFu;
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (uint64_t k = k0; k < k1; k += SEG_U) {
    uint32_t ii[SEG_U];
    uint32_t w[SEG_U][W];
#pragma unroll
    for (int u = 0; u < SEG_U; ++u) {
      const bool in = k + u < k1;
      ii[u] = in ? __ldg(p.skey + k + u) : 0xFFFFFFFFu;
      const uint32_t e = in ? __ldg(p.spos + k + u) : 0u;
      const uint4* r = reinterpret_cast<const uint4*>(p.aos + (size_t)e * W);
#pragma unroll
      for (int q = 0; q < W / 4; ++q) {
        const uint4 x = __ldg(r + q);
        w[u][4 * q] = x.x; w[u][4 * q + 1] = x.y; w[u][4 * q + 2] = x.z; w[u][4 * q + 3] = x.w;
      }
    }
    float4 prod[SEG_U];
    bool ok[SEG_U];
#pragma unroll
    for (int u = 0; u < SEG_U; ++u) {
      const float v = __uint_as_float(w[u][W - 1]);
      prod[u] = make_float4(v, v, v, v);
      ok[u] = ii[u] < dn;
    }
#pragma unroll
    for (int m = 0; m < W - 1; ++m) {
      if (m < p.nmodes && m != p.mode) {
#pragma unroll
        for (int u = 0; u < SEG_U; ++u) {
          const uint32_t im = w[u][m];
          ok[u] = ok[u] && im < p.dims[m];
          if (ok[u]) prod[u] = f4mul(prod[u], ldg_f4(p.fac[m] + (size_t)im * R + 4 * sub));
        }
      }
    }
#pragma unroll
    for (int u = 0; u < SEG_U; ++u) {
      if (k + u >= k1) continue;
      if (ii[u] != cur) {
        if (cur != 0xFFFFFFFFu) red_add_v4(p.out + (size_t)cur * R + 4 * sub, acc);
        acc = make_float4(0.f, 0.f, 0.f, 0.f);
        cur = ii[u] < dn ? ii[u] : 0xFFFFFFFFu;
      }
      if (ok[u]) {
        acc.x += prod[u].x; acc.y += prod[u].y; acc.z += prod[u].z; acc.w += prod[u].w;
      }
    }
  }
  if (cur != 0xFFFFFFFFu) red_add_v4(p.out + (size_t)cur * R + 4 * sub, acc);
}

bool seg_sorted_supported(int rank) { return rank == 16 || rank == 32 || rank == 64; }

int seg_aos_words(int nmodes) { return (nmodes + 1 <= 4) ? 4 : 8; }

struct SegAosParams {
  const uint32_t* ind[SF_MAX_MODES];
  const float* val;
  uint32_t* aos;
  int nmodes, W;
};

__global__ void seg_aos_kernel(SegAosParams a, uint64_t n) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += stride) {
    uint32_t w[8] = {0, 0, 0, 0, 0, 0, 0, 0};
#pragma unroll
    for (int m = 0; m < 7; ++m)
      if (m < a.nmodes) w[m] = __ldg(a.ind[m] + e);
    const uint32_t v = __float_as_uint(__ldg(a.val + e));
    uint4* r = reinterpret_cast<uint4*>(a.aos + e * a.W);
    if (a.W == 8) {
      r[0] = make_uint4(w[0], w[1], w[2], w[3]);
      r[1] = make_uint4(w[4], w[5], w[6], v);
    } else {
      r[0] = make_uint4(w[0], w[1], w[2], v);
    }
  }
}

void launch_seg_aos(int nmodes, uint64_t len, const uint32_t* const* inds, const float* vals, uint32_t* aos,
                    cudaStream_t s) {
  if (len == 0) return;
  if (nmodes > 7) throw StatusError{SF_ERR_UNSUPPORTED, "sorted segments: nmodes <= 7"};
  SegAosParams a{};
  for (int m = 0; m < nmodes; ++m) a.ind[m] = inds[m];
  a.val = vals;
  a.aos = aos;
  a.nmodes = nmodes;
  a.W = seg_aos_words(nmodes);
  seg_aos_kernel<<<(int)std::min<uint64_t>((len + 255) / 256, 148 * 16), 256, 0, s>>>(a, len);
  count_launch();
  SF_CUDA(cudaGetLastError());
}

void launch_seg_sorted(int nmodes, const uint64_t* dims, uint64_t len, const uint32_t* aos, const uint32_t* skey,
                       const uint32_t* spos, const float* const* factors, int rank, int mode, float* out,
                       cudaStream_t s) {
  if (len == 0) return;
  SegParams p{};
  for (int m = 0; m < nmodes; ++m) { p.fac[m] = factors[m]; p.dims[m] = dims[m]; }
  p.aos = aos;
  p.skey = skey;
  p.spos = spos;
  p.out = out;
  p.len = len;
  p.dn = (uint32_t)std::min<uint64_t>(dims[mode], 0xFFFFFFFFull);
  p.nmodes = nmodes;
  p.mode = mode;
  // ~64 nonzeros per lane group: long runs per group, enough groups to fill the GPU
  auto grid_for = [&](int lpn) {
    const uint64_t groups = std::max<uint64_t>(1, len / 64);
    return (int)std::max<uint64_t>(1, std::min<uint64_t>((groups * lpn + 255) / 256, (uint64_t)148 * 16));
  };
  const bool w8 = seg_aos_words(nmodes) == 8;
  if (rank == 16) {
    if (w8) seg_sorted_kernel<16, 8><<<grid_for(4), 256, 0, s>>>(p);
    else seg_sorted_kernel<16, 4><<<grid_for(4), 256, 0, s>>>(p);
  } else if (rank == 32) {
    if (w8) seg_sorted_kernel<32, 8><<<grid_for(8), 256, 0, s>>>(p);
    else seg_sorted_kernel<32, 4><<<grid_for(8), 256, 0, s>>>(p);
  } else {
    if (w8) seg_sorted_kernel<64, 8><<<grid_for(16), 256, 0, s>>>(p);
    else seg_sorted_kernel<64, 4><<<grid_for(16), 256, 0, s>>>(p);
  }
  count_launch();
  SF_CUDA(cudaGetLastError());
}

__global__ void iota_kernel(uint32_t* __restrict__ x, uint64_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    x[i] = (uint32_t)i;
}

void launch_iota(uint32_t* x, uint64_t n, cudaStream_t s) {
  if (!n) return;
  iota_kernel<<<(int)std::min<uint64_t>((n + 255) / 256, 148 * 16), 256, 0, s>>>(x, n);
  count_launch();
  SF_CUDA(cudaGetLastError());
}

// ---------------------------------------------------------------------------
// Boundary-row helper (multi-GPU exchange, §8(e))
// ---------------------------------------------------------------------------
__global__ void rows_op_kernel(float* __restrict__ Y, int R, const int64_t* __restrict__ rows,
                               float* __restrict__ buf, int count, int op) {
  const int k = blockIdx.x;
  if (k >= count) return;
  const int64_t r = rows[k];
  if (r < 0) return;
  for (int c = threadIdx.x; c < R; c += blockDim.x) {
    float* y = Y + (size_t)r * R + c;
    if (op == 0) buf[(size_t)k * R + c] = *y;
    else if (op == 1) atomicAdd(y, buf[(size_t)k * R + c]);  // several entries may target one row
    else *y = 0.f;
  }
}

void launch_rows_op(float* Y, int R, const int64_t* rows, float* buf, int count, int op, cudaStream_t s) {
  if (count <= 0) return;
  rows_op_kernel<<<count, 128, 0, s>>>(Y, R, rows, buf, count, op);
  count_launch();
  SF_CUDA(cudaGetLastError());
}

bool frag_supported(int nmodes, int rank) {
  return nmodes >= 2 && nmodes <= 5 && (rank == 16 || rank == 32 || rank == 64);
}

int frag_slot_order(int nmodes, int mode, uint32_t staged_mask, int* slot_mode) {
  int q = 0;
  for (int m = 0; m < nmodes; ++m)
    if (m != mode && (staged_mask & (1u << m))) slot_mode[q++] = m;
  const int S = q;
  for (int m = 0; m < nmodes; ++m)
    if (m != mode && !(staged_mask & (1u << m))) slot_mode[q++] = m;
  return S;
}

// Hot-row cache fill: cache[begin[k] + j, :] = src[k][rows[k][j], :] (float4 per thread).
struct HotFill {
  const float* src[SF_MAX_MODES];
  const uint32_t* rows[SF_MAX_MODES];
  uint64_t begin[SF_MAX_MODES + 1];
  int nslots;
};

__global__ void hot_fill_kernel(const HotFill h, int R4, float* __restrict__ cache) {
  const uint64_t total = h.begin[h.nslots] * (uint64_t)R4;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += stride) {
    const uint64_t r = e / R4;
    const int c = (int)(e - r * R4);
    int k = 0;
    while (k + 1 < h.nslots && r >= h.begin[k + 1]) ++k;
    const uint32_t src_row = __ldg(h.rows[k] + (r - h.begin[k]));
    const float4 v = __ldg(reinterpret_cast<const float4*>(h.src[k] + (size_t)src_row * R4 * 4) + c);
    reinterpret_cast<float4*>(cache)[e] = v;
  }
}

static int frag3_occ(int N, int R, int S, int threads, size_t smem, bool hot) {
  switch (R) {
    case 16: return frag3_occ_r16(N, S, threads, smem, hot);
    case 32: return frag3_occ_r32(N, S, threads, smem, hot);
    case 64: return frag3_occ_r64(N, S, threads, smem, hot);
    default: return 0;
  }
}

// frag3 path (record plans): A5 owner pre-pass on the frag3 group partition, then the kernel.
static void launch_frag3(const Tensor& t, const Plan& p, const float* const* factors, float* out,
                         cudaStream_t s, bool owner) {
  const int N = t.nmodes, R = p.rank, n = p.mode;
  Frag3Params fp{};
  for (int m = 0; m < N; ++m) {
    fp.fac[m] = factors[m];
    fp.dims[m] = (uint32_t)t.dims[m];
  }
  fp.rec = p.rec.as<uint32_t>();
  fp.out = out;
  fp.chunk_begin = p.chunk_begin.as<uint32_t>();
  fp.chunk_tile = p.chunk_tile.as<uint64_t>();
  fp.tile_chunk = p.tile_chunk.as<uint32_t>();
  fp.num_tiles = (uint32_t)p.num_tiles;
  fp.num_chunks = (uint32_t)p.num_chunks;
  fp.nnz = (uint32_t)p.nnz_local;
  const uint32_t gpw = (uint32_t)frag_groups_per_warp(R);
  fp.K = frag3_K((uint32_t)p.launch.chunk_nnz, gpw);
  fp.W = (uint32_t)p.rec_words;
  fp.out_mask = p.rec_packed ? p.rec_bmask[0] : 0xFFFFFFFFu;
  for (int f = 0; f < SF_MAX_MODES; ++f) {
    fp.boff[f] = p.rec_boff[f];
    fp.bmask[f] = p.rec_bmask[f];
  }
  fp.owner = owner ? 1u : 0u;
  const int S = frag_slot_order(N, n, smem_staged_mask(p.launch), fp.slot_mode);
  if (p.hot_total) {  // hot-row cache: this call's copy of every slot's hot rows
    HotFill hf{};
    int k = 0;
    for (int q = 0; q < N - 1; ++q) {
      if (!p.hot_bit[q] || !p.hot_count[q]) continue;
      hf.src[k] = factors[fp.slot_mode[q]];
      hf.rows[k] = p.hot_rows[q].as<uint32_t>();
      hf.begin[k] = p.hot_off[q];
      ++k;
    }
    hf.nslots = k;
    hf.begin[k] = p.hot_total;
    float* cache = p.hot_cache.as<float>();
    const uint64_t items = p.hot_total * (uint64_t)(R / 4);
    const int g = (int)std::max<uint64_t>(1, std::min<uint64_t>((items + 255) / 256, (uint64_t)t.num_sms * 16));
    hot_fill_kernel<<<g, 256, 0, s>>>(hf, R / 4, cache);
    count_launch();
    SF_CUDA(cudaGetLastError());
    for (int q = 0; q < N - 1; ++q) {
      fp.hot_bit[q] = p.hot_bit[q];
      if (p.hot_bit[q])
        fp.hot_delta[q] = (int64_t)((reinterpret_cast<intptr_t>(cache + p.hot_off[q] * (uint64_t)R) -
                                     reinterpret_cast<intptr_t>(factors[fp.slot_mode[q]])) / 16);
    }
  }
  fp.l2tiles = (p.launch.flags & SF_LAUNCH_L2_TILES) ? 1u : 0u;
  uint32_t off = 0;
  for (int q = 0; q < S; ++q) {
    const int m = fp.slot_mode[q];
    fp.block_rows[q] = p.launch.block_rows[m];
    fp.ntiles[q] = (uint32_t)((t.dims[m] + fp.block_rows[q] - 1) / fp.block_rows[q]);
    fp.fac_off[q] = off;
    off += fp.block_rows[q] * (uint32_t)R;
  }
  const sf_launch_t& l = p.launch;
  const size_t smem = frag_smem_bytes(t, n, R, l);
  const int threads = l.block_threads;
  int per_sm = l.ctas_per_sm;
  if (p.occ_threads != threads || p.occ_smem != smem) {  // occupancy query once per plan launch shape
    p.occ = frag3_occ(N, R, S, threads, smem, p.hot_total > 0);
    p.occ_threads = threads;
    p.occ_smem = smem;
  }
  const int occ = p.occ;
  if (occ <= 0) throw StatusError{SF_ERR_UNSUPPORTED, "frag3 kernel: launch does not fit an SM"};
  if (per_sm <= 0 || per_sm > occ) per_sm = occ;
  int grid = (int)std::min<uint64_t>((uint64_t)per_sm * t.num_sms, p.num_chunks);
  grid = std::max(grid, 1);
  const uint32_t groups = (uint32_t)(threads / 32) * gpw;
  if (p.cta_grid != grid) {  // per-CTA chunk ranges, once per (plan, grid)
    p.cta_chunk.alloc(((size_t)grid + 1) * 4 + 16);
    frag3_cta_range_kernel<<<(grid + 256) / 256, 256, 0, s>>>(fp.chunk_begin, fp.num_chunks, fp.nnz, (uint32_t)grid,
                                                             p.cta_chunk.as<uint32_t>());
    count_launch();
    SF_CUDA(cudaGetLastError());
    p.cta_grid = grid;
  }
  fp.cta_chunk = p.cta_chunk.as<uint32_t>();
  const bool det = owner && (l.flags & SF_LAUNCH_DETERMINISTIC);
  const uint64_t nslots = 2ull * (uint64_t)grid * groups;
  if (det) {  // A7 deterministic option: carry slots instead of atomics (no pre-zero needed)
    const size_t need = nslots * 4 + 16 + nslots * (size_t)R * 4;
    if (p.carry.bytes < need) { p.carry.release(); p.carry.alloc(need); }
    fp.carry_row = p.carry.as<uint32_t>();
    fp.carry_val = reinterpret_cast<float*>(p.carry.as<unsigned char>() + ((nslots * 4 + 15) & ~(size_t)15));
    SF_CUDA(cudaMemsetAsync(fp.carry_row, 0xFF, nslots * 4, s));
  } else if (owner) {
    switch (R) {
      case 16: boundary_zero3_r16(fp, (uint32_t)grid, groups, out, s); break;
      case 32: boundary_zero3_r32(fp, (uint32_t)grid, groups, out, s); break;
      default: boundary_zero3_r64(fp, (uint32_t)grid, groups, out, s); break;
    }
    count_launch();
    SF_CUDA(cudaGetLastError());
  }
  switch (R) {
    case 16: frag3_launch_r16(N, S, fp, grid, threads, smem, s); break;
    case 32: frag3_launch_r32(N, S, fp, grid, threads, smem, s); break;
    case 64: frag3_launch_r64(N, S, fp, grid, threads, smem, s); break;
    default: throw StatusError{SF_ERR_UNSUPPORTED, "frag3 kernel: unsupported rank"};
  }
  count_launch();
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    char msg[256];
    snprintf(msg, sizeof msg, "frag3_kernel<%d,%d,%d> launch grid=%d threads=%d smem=%zu occ=%d: %s", N, R, S,
             grid, threads, smem, occ, cudaGetErrorString(e));
    throw StatusError{SF_ERR_CUDA, msg};
  }
  if (det) {
    const int cgrid = (int)std::max<uint64_t>(1, std::min<uint64_t>((nslots * 32 + 255) / 256, 148 * 16));
    frag3_combine_kernel<<<cgrid, 256, 0, s>>>(fp.carry_row, fp.carry_val, nslots, R, out);
    count_launch();
    SF_CUDA(cudaGetLastError());
  }
}

void launch_mttkrp(const Tensor& t, const Plan& p, const float* const* factors, float* out_block,
                   cudaStream_t s) {
  const int N = t.nmodes, R = p.rank;
  const bool frag = p.launch.kernel == SF_KERNEL_FRAG && frag_supported(N, R) && p.rec_words;
  // A5: unstaged fragment plans run in owner mode (whole runs stored, gaps zeroed by
  // their owner, only run-crossing rows pre-zeroed by launch_frag3); everything else
  // zeroes Y and adds.
  const bool owner = frag && p.launch.staged_mask == 0 && p.nnz_local > 0 &&
                     !(p.launch.flags & SF_LAUNCH_NO_OWNER_STORES);
  const size_t row_bytes = sizeof(float) * (size_t)R;
  // the caller's block holds rows [out_row0, out_row0 + out_rows); the kernels index Y by
  // absolute row and only touch rows in [row_begin, row_end), inside the block
  float* out = out_block - p.out_row0 * (size_t)R;
  const uint64_t blk_end = p.out_row0 + p.out_rows;
  if (!owner) {
    SF_CUDA(cudaMemsetAsync(out_block, 0, row_bytes * p.out_rows, s));
  } else {  // block rows no nonzero of this shard touches (unsharded: rows before/after)
    if (p.row_begin > p.out_row0) SF_CUDA(cudaMemsetAsync(out_block, 0, row_bytes * (p.row_begin - p.out_row0), s));
    if (p.row_end < blk_end)
      SF_CUDA(cudaMemsetAsync(out + p.row_end * (size_t)R, 0, row_bytes * (blk_end - p.row_end), s));
  }
  if (p.nnz_local == 0) return;
  if (frag) return launch_frag3(t, p, factors, out, s, owner);
  uint32_t* ind[SF_MAX_MODES];
  for (int m = 0; m < N; ++m) ind[m] = p.ind[m].as<uint32_t>();
  launch_coo(N, t.dims, p.nnz_local, ind, p.val.as<float>(), factors, R, p.mode, out, s);
}

}  // namespace sf
