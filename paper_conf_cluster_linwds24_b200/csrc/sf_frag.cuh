// sf_frag.cuh - the fragment MTTKRP kernel template (§8(a) A6/A7).
//
// Y(i_n(e), :) += v_e * prod_{m != n} A_m(i_m(e), :)   (Eq. (4))
//
// Persistent CTAs walk the chunks ("segments") of the planned order
// (tile, i_n, i_s, pos).  Per chunk:
//   * one elected thread issues N+1 one-dimensional TMA bulk copies
//     (cp.async.bulk.shared::cluster.global.mbarrier) of the chunk's SoA fields into a
//     double-buffered shared-memory stage; the next chunk streams in while this one is
//     computed;
//   * when the tile changes, the factor blocks of the S "staged" modes are bulk-copied
//     into shared memory (the paper's "times_mat in shared memory");
//   * lane groups of LPN = R/4 lanes (one float4 rank slice per lane) walk contiguous
//     stretches of the chunk; a group accumulates in registers while i_n is unchanged
//     and flushes one red.global.add.v4.f32 per run edge.
// Template parameters: N modes, rank R, S staged gathered modes.  Gathered "slots"
// 0..S-1 are the staged modes (ascending mode id; gathered from shared memory),
// slots S..N-2 the others (gathered from global memory through L1/L2).  Slot order
// only changes the order of the fp32 products, not which terms are summed.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "sf_internal.h"

namespace sf {

struct FragParams {
  const uint32_t* ind[SF_MAX_MODES];  // kernel-order indices of every mode
  const float* val;
  const float* fac[SF_MAX_MODES];     // by mode
  float* out;
  const uint32_t* chunk_begin;        // num_chunks + 1
  const uint64_t* chunk_tile;         // num_chunks
  uint32_t num_chunks;
  uint32_t nnz;
  int mode;
  int slot_mode[SF_MAX_MODES];        // gathered slot -> mode (staged slots first)
  uint32_t block_rows[SF_MAX_MODES];  // per staged slot
  uint32_t ntiles[SF_MAX_MODES];      // per staged slot
  uint32_t dims[SF_MAX_MODES];        // per mode
  uint32_t fac_off[SF_MAX_MODES];     // per staged slot: float offset of its block in smem
  uint32_t stage_words;               // words per field per pipeline stage
  uint32_t owner;                     // A5: unstaged plans store whole runs, zero gaps (no memset)
  uint32_t row_end;                   // this shard's rows end (exclusive)
  uint32_t flags;                     // launch flags (SF_LAUNCH_NO_CARRY)
};

constexpr int kFragStages = 2;
constexpr int kFragUnroll = 4;

// Lane-group stretch of a chunk of n nonzeros (shared with the A5 boundary pre-pass):
// ceil(n / GPW) bumped so the GPW groups of a warp, reading word g*L + k, hit distinct
// banks (gcd(L, 32) <= LPN).
__host__ __device__ __forceinline__ uint32_t stretch_len(uint32_t n, uint32_t GPW, uint32_t LPN) {
  uint32_t L = (n + GPW - 1) / GPW;
  if (LPN < 32)
    while (L % (2u * LPN) == 0u) ++L;
  return L;
}

namespace detail {

__device__ __forceinline__ void st256(float* p, const float4& a, const float4& b) {
  asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "f"(a.x), "f"(a.y), "f"(a.z),
               "f"(a.w), "f"(b.x), "f"(b.y), "f"(b.z), "f"(b.w));
}
__device__ __forceinline__ void st128(float* p, const float4& a) {
  asm volatile("st.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(a.x), "f"(a.y), "f"(a.z), "f"(a.w));
}

__device__ __forceinline__ void red_add_v4_nomem(float* addr, const float4& v) {
  asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(addr), "f"(v.x), "f"(v.y), "f"(v.z),
               "f"(v.w));
}

__device__ __forceinline__ uint32_t su32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ float4 ldg128(const float4* p) { return __ldg(p); }

__device__ __forceinline__ void ldg256_na(const float4* p, float4& a, float4& b) {
  asm("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w), "=f"(b.x), "=f"(b.y), "=f"(b.z), "=f"(b.w)
      : "l"(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(dst)),
      "l"(src), "r"(bytes), "r"(su32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  const uint32_t a = su32(bar);
  do {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  } while (!done);
}

}  // namespace detail

// Lane mapping.  VEC = floats per lane (4 for R <= 16, else 8), LPN = R / VEC lanes per
// nonzero.  VEC = 8: lane t owns the 32 contiguous bytes of 16-byte chunks 2t, 2t+1 of a
// factor row: a global gather is ONE 256-bit load (ld.global.nc.v8.f32, sm_100), and a
// shared-memory gather is two 128-bit loads issued in parity order (quarter-warp
// half p = (lane>>2)&1 reads chunk 2t+p first), so the 8 lanes of a quarter-warp touch
// all 32 banks exactly once per load; the pair is swapped back into (2t, 2t+1).
// VEC = 4: lane t owns chunk t.
template <int R>
struct LaneMap {
  static constexpr int VEC = (R >= 32) ? 8 : 4;  // R = 16 with VEC = 8: 15-30 % slower (profiles/r01_frag3)
  static constexpr int LPN = R / VEC;
};

struct F8 {
  float4 a, b;
};

__device__ __forceinline__ void f4mul_(float4& x, const float4& y) {
  x.x *= y.x; x.y *= y.y; x.z *= y.z; x.w *= y.w;
}
__device__ __forceinline__ void f4fma_(float4& acc, const float4& x, const float4& y) {
  acc.x = fmaf(x.x, y.x, acc.x);
  acc.y = fmaf(x.y, y.y, acc.y);
  acc.z = fmaf(x.z, y.z, acc.z);
  acc.w = fmaf(x.w, y.w, acc.w);
}

template <int N, int R, int S>
__global__ void __launch_bounds__(1024) frag_kernel(const FragParams p) {
  using namespace detail;
  using LM = LaneMap<R>;
  constexpr int VEC = LM::VEC;
  constexpr int LPN = LM::LPN;  // lanes per nonzero
  constexpr int GPW = 32 / LPN; // lane groups per warp
  constexpr int G = N - 1;      // gathered slots
  constexpr int RB = R * 4;     // bytes per factor row
  constexpr int R4 = R / 4;     // float4 per factor row
  constexpr int U = (VEC == 8) ? 2 : kFragUnroll;  // batch (register budget: 64 at 1024 thr)
  extern __shared__ __align__(128) unsigned char smem_raw[];

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & 31;
  const int nwarps = blockDim.x >> 5;
  const int lane_in_group = lane % LPN;
  const int group = lane / LPN;  // group within the warp
  const int c0 = (VEC == 8) ? 2 * lane_in_group : lane_in_group;  // first owned 16-B chunk
  const int par = (lane >> 2) & 1;                                 // smem issue order (VEC 8)

  // smem: [bars: 2 per warp + 1 factor barrier, 128-B aligned] [per-warp stage rings] [factor blocks]
  const uint32_t SW = p.stage_words;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw);
  const uint32_t bar_bytes = ((2u * nwarps + 1u) * 8u + 127u) & ~127u;
  float* ring = reinterpret_cast<float*>(smem_raw + bar_bytes) + (size_t)warp * kFragStages * (N + 1) * SW;
  float* fac_smem = reinterpret_cast<float*>(smem_raw + bar_bytes) + (size_t)nwarps * kFragStages * (N + 1) * SW;
  uint64_t* wbar = bars + 2 * warp;
  uint64_t* fbar = bars + 2 * nwarps;

  // This CTA's chunks: those whose begin lies in [c*nnz/G, (c+1)*nnz/G).
  const uint64_t grid = gridDim.x;
  auto lower = [&](uint64_t target) {
    uint32_t lo = 0, hi = p.num_chunks;
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if ((uint64_t)__ldg(p.chunk_begin + mid) < target) lo = mid + 1; else hi = mid;
    }
    return lo;
  };
  const uint32_t j0 = lower(((uint64_t)blockIdx.x * p.nnz) / grid);
  const uint32_t j1 = lower(((uint64_t)(blockIdx.x + 1) * p.nnz) / grid);
  if (j0 >= j1) return;

  if (lane == 0) {
    mbar_init(&wbar[0], 1);
    mbar_init(&wbar[1], 1);
    if (warp == 0) mbar_init(fbar, 1);
    fence_barrier_init();
  }
  __syncthreads();

  // lane 0 of this warp: bulk-copy chunk j's N+1 fields into stage st (aligned superset)
  auto issue = [&](uint32_t j, int st) {
    const uint32_t b = __ldg(p.chunk_begin + j), e = __ldg(p.chunk_begin + j + 1);
    const uint32_t start = b & ~3u;
    const uint32_t bytes = (((e - start) + 3u) & ~3u) * 4u;
    float* dst = ring + (size_t)st * (N + 1) * SW;
    mbar_expect_tx(&wbar[st], bytes * (N + 1));
#pragma unroll
    for (int m = 0; m < N; ++m) bulk_g2s(dst + (size_t)m * SW, p.ind[m] + start, bytes, &wbar[st]);
    bulk_g2s(dst + (size_t)N * SW, p.val + start, bytes, &wbar[st]);
  };

  // Gather bases (float4 pointers to row 0).  Staged slots point at row 0 of the
  // *virtual* full factor (block base minus the tile's first row).
  const float4* sbase[S > 0 ? S : 1];
  const float4* gbase[G - S > 0 ? G - S : 1];
#pragma unroll
  for (int q = S; q < G; ++q) gbase[q - S] = reinterpret_cast<const float4*>(p.fac[p.slot_mode[q]]);
  uint32_t fac_phase = 0;
  uint32_t it = 0;  // chunks this warp has consumed (stage = it % 2, parity = (it / 2) & 1)
  // A7 carry: a lane group keeps its open run (row `cur`, partial acc) across its
  // consecutive stretches, so a heavy row receives one atomic per (CTA, group) instead of
  // one per stretch (shorter fp32 atomic chains: SURVEY F-c; measured on amazon mode 1).
  bool carry = false;
  uint32_t cur = 0;
  float4 acc0 = make_float4(0.f, 0.f, 0.f, 0.f), acc1 = acc0;
  float* const out0 = p.out + 4 * c0;
  float* const out1 = out0 + 4;

  uint32_t seg = j0;
  while (seg < j1) {
    // tile segment [seg, seg_end): chunks of one tile (the whole range when S == 0)
    uint32_t seg_end = j1;
    if constexpr (S > 0) {
      const uint64_t tile = __ldg(p.chunk_tile + seg);
      uint32_t lo = seg + 1, hi = j1;  // first chunk with a different (larger) tile
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (__ldg(p.chunk_tile + mid) == tile) lo = mid + 1; else hi = mid;
      }
      seg_end = lo;
      uint64_t t = tile;
      uint32_t row0[S];
#pragma unroll
      for (int q = S - 1; q >= 0; --q) {
        const uint32_t qq = (uint32_t)(t % p.ntiles[q]);
        t /= p.ntiles[q];
        row0[q] = qq * p.block_rows[q];
      }
      __syncthreads();  // every warp is done with the previous blocks
      if (tid == 0) {
        uint32_t total = 0;
#pragma unroll
        for (int q = 0; q < S; ++q) total += min(p.block_rows[q], p.dims[p.slot_mode[q]] - row0[q]) * RB;
        mbar_expect_tx(fbar, total);
#pragma unroll
        for (int q = 0; q < S; ++q) {
          const uint32_t rows = min(p.block_rows[q], p.dims[p.slot_mode[q]] - row0[q]);
          bulk_g2s(fac_smem + p.fac_off[q], p.fac[p.slot_mode[q]] + (size_t)row0[q] * R, rows * RB, fbar);
        }
      }
#pragma unroll
      for (int q = 0; q < S; ++q)
        sbase[q] = reinterpret_cast<const float4*>(fac_smem + p.fac_off[q]) - (ptrdiff_t)row0[q] * R4;
    }
    // this warp's chunks of the segment: seg + warp, seg + warp + nwarps, ...
    uint32_t jn = seg + warp;
    if (lane == 0) {
      if (jn < seg_end) issue(jn, it % kFragStages);
      if (jn + nwarps < seg_end) issue(jn + nwarps, (it + 1) % kFragStages);
    }
    if constexpr (S > 0) {
      mbar_wait(fbar, fac_phase);
      fac_phase ^= 1u;
    }
    for (uint32_t j = jn; j < seg_end; j += nwarps, ++it) {
      const int st = (int)(it % kFragStages);
      mbar_wait(&wbar[st], (it / kFragStages) & 1u);
      const uint32_t b = __ldg(p.chunk_begin + j), e = __ldg(p.chunk_begin + j + 1);
      const uint32_t n = e - b;
      const float* sb = ring + (size_t)st * (N + 1) * SW + (b - (b & ~3u));
      const uint32_t L = stretch_len(n, GPW, LPN);
      const uint32_t k0 = group * L;
      const uint32_t k1 = min(n, k0 + L);
      if (k0 < k1) {
        const uint32_t* sOut = reinterpret_cast<const uint32_t*>(sb + (size_t)p.mode * SW);
        const float* sVal = sb + (size_t)N * SW;
        const uint32_t* sIdx[G];
#pragma unroll
        for (int q = 0; q < G; ++q) sIdx[q] = reinterpret_cast<const uint32_t*>(sb + (size_t)p.slot_mode[q] * SW);
        // gather slot q of nonzero kk (staged: shared memory, else global via L1/L2)
        auto gather = [&](int q, uint32_t kk) -> F8 {
          const float4* base = (q < S) ? sbase[q < S ? q : 0] : gbase[q >= S ? q - S : 0];
          const size_t row = (size_t)sIdx[q][kk] * R4;
          F8 r;
          if constexpr (VEC == 8) {
            if (q < S) {
              const float4 x = base[row + c0 + par];
              const float4 y = base[row + c0 + 1 - par];
              r.a = par ? y : x;
              r.b = par ? x : y;
            } else {
              ldg256_na(base + row + c0, r.a, r.b);  // L1::no_allocate (measured faster)
            }
          } else {
            r.a = (q < S) ? base[row + c0] : ldg128(base + row + c0);
          }
          return r;
        };
        bool shared = true;       // current run may be shared with another stretch/tile
        bool last_shared = true;  // the stretch's last run continues past k1
        const uint32_t first = sOut[k0];
        bool first_shared = true;
        uint32_t before = 0xFFFFFFFFu;
        if constexpr (S == 0) {
          if (p.owner) {
            const uint32_t P0 = b + k0, P1 = b + k1;
            const uint32_t* gOut = p.ind[p.mode];
            before = (P0 > 0) ? __ldg(gOut + P0 - 1) : 0xFFFFFFFFu;
            first_shared = (P0 > 0) && before == first;
            last_shared = (P1 < p.nnz) && __ldg(gOut + P1) == sOut[k1 - 1];
          }
        }
        auto flush_run = [&](bool atomic) {
          if (atomic) {
            red_add_v4_nomem(out0 + (size_t)cur * R, acc0);
            if constexpr (VEC == 8) red_add_v4_nomem(out1 + (size_t)cur * R, acc1);
          } else {
            if constexpr (VEC == 8) st256(out0 + (size_t)cur * R, acc0, acc1);
            else st128(out0 + (size_t)cur * R, acc0);
          }
          acc0 = make_float4(0.f, 0.f, 0.f, 0.f);
          acc1 = acc0;
        };
        if (carry && first != cur) {  // the carried run ended before this stretch
          flush_run(true);
          carry = false;
        }
        if (carry) {
          shared = true;  // continuing a run begun in an earlier stretch
        } else {
          cur = first;
          shared = first_shared;
          if constexpr (S == 0) {
            if (p.owner && !first_shared && b + k0 > 0)  // gap rows (before, first) are ours
              for (uint32_t r = before + 1; r < first; ++r) {
                if constexpr (VEC == 8) st256(out0 + (size_t)r * R, make_float4(0.f, 0.f, 0.f, 0.f),
                                              make_float4(0.f, 0.f, 0.f, 0.f));
                else st128(out0 + (size_t)r * R, make_float4(0.f, 0.f, 0.f, 0.f));
              }
          }
        }
        // run edge inside the stretch: close `cur`, zero the gap up to the next row i
        auto flush = [&]() { flush_run(shared); };
        auto advance = [&](uint32_t i) {
          if constexpr (S == 0) {
            if (p.owner) {
              for (uint32_t r = cur + 1; r < i; ++r) {
                if constexpr (VEC == 8) st256(out0 + (size_t)r * R, make_float4(0.f, 0.f, 0.f, 0.f),
                                              make_float4(0.f, 0.f, 0.f, 0.f));
                else st128(out0 + (size_t)r * R, make_float4(0.f, 0.f, 0.f, 0.f));
              }
              shared = false;
            }
          }
          cur = i;
        };
        uint32_t k = k0;
        // y += v * (a_0 * ... * a_{G-1}): G-1 FMUL + 1 FFMA per float
        for (; k + U <= k1; k += U) {
          uint32_t ii[U];
          float vv[U];
          F8 pr[U];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            ii[u] = sOut[k + u];
            vv[u] = sVal[k + u];
          }
#pragma unroll
          for (int q = 0; q < G; ++q) {
#pragma unroll
            for (int u = 0; u < U; ++u) {
              const F8 a = gather(q, k + u);
              if (q == 0) {
                pr[u] = a;
              } else {
                f4mul_(pr[u].a, a.a);
                if constexpr (VEC == 8) f4mul_(pr[u].b, a.b);
              }
            }
          }
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (ii[u] != cur) {
              flush();
              advance(ii[u]);
            }
            const float4 vb = make_float4(vv[u], vv[u], vv[u], vv[u]);
            f4fma_(acc0, vb, pr[u].a);
            if constexpr (VEC == 8) f4fma_(acc1, vb, pr[u].b);
          }
        }
        for (; k < k1; ++k) {
          const uint32_t i = sOut[k];
          const float v = sVal[k];
          F8 pr = gather(0, k);
#pragma unroll
          for (int q = 1; q < G; ++q) {
            const F8 a = gather(q, k);
            f4mul_(pr.a, a.a);
            if constexpr (VEC == 8) f4mul_(pr.b, a.b);
          }
          if (i != cur) {
            flush();
            advance(i);
          }
          const float4 vb = make_float4(v, v, v, v);
          f4fma_(acc0, vb, pr.a);
          if constexpr (VEC == 8) f4fma_(acc1, vb, pr.b);
        }
        // carry only a run that filled the whole stretch (a heavy row); shorter runs that
        // merely cross the boundary are flushed now (cheaper, and their chains are short)
        if (last_shared && first == cur && !(p.flags & SF_LAUNCH_NO_CARRY)) {
          carry = true;  // the run continues past this stretch: keep accumulating
        } else {
          flush_run(shared || last_shared);  // a run crossing into the next stretch is shared
          carry = false;
        }
      }
      __syncwarp();  // every lane is done reading stage st
      if (lane == 0 && j + 2u * nwarps < seg_end) issue(j + 2u * nwarps, st);
    }
    seg = seg_end;
  }
  if (carry) {  // close the run still open at the end of this CTA's range
    red_add_v4_nomem(out0 + (size_t)cur * R, acc0);
    if constexpr (VEC == 8) red_add_v4_nomem(out1 + (size_t)cur * R, acc1);
  }
}

// A5 pre-pass for owner mode: zero the rows whose run crosses a stretch boundary (they
// receive atomic partial sums), i.e. rows(pos) with row(pos) == row(pos-1) at every
// stretch start pos.  One thread per (chunk, group).
template <int R>
__global__ void boundary_zero_kernel(const uint32_t* __restrict__ chunk_begin, uint32_t num_chunks,
                                     const uint32_t* __restrict__ rows, float* __restrict__ out) {
  using LM = LaneMap<R>;
  constexpr uint32_t GPW = 32 / LM::LPN;
  const uint64_t total = (uint64_t)num_chunks * GPW;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
    const uint32_t j = (uint32_t)(t / GPW), g = (uint32_t)(t % GPW);
    const uint32_t b = chunk_begin[j], e = chunk_begin[j + 1];
    const uint32_t pos = b + g * stretch_len(e - b, GPW, LM::LPN);
    if (pos >= e || pos == 0) continue;
    const uint32_t r = rows[pos];
    if (rows[pos - 1] != r) continue;
    float4* y = reinterpret_cast<float4*>(out + (size_t)r * R);
#pragma unroll
    for (int c = 0; c < R / 4; ++c) y[c] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
}

// Per-R dispatch (defined in sf_frag_r{16,32,64}.cu).
void frag_launch_r16(int N, int S, const FragParams& fp, int grid, int threads, size_t smem, cudaStream_t s);
void frag_launch_r32(int N, int S, const FragParams& fp, int grid, int threads, size_t smem, cudaStream_t s);
void frag_launch_r64(int N, int S, const FragParams& fp, int grid, int threads, size_t smem, cudaStream_t s);
int frag_occ_r16(int N, int S, int threads, size_t smem);
void boundary_zero_r16(const uint32_t* cb, uint32_t nc, const uint32_t* rows, float* out, cudaStream_t s);
void boundary_zero_r32(const uint32_t* cb, uint32_t nc, const uint32_t* rows, float* out, cudaStream_t s);
void boundary_zero_r64(const uint32_t* cb, uint32_t nc, const uint32_t* rows, float* out, cudaStream_t s);
int frag_occ_r32(int N, int S, int threads, size_t smem);
int frag_occ_r64(int N, int S, int threads, size_t smem);

template <int N, int R, int S>
void frag_launch_one(const FragParams& fp, int grid, int threads, size_t smem, cudaStream_t s) {
  auto k = frag_kernel<N, R, S>;
  SF_CUDA(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  k<<<grid, threads, smem, s>>>(fp);
}

template <int N, int R, int S>
int frag_occ_one(int threads, size_t smem) {
  auto k = frag_kernel<N, R, S>;
  SF_CUDA(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int nb = 0;
  SF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k, threads, smem));
  return nb;
}

// (N, S) -> instantiation, for one R.
#define SF_FRAG_NS_SWITCH(R, FN, ...)                  \
  switch (N * 10 + S) {                                \
    case 20: return FN<2, R, 0>(__VA_ARGS__);          \
    case 21: return FN<2, R, 1>(__VA_ARGS__);          \
    case 30: return FN<3, R, 0>(__VA_ARGS__);          \
    case 31: return FN<3, R, 1>(__VA_ARGS__);          \
    case 32: return FN<3, R, 2>(__VA_ARGS__);          \
    case 40: return FN<4, R, 0>(__VA_ARGS__);          \
    case 41: return FN<4, R, 1>(__VA_ARGS__);          \
    case 42: return FN<4, R, 2>(__VA_ARGS__);          \
    case 43: return FN<4, R, 3>(__VA_ARGS__);          \
    case 50: return FN<5, R, 0>(__VA_ARGS__);          \
    case 51: return FN<5, R, 1>(__VA_ARGS__);          \
    case 52: return FN<5, R, 2>(__VA_ARGS__);          \
    case 53: return FN<5, R, 3>(__VA_ARGS__);          \
    case 54: return FN<5, R, 4>(__VA_ARGS__);          \
    default: break;                                    \
  }

#define SF_DEFINE_FRAG_R(R)                                                                              \
  void frag_launch_r##R(int N, int S, const FragParams& fp, int grid, int threads, size_t smem,          \
                        cudaStream_t s) {                                                                \
    SF_FRAG_NS_SWITCH(R, frag_launch_one, fp, grid, threads, smem, s);                                   \
    throw StatusError{SF_ERR_UNSUPPORTED, "frag kernel: unsupported (N, S)"};                           \
  }                                                                                                      \
  int frag_occ_r##R(int N, int S, int threads, size_t smem) {                                            \
    SF_FRAG_NS_SWITCH(R, frag_occ_one, threads, smem);                                                   \
    return 0;                                                                                            \
  }                                                                                                      \
  void boundary_zero_r##R(const uint32_t* cb, uint32_t nc, const uint32_t* rows, float* out,            \
                          cudaStream_t s) {                                                              \
    const uint64_t total = (uint64_t)nc * (32 / LaneMap<R>::LPN);                                        \
    const int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>((total + 255) / 256, 148 * 16));     \
    boundary_zero_kernel<R><<<grid, 256, 0, s>>>(cb, nc, rows, out);                                    \
  }

}  // namespace sf
