// sf_frag3.cuh - record-packed, group-contiguous fragment MTTKRP kernel (§8(a) A5-A7).
//
// Y(i_n(e), :) += v_e * prod_{m != n} A_m(i_m(e), :)   (Eq. (4))
//
// Same method as the round-1 SoA frag_kernel (chunks of 128 nonzeros cut into 8 stretches), with two changes that cut L1TEX work per
// nonzero -- the resource that binds on sm_100a when the factors are L2-resident
// (profiles/r01_ncu_full_nell2.json: l1tex 92 %, DRAM 16 %):
//   1. Records.  The plan stores each nonzero as one W-word record in *slot order*
//      [i_n, g_0, ..., g_{N-2}, v, pad] (W = 4 for N <= 3, 8 for N <= 7), so a lane group
//      reads its nonzero with one (W = 4) or two 128-bit shared loads instead of N+1
//      32-bit loads, and one TMA bulk copy moves a group's K records per stage.
//      PK (N >= 4 with sum_m bits(I_m) <= 96): the N indices are bit-packed into words
//      0..2 (field f at bit p.boff[f], width from p.bmask[f]; i_n at bit 0) and v is
//      word 3, so N = 4, 5 records stay 16 bytes (the SoA layout streams 4(N+1)).
//   2. Group-contiguous work.  Each tile segment of a CTA's range (the CTA range is
//      nnz-balanced as before) is cut into Gamma = warps x groups equal contiguous
//      sub-ranges, one per lane group; a group walks its sub-range stage by stage, so a
//      run (i_n unchanged) is broken only at a sub-range edge: one flush per run instead
//      of one per 16-nonzero stretch (10x fewer vector atomics on nell-2), and a heavy
//      row gets one atomic per group that touches it (short fp32 atomic chains, F-c).
// Pipeline: per warp, a double-buffered stage holds K records for each of its GPW
// groups; the first lane of every group issues its own bulk copy
// (cp.async.bulk ... mbarrier::complete_tx) after declaring its bytes with
// mbarrier.expect_tx, and lane 0 arrives once all leaders have declared.
// Hot-row cache (SF launch hot_kb): a gathered slot's most frequent rows are
// copied per call into one dense block (hot_fill_kernel); their records carry the row's
// slot in that block with the slot's hot bit set, so the gathers of the hot rows touch a
// compact, TLB- and L2-friendly region instead of rows scattered over the whole factor.
#pragma once

#include "sf_frag.cuh"

#ifndef SF_FRAG_U_WIDE
#define SF_FRAG_U_WIDE 1  // U for N >= 4 at R >= 32: 1 avoids spills (deli-4d +3 %; A/B: -DSF_FRAG_U_WIDE=2)
#endif

namespace sf {

// First position of group gam (of Gam) inside the tile segment [a, a + len).
__host__ __device__ __forceinline__ uint32_t frag3_group_begin(uint32_t a, uint32_t len, uint32_t gam,
                                                               uint32_t Gam) {
  return a + (uint32_t)(((uint64_t)gam * len) / Gam);
}

// CTA c's chunk range [j0, j1): chunks whose first nonzero lies in [c*nnz/G, (c+1)*nnz/G).
__device__ __forceinline__ uint32_t frag3_lower_chunk(const uint32_t* cb, uint32_t num_chunks, uint64_t target) {
  uint32_t lo = 0, hi = num_chunks;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if ((uint64_t)__ldg(cb + mid) < target) lo = mid + 1; else hi = mid;
  }
  return lo;
}

struct Frag3Params {
  const uint32_t* rec;                // kernel-order records (slot order), W words each
  const float* fac[SF_MAX_MODES];     // by mode
  int64_t hot_delta[SF_MAX_MODES];    // per gathered slot: hot block - factor, in float4 units
  uint32_t hot_bit[SF_MAX_MODES];     // per gathered slot: the record's hot flag bit (0 = none)
  float* out;
  const uint32_t* chunk_begin;        // num_chunks + 1
  const uint64_t* chunk_tile;         // num_chunks
  const uint32_t* tile_chunk;         // num_tiles + 1: first chunk of every tile, then num_chunks
  const uint32_t* cta_chunk;          // grid + 1: first chunk of every CTA (frag3_cta_range_kernel)
  uint32_t num_tiles;
  uint32_t num_chunks;
  uint32_t nnz;
  int slot_mode[SF_MAX_MODES];        // gathered slot -> mode (staged slots first)
  uint32_t block_rows[SF_MAX_MODES];  // per staged slot
  uint32_t ntiles[SF_MAX_MODES];      // per staged slot
  uint32_t dims[SF_MAX_MODES];        // per mode
  uint32_t fac_off[SF_MAX_MODES];     // per staged slot: float offset of its block in smem
  uint32_t K;                         // records per group per stage
  uint32_t W;                         // words per record (== RecWords<N, PK>::W)
  uint32_t boff[SF_MAX_MODES];        // PK: bit offset of field f (slot order, f = 0 is i_n)
  uint32_t bmask[SF_MAX_MODES];       // PK: (1 << width) - 1 of field f
  uint32_t out_mask;                  // mask applied to word 0 to read i_n (PK: bmask[0])
  uint32_t owner;                     // A5: unstaged plans store whole runs, zero gaps (no memset)
  uint32_t l2tiles;                   // SF_LAUNCH_L2_TILES: every CTA takes 1/grid of every tile, in tile
                                      // order (S == 0: the tiled modes are gathered from L2)
  // A7 deterministic option (owner mode only): shared runs go to per-group carry slots
  // (head = 2*gid, tail = 2*gid+1, gid = blockIdx.x * groups + group) instead of atomics;
  // frag3_combine_kernel then adds them per row in slot order.
  uint32_t* carry_row;                // [2 * grid * groups], 0xFFFFFFFF = empty (memset per launch)
  float* carry_val;                   // [2 * grid * groups * R]
};

namespace detail {
__device__ __forceinline__ void mbar_expect_tx_only(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(su32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(bar)) : "memory");
}
__device__ __forceinline__ uint4 lds128(const uint32_t* p) { return *reinterpret_cast<const uint4*>(p); }
}  // namespace detail

// Field f of a packed record (words w0..w2): bits [off, off + width) -- a field never
// spans more than two consecutive words (width <= 32).
__device__ __forceinline__ uint32_t pk_field(uint32_t w0, uint32_t w1, uint32_t w2, uint32_t off, uint32_t mask) {
  const uint32_t wi = off >> 5, sh = off & 31u;
  const uint32_t lo = wi == 0 ? w0 : (wi == 1 ? w1 : w2);
  const uint32_t hi = wi == 0 ? w1 : (wi == 1 ? w2 : 0u);
  return __funnelshift_r(lo, hi, sh) & mask;
}

// Record formats (RF): kRecPlain [i_n, g_0 .. g_{N-2}, v, 0..] (W = 4 or 8); kRecPacked
// (N >= 4: N bit fields in words 0..2, v in word 3).  (8-byte compact records with run
// deltas were measured 9 % slower on nell-2 and removed.)
constexpr int kRecPlain = 0, kRecPacked = 1;

// HOT: the plan has a hot-row cache (the per-gather select is compiled only into these
// instantiations: on L2-resident plans it cost 5 %, nell-2 0.767 vs 0.729 ms per mode).
template <int N, int R, int S, int RF, bool HOT>
__global__ void __launch_bounds__(1024) frag3_kernel(const Frag3Params p) {
  using namespace detail;
  using LM = LaneMap<R>;
  constexpr int VEC = LM::VEC;
  constexpr int LPN = LM::LPN;  // lanes per nonzero
  constexpr int GPW = 32 / LPN; // lane groups per warp
  constexpr int G = N - 1;      // gathered slots
  constexpr bool PK = RF == kRecPacked;
  constexpr int W = PK ? 4 : RecWords<N>::W;
  static_assert(!PK || N >= 4, "packed records are for N >= 4");
  constexpr int RB = R * 4;     // bytes per factor row
  constexpr int R4 = R / 4;     // float4 per factor row
  // batch of nonzeros in flight per lane group (register budget: 64 at 1024 threads)
  constexpr int U = (VEC == 8) ? (N >= 4 ? SF_FRAG_U_WIDE : 2) : kFragUnroll;
  extern __shared__ __align__(128) unsigned char smem_raw[];

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & 31;
  const int nwarps = blockDim.x >> 5;
  const int lane_in_group = lane % LPN;
  const int group = lane / LPN;
  const int c0 = (VEC == 8) ? 2 * lane_in_group : lane_in_group;  // first owned 16-B chunk
  const int par = (lane >> 2) & 1;                                 // smem issue order (VEC 8)
  const bool leader = lane_in_group == 0;

  const uint32_t K = p.K;
  const uint32_t RS = frag3_region_words(K, W);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw);
  const uint32_t bar_bytes = ((2u * nwarps + 1u) * 8u + 127u) & ~127u;
  uint32_t* ring = reinterpret_cast<uint32_t*>(smem_raw + bar_bytes) + (size_t)warp * kFragStages * GPW * RS;
  float* fac_smem = reinterpret_cast<float*>(smem_raw + bar_bytes) + (size_t)nwarps * kFragStages * GPW * RS;
  uint64_t* wbar = bars + 2 * warp;
  uint64_t* fbar = bars + 2 * nwarps;

  const uint64_t grid = gridDim.x;
  // CTA range: nnz-balanced chunks [j0, j1) of the plan order, or (L2 tiles) every chunk,
  // of which each tile segment contributes its blockIdx.x-th 1/grid share.
  const bool l2t = (S == 0) && p.l2tiles;
  const uint32_t j0 = l2t ? 0u : __ldg(p.cta_chunk + blockIdx.x);
  const uint32_t j1 = l2t ? p.num_chunks : __ldg(p.cta_chunk + blockIdx.x + 1);
  if (j0 >= j1) return;
  // tile of chunk j0 (tiles are walked by index from there: no per-segment search)
  uint32_t ti = 0;
  if (S > 0 || l2t) {
    uint32_t lo = 0, hi = p.num_tiles;  // last tile with tile_chunk <= j0
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (__ldg(p.tile_chunk + mid) <= j0) lo = mid; else hi = mid;
    }
    ti = lo;
  }

  if (lane == 0) {
    mbar_init(&wbar[0], 1);
    mbar_init(&wbar[1], 1);
    if (warp == 0) mbar_init(fbar, 1);
    fence_barrier_init();
  }
  __syncthreads();

  const uint32_t Gam = (uint32_t)nwarps * GPW;
  const uint32_t gam = (uint32_t)warp * GPW + group;

  const float4* sbase[S > 0 ? S : 1];
  const float4* gbase[G - S > 0 ? G - S : 1];
#pragma unroll
  for (int q = S; q < G; ++q) gbase[q - S] = reinterpret_cast<const float4*>(p.fac[p.slot_mode[q]]);
  uint32_t fac_phase = 0;
  uint32_t it = 0;  // stages this warp has consumed (stage = it % 2, parity = (it / 2) & 1)
  float* const out0 = p.out + 4 * c0;
  float* const out1 = out0 + 4;

  uint32_t seg = j0;
  while (seg < j1) {
    uint32_t seg_end = j1;
    if (S > 0 || l2t) {  // this tile's chunks inside [seg, j1)
      seg_end = min(j1, __ldg(p.tile_chunk + ti + 1));
      ++ti;
    }
    if constexpr (S > 0) {
      const uint64_t tile = __ldg(p.chunk_tile + seg);
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
    // this group's sub-range [gs, ge) of the tile segment [a, b)
    uint32_t a = __ldg(p.chunk_begin + seg), b = __ldg(p.chunk_begin + seg_end);
    if (l2t) {  // this CTA's share of the tile
      const uint32_t len = b - a;
      b = a + (uint32_t)(((uint64_t)(blockIdx.x + 1) * len) / grid);
      a = a + (uint32_t)(((uint64_t)blockIdx.x * len) / grid);
    }
    const uint32_t gs = frag3_group_begin(a, b - a, gam, Gam);
    const uint32_t ge = frag3_group_begin(a, b - a, gam + 1, Gam);
    const uint32_t T = (__reduce_max_sync(0xFFFFFFFFu, ge - gs) + K - 1) / K;  // stages of this warp
    uint32_t* const my_region0 = ring + (size_t)group * RS;

    // stage t of this warp into ring slot st: every group leader copies its own records
    auto issue = [&](uint32_t t, int st) {
      if (leader) {
        const uint32_t s0 = gs + t * K;
        if (s0 < ge) {
          const uint32_t first = s0, cnt = min(K, ge - s0);
          const uint32_t bytes = cnt * (uint32_t)(W * 4);
          mbar_expect_tx_only(&wbar[st], bytes);
          bulk_g2s(my_region0 + (size_t)st * GPW * RS, p.rec + (size_t)first * W, bytes, &wbar[st]);
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&wbar[st]);
    };
    if (T > 0) issue(0, it % kFragStages);
    if (T > 1) issue(1, (it + 1) % kFragStages);

    // A5 owner bookkeeping from the neighbouring records (global, one-time per sub-range)
    bool first_shared = true, last_shared = true;
    uint32_t before = 0xFFFFFFFFu;
    if constexpr (S == 0) {
      if (p.owner && gs < ge) {
        const uint32_t om = p.out_mask;
        before = (gs > 0) ? (__ldg(p.rec + (size_t)(gs - 1) * W) & om) : 0xFFFFFFFFu;
        const uint32_t first_g = __ldg(p.rec + (size_t)gs * W) & om;
        first_shared = (gs > 0) && before == first_g;
        last_shared = (ge < p.nnz) &&
                      (__ldg(p.rec + (size_t)ge * W) & om) == (__ldg(p.rec + (size_t)(ge - 1) * W) & om);
      }
    }
    if constexpr (S > 0) {
      mbar_wait(fbar, fac_phase);
      fac_phase ^= 1u;
    }

    bool shared = first_shared;
    uint32_t cur = 0;
    float4 acc0 = make_float4(0.f, 0.f, 0.f, 0.f), acc1 = acc0;
    auto gather = [&](int q, uint32_t row_idx) -> F8 {
      const float4* base = (q < S) ? sbase[q < S ? q : 0] : gbase[q >= S ? q - S : 0];
      size_t row = (size_t)row_idx * R4;
      if (HOT && q >= S) {  // hot-row cache: the slot inside the dense hot block
        const uint32_t hb = p.hot_bit[q];
        if (row_idx & hb) row = (size_t)((int64_t)(row_idx & ~hb) * R4 + p.hot_delta[q]);
      }
      F8 r;
      if constexpr (VEC == 8) {
        if (q < S) {
          const float4 x = base[row + c0 + par];
          const float4 y = base[row + c0 + 1 - par];
          r.a = par ? y : x;
          r.b = par ? x : y;
        } else {
          if constexpr (HOT) ldg256_l1(base + row + c0, r.a, r.b);
          else ldg256_na(base + row + c0, r.a, r.b);
        }
      } else {
        r.a = (q < S) ? base[row + c0] : ldg128(base + row + c0);
      }
      return r;
    };
    bool advanced = false;  // the first run of the sub-range has been closed
    auto flush_run = [&](bool atomic) {
      if (atomic && p.carry_row) {  // deterministic: park the partial in this group's slot
        const size_t slot = 2 * ((size_t)blockIdx.x * Gam + gam) + (advanced ? 1 : 0);
        if (lane_in_group == 0) p.carry_row[slot] = cur;
        float* dst = p.carry_val + slot * R + 4 * c0;
        if constexpr (VEC == 8) st256(dst, acc0, acc1);
        else st128(dst, acc0);
      } else if (atomic) {
        red_add_v4_nomem(out0 + (size_t)cur * R, acc0);
        if constexpr (VEC == 8) red_add_v4_nomem(out1 + (size_t)cur * R, acc1);
      } else {
        if constexpr (VEC == 8) st256(out0 + (size_t)cur * R, acc0, acc1);
        else st128(out0 + (size_t)cur * R, acc0);
      }
      acc0 = make_float4(0.f, 0.f, 0.f, 0.f);
      acc1 = acc0;
    };
    auto zero_rows = [&](uint32_t r0, uint32_t r1) {  // rows (r0, r1) exclusive
      for (uint32_t r = r0 + 1; r < r1; ++r) {
        if constexpr (VEC == 8) st256(out0 + (size_t)r * R, make_float4(0.f, 0.f, 0.f, 0.f),
                                             make_float4(0.f, 0.f, 0.f, 0.f));
        else st128(out0 + (size_t)r * R, make_float4(0.f, 0.f, 0.f, 0.f));
      }
    };
    auto advance = [&](uint32_t i) {  // run edge inside the sub-range: close `cur`, open i
      flush_run(shared);
      advanced = true;
      if constexpr (S == 0) {
        if (p.owner) {
          zero_rows(cur, i);
          shared = false;
        }
      }
      cur = i;
    };

    for (uint32_t t = 0; t < T; ++t, ++it) {
      const int st = (int)(it % kFragStages);
      mbar_wait(&wbar[st], (it / kFragStages) & 1u);
      const uint32_t* reg = my_region0 + (size_t)st * GPW * RS;
      const uint32_t s0 = gs + t * K;
      const uint32_t n = (s0 < ge) ? min(K, ge - s0) : 0u;
      if (n > 0) {
        if (t == 0) {  // open the sub-range's first run
          cur = reg[0] & p.out_mask;
          if constexpr (S == 0) {
            if (p.owner && !first_shared && gs > 0) zero_rows(before, cur);  // gap rows are ours
          }
        }
        // record k of this group: [i_n, g_0 .. g_{G-1}, v]
        auto load_rec = [&](uint32_t k, uint32_t& i, uint32_t (&g)[G], float& v) {
          const uint32_t* rp = reg + (size_t)k * W;
          const uint4 w0 = lds128(rp);
          uint32_t w[W];
          w[0] = w0.x; w[1] = w0.y; w[2] = w0.z; w[3] = w0.w;
          if constexpr (W == 8) {
            const uint4 w1 = lds128(rp + 4);
            w[4] = w1.x; w[5] = w1.y; w[6] = w1.z; w[7] = w1.w;
          }
          if constexpr (PK) {
            i = w[0] & p.out_mask;  // i_n at bit 0
#pragma unroll
            for (int q = 0; q < G; ++q) g[q] = pk_field(w[0], w[1], w[2], p.boff[1 + q], p.bmask[1 + q]);
            v = __uint_as_float(w[3]);
          } else {
            i = w[0];
#pragma unroll
            for (int q = 0; q < G; ++q) g[q] = w[1 + q];
            v = __uint_as_float(w[N]);
          }
        };
        uint32_t k = 0;
        for (; k + U <= n; k += U) {
          uint32_t ii[U], gi[U][G];
          float vv[U];
          F8 pr[U];
#pragma unroll
          for (int u = 0; u < U; ++u) load_rec(k + u, ii[u], gi[u], vv[u]);
#pragma unroll
          for (int q = 0; q < G; ++q) {
#pragma unroll
            for (int u = 0; u < U; ++u) {
              const F8 x = gather(q, gi[u][q]);
              if (q == 0) {
                pr[u] = x;
              } else {
                f4mul_(pr[u].a, x.a);
                if constexpr (VEC == 8) f4mul_(pr[u].b, x.b);
              }
            }
          }
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (ii[u] != cur) advance(ii[u]);
            const float4 vb = make_float4(vv[u], vv[u], vv[u], vv[u]);
            f4fma_(acc0, vb, pr[u].a);
            if constexpr (VEC == 8) f4fma_(acc1, vb, pr[u].b);
          }
        }
        for (; k < n; ++k) {
          uint32_t i, gi[G];
          float v;
          load_rec(k, i, gi, v);
          F8 pr = gather(0, gi[0]);
#pragma unroll
          for (int q = 1; q < G; ++q) {
            const F8 x = gather(q, gi[q]);
            f4mul_(pr.a, x.a);
            if constexpr (VEC == 8) f4mul_(pr.b, x.b);
          }
          if (i != cur) advance(i);
          const float4 vb = make_float4(v, v, v, v);
          f4fma_(acc0, vb, pr.a);
          if constexpr (VEC == 8) f4fma_(acc1, vb, pr.b);
        }
      }
      __syncwarp();  // every lane is done reading stage st
      if (t + 2u < T) issue(t + 2u, st);
    }
    if (gs < ge) flush_run(shared || last_shared);  // the sub-range's last run
    seg = seg_end;
  }
}

// A5 pre-pass for owner mode: zero the rows whose run crosses a group sub-range start
// (they receive atomic partial sums).  One thread per (CTA, group) of the frag3 launch.
// CTA c's chunk range [cta_chunk[c], cta_chunk[c+1]): chunks whose first nonzero lies in
// [c*nnz/G, (c+1)*nnz/G), computed once per (plan, grid) instead of by every CTA.
static __global__ void frag3_cta_range_kernel(const uint32_t* __restrict__ cb, uint32_t num_chunks, uint32_t nnz,
                                              uint32_t ctas, uint32_t* __restrict__ cta_chunk) {
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c <= ctas; c += gridDim.x * blockDim.x)
    cta_chunk[c] = frag3_lower_chunk(cb, num_chunks, ((uint64_t)c * nnz) / ctas);
}

template <int R>
__global__ void boundary_zero3_kernel(const uint32_t* __restrict__ chunk_begin, const uint32_t* __restrict__ cta_chunk,
                                      uint32_t ctas, uint32_t groups_per_cta,
                                      const uint32_t* __restrict__ rec, uint32_t W, uint32_t om,
                                      float* __restrict__ out) {
  const uint64_t total = (uint64_t)ctas * groups_per_cta;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
    const uint32_t c = (uint32_t)(t / groups_per_cta), gam = (uint32_t)(t % groups_per_cta);
    const uint32_t j0 = cta_chunk[c];
    const uint32_t j1 = cta_chunk[c + 1];
    if (j0 >= j1) continue;
    const uint32_t a = chunk_begin[j0], b = chunk_begin[j1];
    const uint32_t pos = frag3_group_begin(a, b - a, gam, groups_per_cta);
    const uint32_t end = frag3_group_begin(a, b - a, gam + 1, groups_per_cta);
    if (pos >= end || pos == 0) continue;
    const uint32_t r = rec[(size_t)pos * W] & om;
    if ((rec[(size_t)(pos - 1) * W] & om) != r) continue;
    float4* y = reinterpret_cast<float4*>(out + (size_t)r * R);
#pragma unroll
    for (int q = 0; q < R / 4; ++q) y[q] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
}

// A7 deterministic combine: one warp per carry slot; the first non-empty slot of a row
// sums that row's slots in slot order (= nonzero order) and stores the row.
static __global__ void frag3_combine_kernel(const uint32_t* __restrict__ carry_row, const float* __restrict__ carry_val,
                                     uint64_t nslots, int R, float* __restrict__ out) {
  const uint64_t warps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  const int lane = threadIdx.x & 31;
  for (uint64_t k = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < nslots; k += warps) {
    const uint32_t r = carry_row[k];
    if (r == 0xFFFFFFFFu) continue;
    uint64_t prev = k;
    uint32_t pr = 0xFFFFFFFFu;
    while (prev > 0) {
      pr = carry_row[--prev];
      if (pr != 0xFFFFFFFFu) break;
    }
    if (pr == r) continue;  // not the first slot of row r
    for (int c = lane; c < R; c += 32) {
      float sum = 0.f;
      for (uint64_t q = k; q < nslots; ++q) {
        const uint32_t rq = carry_row[q];
        if (rq == 0xFFFFFFFFu) continue;
        if (rq != r) break;
        sum += carry_val[q * R + c];
      }
      out[(size_t)r * R + c] = sum;
    }
  }
}

void frag3_launch_r16(int N, int S, const Frag3Params& fp, int grid, int threads, size_t smem, cudaStream_t s);
void frag3_launch_r32(int N, int S, const Frag3Params& fp, int grid, int threads, size_t smem, cudaStream_t s);
void frag3_launch_r64(int N, int S, const Frag3Params& fp, int grid, int threads, size_t smem, cudaStream_t s);
int frag3_occ_r16(int N, int S, int threads, size_t smem, bool hot);
int frag3_occ_r32(int N, int S, int threads, size_t smem, bool hot);
int frag3_occ_r64(int N, int S, int threads, size_t smem, bool hot);
void boundary_zero3_r16(const Frag3Params& fp, uint32_t ctas, uint32_t groups, float* out, cudaStream_t s);
void boundary_zero3_r32(const Frag3Params& fp, uint32_t ctas, uint32_t groups, float* out, cudaStream_t s);
void boundary_zero3_r64(const Frag3Params& fp, uint32_t ctas, uint32_t groups, float* out, cudaStream_t s);

// Dynamic shared memory opted in per (device, instantiation, variant v = record format +
// 2 * HOT): only ever RAISED (the occupancy query and the launch share it; lowering the
// attribute for a smaller plan would make a later launch of a larger plan fail with
// "invalid argument").
template <int N, int R, int S>
size_t& frag3_smem_optin(int dev, int v) {
  static size_t set[16][4] = {};
  static size_t spill = 0;
  return (dev < 16 && v < 4) ? set[dev][v] : spill;
}

template <int N, int R, int S, class K>
void frag3_ensure_smem(K k, int v, size_t smem) {
  int dev = 0;
  SF_CUDA(cudaGetDevice(&dev));
  size_t& cur = frag3_smem_optin<N, R, S>(dev, v);
  if (dev >= 16 || smem > cur) {
    SF_CUDA(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    if (dev < 16) cur = smem;
  }
}

// The instantiation a plan runs: record format from fp.W, HOT when a gathered slot has hot
// rows (never when every gathered slot is staged in shared memory).
template <int N, int R, int S>
void (*frag3_pick(bool packed, bool hot, int* v))(const Frag3Params) {
  constexpr bool kHotPossible = S < N - 1;
  void (*k)(const Frag3Params) = frag3_kernel<N, R, S, kRecPlain, false>;
  *v = 0;
  if constexpr (kHotPossible) {
    if (hot) {
      k = frag3_kernel<N, R, S, kRecPlain, true>;
      *v = 2;
    }
  }
  if constexpr (N >= 4) {
    if (packed) {
      k = frag3_kernel<N, R, S, kRecPacked, false>;
      *v = 1;
      if constexpr (kHotPossible) {
        if (hot) {
          k = frag3_kernel<N, R, S, kRecPacked, true>;
          *v = 3;
        }
      }
    }
  }
  return k;
}

template <int N, int R, int S>
void frag3_launch_one(const Frag3Params& fp, int grid, int threads, size_t smem, cudaStream_t s) {
  bool hot = false;
  for (int q = 0; q < SF_MAX_MODES; ++q) hot = hot || fp.hot_bit[q] != 0;
  int v = 0;
  auto k = frag3_pick<N, R, S>(fp.W == 4 && N >= 4, hot, &v);
  frag3_ensure_smem<N, R, S>(k, v, smem);
  k<<<grid, threads, smem, s>>>(fp);
}

template <int N, int R, int S>
int frag3_occ_one(int threads, size_t smem, bool hot) {
  int v = 0;
  auto k = frag3_pick<N, R, S>(false, hot, &v);
  frag3_ensure_smem<N, R, S>(k, v, smem);
  int nb = 0;
  SF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k, threads, smem));
  return nb;
}

#define SF_DEFINE_FRAG3_R(R)                                                                             \
  void frag3_launch_r##R(int N, int S, const Frag3Params& fp, int grid, int threads, size_t smem,        \
                         cudaStream_t s) {                                                               \
    SF_FRAG_NS_SWITCH(R, frag3_launch_one, fp, grid, threads, smem, s);                                  \
    throw StatusError{SF_ERR_UNSUPPORTED, "frag3 kernel: unsupported (N, S)"};                          \
  }                                                                                                      \
  int frag3_occ_r##R(int N, int S, int threads, size_t smem, bool hot) {                                 \
    SF_FRAG_NS_SWITCH(R, frag3_occ_one, threads, smem, hot);                                             \
    return 0;                                                                                            \
  }                                                                                                      \
  void boundary_zero3_r##R(const Frag3Params& fp, uint32_t ctas, uint32_t groups, float* out,           \
                           cudaStream_t s) {                                                             \
    const uint64_t total = (uint64_t)ctas * groups;                                                      \
    const int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>((total + 255) / 256, 148 * 16));     \
    boundary_zero3_kernel<R><<<grid, 256, 0, s>>>(fp.chunk_begin, fp.cta_chunk, ctas, groups,           \
                                                  fp.rec, fp.W, fp.out_mask, out);      \
  }

}  // namespace sf
