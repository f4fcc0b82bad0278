// sf_plan.cu - device-side preprocessing (§8(a) A2-A4): integer-exact.
//
// "ScalFrag first matricizes the input tensor and then chunks the
// matricized tensor ... uses a trained model to select the best combination of
// launch parameters based on the sparsity features of the matrixed tensor after
// chunking."  Here, per (mode n, rank):
//   1. matricized order: stable LSD radix sort of the key i_n * I_s + i_s with the
//      input position as payload (s = smallest gathered mode; reading R10), or
//      the merge of the segment runs sorted during the upload (presort);
//   2. features from run lengths of that order (run_stats_kernel);
//   3. shard cut [floor(p*nnz/P), floor((p+1)*nnz/P)) of that order (§8(e));
//   4. tiles ("tensor blocks ... based on the resource constraints of hardware",
//      PAPER.md L34): a second stable sort by tile id -> order (tile, i_n, i_s, pos);
//   5. the hot-row cache: row counts, one global threshold, slots and the index map;
//   6. gather the kernel-order records from the AoS copy (COO-kernel plans: SoA arrays);
//   7. chunks ("segments"): a new chunk at every tile start and every
//      C nonzeros inside a tile.
// All of it is integer work; tests compare it == against oracle/plan.py.
#include <cub/cub.cuh>

#include <cub/device/device_merge.cuh>

#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "sf_internal.h"


namespace sf {

static inline int bitlen(uint64_t x) {
  int b = 0;
  while (x) { ++b; x >>= 1; }
  return b;
}

static inline int grid_for(uint64_t n, int threads = 256) {
  return (int)std::max<uint64_t>(1, std::min<uint64_t>((n + threads - 1) / threads, 148ull * 32));
}

// x / d for a divisor fixed per launch (d < 2^32): the quotient estimate hi64(x * m),
// m = floor((2^64 - 1) / d), is at most 2 below floor(x / d); two corrections make it exact.
// (A 64-bit `/` compiles to a ~70-instruction software routine.)
struct Div64 {
  uint64_t d, m;
  explicit Div64(uint64_t d_) : d(d_), m(~0ull / d_) {}
  __device__ __forceinline__ uint64_t div(uint64_t x) const {
    uint64_t q = __umul64hi(x, m);
    uint64_t r = x - q * d;
    if (r >= d) { ++q; r -= d; }
    if (r >= d) ++q;
    return q;
  }
};

// ---------------------------------------------------------------------------
// key = i_n * I_s + i_s; with `io`, the bits of (i_o >> kCarryShift) ride above bit kb (the
// sort covers bits [0, kb) only, so they travel with the key unsorted: tile ids of the other
// gathered mode without a random gather later, tile_key_from_carry_kernel)
constexpr int kCarryShift = 17;
__global__ void key_matricized_kernel(const uint32_t* __restrict__ in, const uint32_t* __restrict__ is,
                                      uint64_t Is, uint64_t n, uint64_t* __restrict__ key,
                                      uint32_t* __restrict__ pos, const uint32_t* __restrict__ io = nullptr,
                                      int kb = 0) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += stride) {
    uint64_t k = (uint64_t)in[e] * Is + (uint64_t)is[e];
    if (io) k |= (uint64_t)(io[e] >> kCarryShift) << kb;
    key[e] = k;
    pos[e] = (uint32_t)e;
  }
}

struct FeatAcc {
  unsigned long long max_slice, max_fiber, sum_sq;
  unsigned long long hist[SF_HIST_BINS];
};


// ---------------------------------------------------------------------------
// A8 upload || presort.  Composite key c = (i_n * I_s + i_s) << pb | e (e = input position,
// pb = bits(nnz - 1)) is unique, so sorting / merging c is the stable matricized sort.
static inline int key_bits(const Tensor& t, int mode) {
  const int s = secondary_mode(t, mode);
  return std::max(1, bitlen(t.dims[mode] * t.dims[s] - 1));
}

__global__ void compose_key_kernel(const uint32_t* __restrict__ in, const uint32_t* __restrict__ is, uint64_t Is,
                                   uint64_t a, uint64_t len, int pb, uint64_t* __restrict__ out) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < len; e += stride)
    out[e] = (((uint64_t)in[e] * Is + (uint64_t)is[e]) << pb) | (a + e);
}

__global__ void split_key_kernel(const uint64_t* __restrict__ c, uint64_t n, int pb, uint64_t* __restrict__ key,
                                 uint32_t* __restrict__ pos) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t mask = (1ull << pb) - 1ull;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += stride) {
    const uint64_t x = c[e];
    key[e] = x >> pb;
    pos[e] = (uint32_t)(x & mask);
  }
}

static void aos_segment(Tensor& t, uint64_t a, uint64_t len, cudaStream_t st);  // below

bool presort_begin(Tensor& t, uint64_t seg_len) {
  if (debug_opt("no_presort")) return false;  // SF_DEBUG A/B
  const uint64_t n = t.nnz;
  if (n < 2 || seg_len >= n || n >= (1ull << 30)) return false;
  const int pb = std::max(1, bitlen(n - 1));
  // Modes whose key and position need more than 64 bits are not presorted: (key, position)
  // pair runs merged with a pair comparison were measured slower end to end on nell-1 (the
  // per-segment pair sorts lengthen the upload more than the merge saves)
  int modes = 0;
  for (int m = 0; m < t.nmodes; ++m) modes += (key_bits(t, m) + pb <= 64);
  if (!modes) return false;
  const size_t free_b = device_free_bytes();
  // pre keys + the segment staging buffer now, and a merge buffer + split keys/positions later
  if ((double)n * 8.0 * (modes + 4) > 0.6 * (double)free_b) return false;
  t.pre_pb = pb;
  t.pre_seg_len = seg_len;
  for (int m = 0; m < t.nmodes; ++m) {
    t.have_pre[m] = key_bits(t, m) + pb <= 64;
    if (t.have_pre[m]) t.pre[m].alloc(n * 8 + 16);
  }
  t.pre_alt.alloc(n * 8 + 16);
  const int WR = (t.nmodes + 1 <= 4) ? 4 : (t.nmodes + 1 <= 8 ? 8 : 16);
  t.aos.alloc((size_t)n * WR * 4 + 64);  // the AoS copy is built per segment too
  t.aos_words = WR;
  return true;
}

size_t presort_temp_bytes(const Tensor& t, uint64_t seg_len) {
  size_t b = 0;
  SF_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, b, (const uint64_t*)nullptr, (uint64_t*)nullptr, (int64_t)seg_len,
                                         0, 64, (cudaStream_t)0));
  (void)t;
  return b;
}

void presort_segment(Tensor& t, uint64_t a, uint64_t len, cudaStream_t st, void* temp, size_t temp_bytes) {
  aos_segment(t, a, len, st);
  for (int m = 0; m < t.nmodes; ++m) {
    if (!t.have_pre[m]) continue;
    const int s = secondary_mode(t, m);
    uint64_t* alt = t.pre_alt.as<uint64_t>() + a;
    compose_key_kernel<<<grid_for(len), 256, 0, st>>>(t.ind[m].as<uint32_t>() + a, t.ind[s].as<uint32_t>() + a,
                                                      t.dims[s], a, len, t.pre_pb, alt);
    // the position bits are already ascending inside the segment and LSD radix sorting is
    // stable: sorting only the key bits [pb, pb + kb) orders the composites completely
    size_t tb = temp_bytes;
    SF_CUDA(cub::DeviceRadixSort::SortKeys(temp, tb, alt, t.pre[m].as<uint64_t>() + a, (int64_t)len, t.pre_pb,
                                           t.pre_pb + key_bits(t, m), st));
    count_launch(1 + (uint64_t)((key_bits(t, m) + 7) / 8) * 3);
  }
  SF_CUDA(cudaGetLastError());
}

// cnt[x] += #{k < n : ind[perm ? perm[k] : k] == x}, indices >= dim skipped (not yet validated
// during the upload).  Up to kSmemCountRows rows: a per-block shared-memory histogram flushed
// once per block; more: warp-aggregated atomics (the lanes holding the same row add once), as
// skewed (Zipf) rows would otherwise serialise on a few addresses.
constexpr uint64_t kSmemCountRows = 12288;
__global__ void row_count_kernel(const uint32_t* __restrict__ ind, const uint32_t* __restrict__ perm, uint64_t n,
                                 uint64_t dim, uint32_t* __restrict__ cnt) {
  extern __shared__ uint32_t hist[];
  const bool small = dim <= kSmemCountRows;
  if (small) {
    for (uint64_t i = threadIdx.x; i < dim; i += blockDim.x) hist[i] = 0;
    __syncthreads();
  }
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  if (small) {
    for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += stride) {
      const uint32_t x = __ldg(ind + (perm ? __ldg(perm + k) : k));
      if (x < dim) atomicAdd(hist + x, 1u);
    }
  } else {
    // warp-uniform trip count, so every lane takes part in the match
    const uint64_t k0 = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
    for (uint64_t kw = k0; kw < n; kw += stride) {
      const uint64_t k = kw + (threadIdx.x & 31u);
      const uint32_t x = (k < n) ? __ldg(ind + (perm ? __ldg(perm + k) : k)) : 0xffffffffu;
      const unsigned peers = __match_any_sync(0xffffffffu, x);
      if (x < dim && (threadIdx.x & 31u) == (unsigned)(__ffs(peers) - 1)) atomicAdd(cnt + x, (uint32_t)__popc(peers));
    }
  }
  if (small) {
    __syncthreads();
    for (uint64_t i = threadIdx.x; i < dim; i += blockDim.x)
      if (hist[i]) atomicAdd(cnt + i, hist[i]);
  }
}

static void count_rows(const uint32_t* ind, const uint32_t* perm, uint64_t n, uint64_t dim, uint32_t* cnt,
                       cudaStream_t st) {
  if (!n) return;
  const bool small = dim <= kSmemCountRows;
  row_count_kernel<<<small ? std::min(grid_for(n), 148 * 4) : grid_for(n), 256, small ? dim * 4 : 0, st>>>(
      ind, perm, n, dim, cnt);
  count_launch();
  SF_CUDA(cudaGetLastError());
}

Ingest ingest_begin(Tensor& t) {
  Ingest g;
  const uint64_t n = t.nnz;
  if (!n) return g;
  const int N = t.nmodes;
  const int WR = (N + 1 <= 4) ? 4 : (N + 1 <= 8 ? 8 : 16);
  uint64_t need = t.aos.p ? 0 : n * WR * 4;
  uint32_t mask = 0;
  for (int m = 0; m < N; ++m)
    if (t.dims[m] >= (1ull << 18) && t.dims[m] < (1ull << 31) && !t.hot_cnt[m].p) {
      mask |= 1u << m;
      need += t.dims[m] * 4;
    }
  const size_t free_b = device_free_bytes();
  if ((double)need > 0.4 * (double)free_b) return g;  // leave it to the first plan
  if (!t.aos.p) {
    t.aos.alloc((size_t)n * WR * 4 + 64);
    t.aos_words = WR;
    g.aos = true;
  }
  for (int m = 0; m < N; ++m)
    if (mask >> m & 1) {
      t.hot_cnt[m].alloc(t.dims[m] * 4 + 16);
      SF_CUDA(cudaMemsetAsync(t.hot_cnt[m].p, 0, t.dims[m] * 4, t.stream));
    }
  g.cnt_mask = mask;
  SF_CUDA(cudaStreamSynchronize(t.stream));  // the segment streams count into zeroed arrays
  return g;
}

void ingest_segment(Tensor& t, const Ingest& g, uint64_t a, uint64_t len, cudaStream_t st) {
  if (g.aos) aos_segment(t, a, len, st);
  for (int m = 0; m < t.nmodes; ++m)
    if (g.cnt_mask >> m & 1) {
      count_rows(t.ind[m].as<uint32_t>() + a, nullptr, len, t.dims[m], t.hot_cnt[m].as<uint32_t>(), st);
    }
  SF_CUDA(cudaGetLastError());
}

// Merge the sorted segment runs of mode `mode` (pairwise, log2(#runs) rounds) and split the
// composite keys into the matricized keys + input positions.
static void presort_finish(Tensor& t, int mode, DevBuf& keys_out, DevBuf& pos_out) {
  const uint64_t n = t.nnz;
  DevBuf cur = std::move(t.pre[mode]);
  t.have_pre[mode] = false;
  DevBuf nxt(n * 8 + 16), tmp;
  size_t tmp_bytes = 0;
  for (uint64_t L = t.pre_seg_len; L < n; L *= 2) {
    for (uint64_t a = 0; a < n; a += 2 * L) {
      const uint64_t b = std::min(n, a + L), c = std::min(n, a + 2 * L);
      if (b >= c) {  // odd run out: carried over
        d2d_copy(nxt.as<uint64_t>() + a, cur.as<uint64_t>() + a, (b - a) * 8, t.stream);
        continue;
      }
      size_t need = 0;
      SF_CUDA(cub::DeviceMerge::MergeKeys(nullptr, need, cur.as<uint64_t>() + a, (int)(b - a),
                                          cur.as<uint64_t>() + b, (int)(c - b), nxt.as<uint64_t>() + a,
                                          cuda::std::less<uint64_t>{}, t.stream));
      if (need > tmp_bytes) {
        tmp.alloc(need + 16);
        tmp_bytes = need;
      }
      SF_CUDA(cub::DeviceMerge::MergeKeys(tmp.p, need, cur.as<uint64_t>() + a, (int)(b - a),
                                          cur.as<uint64_t>() + b, (int)(c - b), nxt.as<uint64_t>() + a,
                                          cuda::std::less<uint64_t>{}, t.stream));
      count_launch(2);
    }
    std::swap(cur, nxt);
  }
  keys_out = std::move(nxt);  // n * 8 bytes, reused for the split keys
  pos_out.alloc(n * 4 + 16);
  split_key_kernel<<<grid_for(n), 256, 0, t.stream>>>(cur.as<uint64_t>(), n, t.pre_pb, keys_out.as<uint64_t>(),
                                                      pos_out.as<uint32_t>());
  count_launch();
  SF_CUDA(cudaGetLastError());
}

// Matricized sort of the whole tensor for `mode`. Returns sorted keys + positions.
static void matricized_sort(Tensor& t, int mode, DevBuf& keys_out, DevBuf& pos_out) {
  t.carry_kb[mode] = 0;
  if (t.have_pre[mode]) return presort_finish(t, mode, keys_out, pos_out);
  const uint64_t n = t.nnz;
  const int s = secondary_mode(t, mode);
  const uint64_t Is = t.dims[s];
  const int end_bit = std::max(1, bitlen(t.dims[mode] * Is - 1));
  // 3-way: carry the other gathered mode's coarse index when it fits above the key bits
  const uint32_t* io = nullptr;
  if (t.nmodes == 3) {
    const int o = 3 - mode - s;
    const int cb = bitlen((t.dims[o] - 1) >> kCarryShift);
    if (cb > 0 && end_bit + cb <= 64) {
      io = t.ind[o].as<uint32_t>();
      t.carry_kb[mode] = end_bit;
    }
  }
  DevBuf k0(n * 8 + 16), k1(n * 8 + 16), p0(n * 4 + 16), p1(n * 4 + 16);
  key_matricized_kernel<<<grid_for(n), 256, 0, t.stream>>>(t.ind[mode].as<uint32_t>(),
                                                         t.ind[s].as<uint32_t>(), Is, n,
                                                         k0.as<uint64_t>(), p0.as<uint32_t>(), io, end_bit);
  count_launch();
  SF_CUDA(cudaGetLastError());
  cub::DoubleBuffer<uint64_t> dk(k0.as<uint64_t>(), k1.as<uint64_t>());
  cub::DoubleBuffer<uint32_t> dv(p0.as<uint32_t>(), p1.as<uint32_t>());
  size_t temp = 0;
  SF_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, temp, dk, dv, (int64_t)n, 0, end_bit, t.stream));
  DevBuf tmp(temp + 16);
  SF_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, temp, dk, dv, (int64_t)n, 0, end_bit, t.stream));
  count_launch((uint64_t)((end_bit + 7) / 8) * 3);
  if (dk.Current() == k0.as<uint64_t>()) keys_out = std::move(k0); else keys_out = std::move(k1);
  if (dv.Current() == p0.as<uint32_t>()) pos_out = std::move(p0); else pos_out = std::move(p1);
}

// First j > k with keys[j] >= target, or n (keys sorted ascending, keys[k] < target):
// galloping from k, then bisection -- O(log(run length)) reads, mostly cached for short runs.
__device__ __forceinline__ uint64_t run_end(const uint64_t* __restrict__ keys, uint64_t n, uint64_t k,
                                            uint64_t target, uint64_t kmask) {
  uint64_t lo = k, hi = n, step = 1;
  while (true) {
    const uint64_t j = lo + step;
    if (j >= n) break;
    if ((__ldg(keys + j) & kmask) >= target) {
      hi = j;
      break;
    }
    lo = j;
    step <<= 1;
  }
  while (hi - lo > 1) {
    const uint64_t mid = lo + (hi - lo) / 2;
    if ((__ldg(keys + mid) & kmask) >= target) hi = mid; else lo = mid;
  }
  return hi;
}

// Slice and fiber statistics of the sorted matricized keys in one pass (
// reading R4): slices = runs of i_n = key / I_s, fibers = runs of the key.  A warp reads a
// tile of 32 x RS_ITEMS consecutive keys (RS_ITEMS per lane, coalesced); a run's length is the
// distance to the next run start -- in the lane, in a later lane (warp suffix-min of each
// lane's first start), or, for the one run of each kind that leaves the tile, found by
// galloping in global memory (run_end).
constexpr int RS_ITEMS = 8;
__global__ void __launch_bounds__(256) run_stats_kernel(const uint64_t* __restrict__ keys, uint64_t n, Div64 Is,
                                                        uint64_t kmask, unsigned long long* __restrict__ runs,
                                                        FeatAcc* __restrict__ acc) {
  __shared__ unsigned long long h[SF_HIST_BINS];
  for (int i = threadIdx.x; i < SF_HIST_BINS; i += blockDim.x) h[i] = 0;
  __syncthreads();
  constexpr uint64_t NONE = ~0ull;
  constexpr uint64_t TILE = 32 * RS_ITEMS;
  const unsigned full = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x / 32);
  const uint64_t ntiles = (n + TILE - 1) / TILE;
  unsigned long long ns = 0, nf = 0, ms = 0, mf = 0, sq = 0;
  // slices of < 2^RS_LOW_BINS nonzeros (nearly all in hyper-sparse modes) are binned in
  // registers: shared-memory atomics on a handful of bins would serialise
  constexpr int RS_LOW_BINS = 6;
  unsigned hlow[RS_LOW_BINS] = {};
  for (uint64_t w = (uint64_t)blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32; w < ntiles; w += nwarps) {
    const uint64_t t0 = w * TILE, t1 = min(n, t0 + TILE);
    const uint64_t base = t0 + (uint64_t)lane * RS_ITEMS;
    uint64_t x[RS_ITEMS];
    if (base + RS_ITEMS <= n) {
      const ulonglong2* v = reinterpret_cast<const ulonglong2*>(keys + base);
#pragma unroll
      for (int q = 0; q < RS_ITEMS / 2; ++q) {
        const ulonglong2 u = __ldg(v + q);
        x[2 * q] = u.x & kmask;
        x[2 * q + 1] = u.y & kmask;
      }
    } else {
#pragma unroll
      for (int i = 0; i < RS_ITEMS; ++i) x[i] = (base + i < n) ? (__ldg(keys + base + i) & kmask) : 0;
    }
    uint64_t prev = __shfl_up_sync(full, x[RS_ITEMS - 1], 1);
    if (lane == 0) prev = t0 ? (__ldg(keys + t0 - 1) & kmask) : 0;
    // start flags (bit i: item i starts a fiber / a slice; items past n start nothing)
    unsigned fs = 0, ss = 0;
    uint64_t sprev = Is.div(prev);
#pragma unroll
    for (int i = 0; i < RS_ITEMS; ++i) {
      const uint64_t k = base + i;
      const uint64_t sl = Is.div(x[i]);
      if (k < n) {
        if (k == 0 || x[i] != prev) fs |= 1u << i;
        if (k == 0 || sl != sprev) ss |= 1u << i;
      }
      prev = x[i];
      sprev = sl;
    }
    // the first start at or after the next lane, for either kind; t1 when the tile ends there
    // with n (the runs end at n), NONE when a run may continue past the tile
    uint64_t ffirst = fs ? base + (__ffs(fs) - 1) : NONE, sfirst = ss ? base + (__ffs(ss) - 1) : NONE;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const uint64_t a = __shfl_down_sync(full, ffirst, off), b = __shfl_down_sync(full, sfirst, off);
      if (lane + off < 32) {
        ffirst = min(ffirst, a);
        sfirst = min(sfirst, b);
      }
    }
    uint64_t fnext = __shfl_down_sync(full, ffirst, 1), snext = __shfl_down_sync(full, sfirst, 1);
    if (lane == 31) fnext = snext = NONE;
    if (t1 == n) {
      fnext = min(fnext, n);
      snext = min(snext, n);
    }
#pragma unroll
    for (int i = RS_ITEMS - 1; i >= 0; --i) {
      const uint64_t k = base + i;
      if (fs >> i & 1) {
        const uint64_t e = (fnext != NONE) ? fnext : run_end(keys, n, t1 - 1, x[i] + 1, kmask);
        const unsigned long long len = e - k;
        ++nf;
        mf = max(mf, len);
        fnext = k;
      }
      if (ss >> i & 1) {
        const uint64_t e = (snext != NONE) ? snext : run_end(keys, n, t1 - 1, (Is.div(x[i]) + 1) * Is.d, kmask);
        const unsigned long long len = e - k;
        ++ns;
        ms = max(ms, len);
        sq += len * len;
        const int bin = 63 - __clzll((long long)len);
        if (bin < RS_LOW_BINS) {
#pragma unroll
          for (int b = 0; b < RS_LOW_BINS; ++b) hlow[b] += (b == bin);
        } else {
          atomicAdd(&h[bin], 1ull);
        }
        snext = k;
      }
    }
  }
#pragma unroll
  for (int b = 0; b < RS_LOW_BINS; ++b) {
    const unsigned v = __reduce_add_sync(full, hlow[b]);
    if (lane == 0 && v) atomicAdd(&h[b], (unsigned long long)v);
  }
  typedef cub::BlockReduce<unsigned long long, 256> BR;
  __shared__ typename BR::TempStorage tmp;
  unsigned long long r[5];
  r[0] = BR(tmp).Sum(ns);
  __syncthreads();
  r[1] = BR(tmp).Sum(nf);
  __syncthreads();
  r[2] = BR(tmp).Reduce(ms, cub::Max());
  __syncthreads();
  r[3] = BR(tmp).Reduce(mf, cub::Max());
  __syncthreads();
  r[4] = BR(tmp).Sum(sq);
  if (threadIdx.x == 0) {
    if (r[0]) atomicAdd(runs, r[0]);
    if (r[1]) atomicAdd(runs + 1, r[1]);
    atomicMax(&acc->max_slice, r[2]);
    atomicMax(&acc->max_fiber, r[3]);
    if (r[4]) atomicAdd(&acc->sum_sq, r[4]);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < SF_HIST_BINS; i += blockDim.x)
    if (h[i]) atomicAdd(&acc->hist[i], h[i]);
}

// Features (reading R4) of the matricized order.
static void features_from_sorted(Tensor& t, int mode, const uint64_t* keys, sf_features_t* f) {
  const uint64_t n = t.nnz;
  const int s = secondary_mode(t, mode);
  const uint64_t Is = t.dims[s];
  memset(f, 0, sizeof(*f));
  f->nnz = n;
  f->dim = t.dims[mode];
  f->nmodes = t.nmodes;
  f->mode = mode;
  f->secondary = s;
  if (n > 0) {
    DevBuf accb(sizeof(FeatAcc) + 16);
    unsigned long long* runs = reinterpret_cast<unsigned long long*>(accb.as<char>() + sizeof(FeatAcc));
    SF_CUDA(cudaMemsetAsync(accb.p, 0, sizeof(FeatAcc) + 16, t.stream));
    const uint64_t kmask = t.carry_kb[mode] ? (1ull << t.carry_kb[mode]) - 1 : ~0ull;
    run_stats_kernel<<<grid_for((n + RS_ITEMS - 1) / RS_ITEMS), 256, 0, t.stream>>>(keys, n, Div64(Is), kmask, runs,
                                                                                  accb.as<FeatAcc>());
    count_launch();
    SF_CUDA(cudaGetLastError());
    FeatAcc a;
    unsigned long long c[2];
    {
      void* dst[2] = {&a, c};
      const void* src[2] = {accb.p, runs};
      const size_t nb[2] = {sizeof(FeatAcc), 16};
      d2h_small(t.stream, 2, dst, src, nb);
    }
    f->num_slices = c[0];
    f->num_fibers = c[1];
    f->max_nnz_per_slice = a.max_slice;
    f->max_nnz_per_fiber = a.max_fiber;
    f->sum_sq_nnz_per_slice = a.sum_sq;
    for (int i = 0; i < SF_HIST_BINS; ++i) f->slice_hist[i] = a.hist[i];
  }
  f->slice_ratio = f->dim ? (double)f->num_slices / (double)f->dim : 0.0;
  f->fiber_ratio = f->num_slices ? (double)f->num_fibers / (double)f->num_slices : 0.0;
  f->avg_nnz_per_slice = f->num_slices ? (double)n / (double)f->num_slices : 0.0;
  f->avg_nnz_per_fiber = f->num_fibers ? (double)n / (double)f->num_fibers : 0.0;
  if (f->num_slices) {
    double var = (double)f->sum_sq_nnz_per_slice / (double)f->num_slices -
                 f->avg_nnz_per_slice * f->avg_nnz_per_slice;
    f->std_nnz_per_slice = var > 0 ? sqrt(var) : 0.0;
  }
}

void compute_features(Tensor& t, int mode, sf_features_t* out, DevBuf* keys_out, DevBuf* pos_out) {
  if (!t.have_features[mode]) {
    DevBuf keys, pos;
    if (t.nnz) matricized_sort(t, mode, keys, pos);
    features_from_sorted(t, mode, keys.as<uint64_t>(), &t.features[mode]);
    t.have_features[mode] = true;
    if (keys_out && pos_out) {
      *keys_out = std::move(keys);
      *pos_out = std::move(pos);
    }
  }
  *out = t.features[mode];
}

// ---------------------------------------------------------------------------
struct TileParams {
  const uint32_t* ind[SF_MAX_MODES];
  uint32_t block_rows[SF_MAX_MODES];
  uint64_t ntiles[SF_MAX_MODES];
  uint32_t staged_mask;
  int nmodes;
};

// Single staged mode == the secondary key s: the tile id is (key % I_s) / block_rows, read
// from the (sequential) matricized keys instead of a random 4-byte gather of i_s.
__global__ void tile_key_from_keys_kernel(const uint64_t* __restrict__ keys, const uint32_t* __restrict__ pos,
                                          uint64_t n, Div64 Is, uint64_t kmask, uint32_t block_rows,
                                          uint64_t* __restrict__ tkey, uint32_t* __restrict__ tpos) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += stride) {
    const uint64_t key = keys[k] & kmask;
    tkey[k] = (uint32_t)(key - Is.div(key) * Is.d) / block_rows;
    tpos[k] = pos[k];
  }
}

// Single staged mode == the carried other mode o (3-way): tile id = i_o / block_rows =
// (i_o >> 17) / (block_rows >> 17) for block_rows a multiple of 2^17, from the key's high bits.
__global__ void tile_key_from_carry_kernel(const uint64_t* __restrict__ keys, const uint32_t* __restrict__ pos,
                                           uint64_t n, int kb, uint32_t coarse_rows, uint64_t* __restrict__ tkey,
                                           uint32_t* __restrict__ tpos) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += stride) {
    tkey[k] = (uint32_t)(keys[k] >> kb) / coarse_rows;
    tpos[k] = pos[k];
  }
}

__global__ void tile_key_kernel(TileParams tp, const uint32_t* __restrict__ pos, uint64_t n,
                                uint64_t* __restrict__ tkey, uint32_t* __restrict__ tpos) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += stride) {
    const uint32_t e = pos[k];
    uint64_t t = 0;
    for (int m = 0; m < tp.nmodes; ++m)
      if (tp.staged_mask & (1u << m)) t = t * tp.ntiles[m] + tp.ind[m][e] / tp.block_rows[m];
    tkey[k] = t;
    tpos[k] = e;
  }
}

// AoS copy of the raw COO: one record of W words per nonzero (N indices, value, padding),
// W = 4 / 8 / 16, so the permutation gather reads one 16/32/64-byte record per nonzero
// (one or two sectors) instead of N+1 scattered 4-byte words.
struct AosParams {
  const uint32_t* ind[SF_MAX_MODES];
  const float* val;
  uint32_t* aos;
  int nmodes, W;
};

__global__ void build_aos_kernel(AosParams a, uint64_t n) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += stride) {
    uint32_t* r = a.aos + e * a.W;
    for (int m = 0; m < a.nmodes; ++m) r[m] = a.ind[m][e];
    r[a.nmodes] = __float_as_uint(a.val[e]);
  }
}

static void aos_segment(Tensor& t, uint64_t a, uint64_t len, cudaStream_t st) {
  AosParams p{};
  for (int m = 0; m < t.nmodes; ++m) p.ind[m] = t.ind[m].as<uint32_t>() + a;
  p.val = t.val.as<float>() + a;
  p.aos = t.aos.as<uint32_t>() + a * (uint64_t)t.aos_words;
  p.nmodes = t.nmodes;
  p.W = t.aos_words;
  build_aos_kernel<<<grid_for(len), 256, 0, st>>>(p, len);
  count_launch();
}

template <int W>
__global__ void gather_aos_kernel(const uint32_t* __restrict__ aos, const uint32_t* __restrict__ perm,
                                  uint64_t n, int nmodes, uint32_t* const* __restrict__ dst,
                                  float* __restrict__ vdst) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += stride) {
    const uint4* rec = reinterpret_cast<const uint4*>(aos + (uint64_t)perm[k] * W);
    uint32_t w[W];
#pragma unroll
    for (int q = 0; q < W / 4; ++q) {
      const uint4 v = __ldg(rec + q);
      w[4 * q] = v.x; w[4 * q + 1] = v.y; w[4 * q + 2] = v.z; w[4 * q + 3] = v.w;
    }
#pragma unroll
    for (int m = 0; m < W - 1; ++m)
      if (m < nmodes) dst[m][k] = w[m];
    vdst[k] = __uint_as_float(w[nmodes < W ? nmodes : 0]);
  }
}

// ---- hot-row cache (launch.hot_kb; DESIGN.md §5 "hot-row cache") ----
// cnt[x] = nonzeros of the handle whose mode-m index is x

struct HotCount {
  const uint32_t* cnt[SF_MAX_MODES];
  uint64_t dim[SF_MAX_MODES];
  int n;
  uint32_t tau[32];
};

// above[j] = rows (over every hot-enabled factor) with cnt > tau[j], for 32 thresholds at once
__global__ void hot_above_kernel(const HotCount h, unsigned long long* __restrict__ above) {
  __shared__ unsigned long long acc[32];
  if (threadIdx.x < 32) acc[threadIdx.x] = 0;
  __syncthreads();
  uint32_t c[32];
#pragma unroll
  for (int j = 0; j < 32; ++j) c[j] = 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (int q = 0; q < h.n; ++q)
    for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < h.dim[q]; x += stride) {
      const uint32_t v = __ldg(h.cnt[q] + x);
#pragma unroll
      for (int j = 0; j < 32; ++j) c[j] += v > h.tau[j];
    }
#pragma unroll
  for (int j = 0; j < 32; ++j) {
    uint32_t v = c[j];
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(&acc[j], (unsigned long long)v);
  }
  __syncthreads();
  if (threadIdx.x < 32 && acc[threadIdx.x]) atomicAdd(above + threadIdx.x, acc[threadIdx.x]);
}

__global__ void hot_flag_kernel(const uint32_t* __restrict__ cnt, uint64_t dim, uint32_t tau, uint32_t* __restrict__ flag) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < dim; x += stride)
    flag[x] = __ldg(cnt + x) > tau ? 1u : 0u;
}

// rows[slot[x]] = x for every hot row x, and slot[] becomes the record's index map in place:
// map[x] = slot[x] | bit for hot rows, x for the others (one lookup per field in the gather)
__global__ void hot_rows_kernel(const uint32_t* __restrict__ cnt, uint32_t* __restrict__ slot, uint64_t dim,
                                uint32_t tau, uint32_t bit, uint32_t* __restrict__ rows) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < dim; x += stride) {
    if (__ldg(cnt + x) > tau) {
      const uint32_t q = slot[x];
      rows[q] = (uint32_t)x;
      slot[x] = q | bit;
    } else {
      slot[x] = (uint32_t)x;
    }
  }
}

// The smallest threshold tau with #{rows of every slot in hc with count > tau} <= budget: 32
// geometric candidates (0, 1, 3, 7, ...), then 32 linear ones inside the bracketing interval.
static uint32_t hot_threshold(Tensor& t, HotCount hc, uint64_t budget) {
  DevBuf above(32 * 8);
  uint64_t dimmax = 0;
  for (int q = 0; q < hc.n; ++q) dimmax = std::max(dimmax, hc.dim[q]);
  auto count_above = [&](unsigned long long* h) {
    SF_CUDA(cudaMemsetAsync(above.p, 0, 32 * 8, t.stream));
    hot_above_kernel<<<grid_for(dimmax), 256, 0, t.stream>>>(hc, above.as<unsigned long long>());
    count_launch();
    d2h_small(t.stream, h, above.p, 32 * 8);
  };
  unsigned long long h[32];
  for (int j = 0; j < 32; ++j) hc.tau[j] = (j == 31) ? 0xFFFFFFFFu : ((1u << j) - 1u);
  count_above(h);
  int j = 0;
  while (j < 31 && h[j] > budget) ++j;
  uint32_t tau = hc.tau[j];
  if (j > 0) {  // refine inside (tau[j-1], tau[j]]
    const uint64_t lo = (uint64_t)hc.tau[j - 1] + 1, hi = hc.tau[j];
    for (int i = 0; i < 32; ++i) hc.tau[i] = (uint32_t)std::min<uint64_t>(hi, lo + ((hi - lo) * i + 30) / 31);
    count_above(h);
    for (int i = 0; i < 32; ++i)
      if (h[i] <= budget) { tau = hc.tau[i]; break; }
  }
  return tau;
}

__global__ void hot_sum_kernel(const uint32_t* __restrict__ cnt, uint64_t dim, uint32_t tau,
                               unsigned long long* __restrict__ sum) {
  unsigned long long a = 0;
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < dim; x += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t c = __ldg(cnt + x);
    if (c > tau) a += c;
  }
  for (int o = 16; o; o >>= 1) a += __shfl_xor_sync(0xFFFFFFFFu, a, o);
  if ((threadIdx.x & 31) == 0 && a) atomicAdd(sum, a);
}

static void ensure_hot_counts(Tensor& t, int m) {
  if (t.hot_cnt[m].p) return;
  t.hot_cnt[m].alloc(t.dims[m] * 4 + 16);
  SF_CUDA(cudaMemsetAsync(t.hot_cnt[m].p, 0, t.dims[m] * 4, t.stream));
  count_rows(t.ind[m].as<uint32_t>(), nullptr, t.nnz, t.dims[m], t.hot_cnt[m].as<uint32_t>(), t.stream);
}

void hot_coverage(Tensor& t, int m, uint64_t rows) {
  if (t.hot_cover[m] >= 0) return;
  ensure_hot_counts(t, m);
  HotCount hc{};
  hc.cnt[0] = t.hot_cnt[m].as<uint32_t>();
  hc.dim[0] = t.dims[m];
  hc.n = 1;
  const uint32_t tau = hot_threshold(t, hc, rows);
  DevBuf sum(16);
  SF_CUDA(cudaMemsetAsync(sum.p, 0, 8, t.stream));
  hot_sum_kernel<<<grid_for(t.dims[m]), 256, 0, t.stream>>>(hc.cnt[0], t.dims[m], tau, sum.as<unsigned long long>());
  count_launch();
  unsigned long long v = 0;
  d2h_small(t.stream, &v, sum.p, 8);
  t.hot_cover[m] = t.nnz ? (double)v / (double)t.nnz : 0.0;
}

// frag3 records: kernel-order record k = [raw field fmap[0], ..., fmap[WK-1]] of the raw
// AoS record perm[k] (fmap < 0: zero padding).  Slot order: i_n, gathered slots, value.
// Packed (nfields > 0): fields f < nfields (raw word fmap[f]) are OR-ed in at bit boff[f]
// of words 0..2, and word 3 = raw word fmap[nfields] (the value).
struct RecParams {
  int fmap[8];
  int nfields;
  uint32_t boff[8];
  // hot-row cache: field d (a gathered slot) with hmap[d] != nullptr becomes hmap[d][x]
  // (the row's slot in the hot block with the slot's hot bit set, or x itself)
  const uint32_t* hmap[8];
};

// Record fields in slot order from a raw AoS record (with the hot-row index map applied).
template <int WR, int WK>
__device__ __forceinline__ void rec_fields(const uint32_t (&w)[WR], const RecParams& rp, uint32_t (&o)[WK]) {
#pragma unroll
  for (int d = 0; d < WK; ++d) {
    uint32_t x = 0;
#pragma unroll
    for (int q = 0; q < WR; ++q) x = (rp.fmap[d] == q) ? w[q] : x;
    if (rp.hmap[d]) x = __ldg(rp.hmap[d] + x);
    o[d] = x;
  }
}

template <int WK>
__device__ __forceinline__ void rec_store(const uint32_t (&o)[WK], const RecParams& rp, uint32_t* __restrict__ rec,
                                          uint64_t k) {
  if (WK == 8 && rp.nfields > 0) {  // packed 16-byte record
    uint32_t o0 = 0, o1 = 0, o2 = 0;
#pragma unroll
    for (int f = 0; f < 8; ++f) {
      if (f >= rp.nfields) break;
      const uint32_t x = o[f < WK ? f : 0], off = rp.boff[f], wi = off >> 5, sh = off & 31u;
      const uint32_t lo = x << sh, hi = sh ? (x >> (32u - sh)) : 0u;
      if (wi == 0) { o0 |= lo; o1 |= hi; } else if (wi == 1) { o1 |= lo; o2 |= hi; } else { o2 |= lo; }
    }
    uint32_t val = 0;
#pragma unroll
    for (int f = 0; f < WK; ++f) val = (f == rp.nfields) ? o[f] : val;
    reinterpret_cast<uint4*>(rec)[k] = make_uint4(o0, o1, o2, val);
    return;
  }
  uint4* dst = reinterpret_cast<uint4*>(rec + k * WK);
#pragma unroll
  for (int q = 0; q < WK / 4; ++q) dst[q] = make_uint4(o[4 * q], o[4 * q + 1], o[4 * q + 2], o[4 * q + 3]);
}

// Kernel-order records from the AoS copy: rec[k] = record(aos[perm[k]]).  (Four independent
// gathers per thread were measured 10-20 % slower: fewer resident warps.)
template <int WR, int WK>
__global__ void gather_rec_kernel(const uint32_t* __restrict__ aos, const uint32_t* __restrict__ perm,
                                  uint64_t n, RecParams rp, uint32_t* __restrict__ rec) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += stride) {
    const uint4* src = reinterpret_cast<const uint4*>(aos + (uint64_t)__ldg(perm + k) * WR);
    uint32_t w[WR];
#pragma unroll
    for (int q = 0; q < WR / 4; ++q) {
      const uint4 v = __ldg(src + q);
      w[4 * q] = v.x; w[4 * q + 1] = v.y; w[4 * q + 2] = v.z; w[4 * q + 3] = v.w;
    }
    uint32_t o[WK];
    rec_fields<WR, WK>(w, rp, o);
    rec_store<WK>(o, rp, rec, k);
  }
}


struct GatherParams {
  const uint32_t* src[SF_MAX_MODES];
  uint32_t* dst[SF_MAX_MODES];
  const float* vsrc;
  float* vdst;
  int nmodes;
};

// Chunks of tile t: nch[t] = ceil(cnt[t] / C) (0 past the encoded runs: cnt was zeroed).
__global__ void chunk_count_kernel(const uint32_t* __restrict__ cnt, uint64_t ntiles, uint32_t C,
                                   uint32_t* __restrict__ nch) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < ntiles; t += stride)
    nch[t] = (cnt[t] + C - 1) / C;
}

// tile_chunk[t] = first chunk of tile t (coff, or 0 for the single tile of an unstaged plan),
// tile_chunk[nr] = nchunks: the kernel walks tiles by index instead of searching chunk_tile.
__global__ void tile_chunk_kernel(const uint32_t* __restrict__ coff, uint32_t nr, uint64_t nchunks,
                                  uint32_t* __restrict__ tile_chunk) {
  for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t <= nr; t += gridDim.x * blockDim.x)
    tile_chunk[t] = (t == nr) ? (uint32_t)nchunks : (coff ? coff[t] : 0u);
}

// chunk j (< nchunks) of tile t (coff[t] <= j < coff[t+1], binary search over the nr tiles):
// begins at tstart[t] + (j - coff[t]) * C, tile id uniq[t]; cbegin[nchunks] = n.  Without
// tiles (uniq == nullptr) every chunk is j * C of tile 0.
__global__ void chunk_fill_kernel(const uint64_t* __restrict__ uniq, const uint32_t* __restrict__ tstart,
                                  const uint32_t* __restrict__ coff, const void* unused, uint32_t nr, uint32_t C,
                                  uint64_t n, uint64_t nchunks, uint32_t* __restrict__ cbegin,
                                  uint64_t* __restrict__ ctile) {
  (void)unused;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j <= nchunks; j += stride) {
    if (j == nchunks) { cbegin[j] = (uint32_t)n; continue; }
    if (!uniq) { cbegin[j] = (uint32_t)(j * C); ctile[j] = 0; continue; }
    uint32_t lo = 0, hi = nr;  // last tile with coff <= j
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (coff[mid] <= j) lo = mid; else hi = mid;
    }
    cbegin[j] = tstart[lo] + (uint32_t)(j - coff[lo]) * C;
    ctile[j] = uniq[lo];
  }
}


void build_plan(Tensor& t, Plan& p, int mode, int rank, const sf_launch_t& launch, DevBuf* keys_in,
                DevBuf* pos_in) {
  cudaEvent_t ev0, ev1;
  SF_CUDA(cudaEventCreate(&ev0));
  SF_CUDA(cudaEventCreate(&ev1));
  SF_CUDA(cudaEventRecord(ev0, t.stream));
  const int N = t.nmodes;
  p.mode = mode;
  p.rank = rank;
  p.launch = launch;
  const uint64_t n = t.nnz;
  const uint64_t lo = (uint64_t)(((unsigned __int128)t.rank * n) / t.nranks);
  const uint64_t hi = (uint64_t)(((unsigned __int128)(t.rank + 1) * n) / t.nranks);
  const uint64_t nl = hi - lo;
  p.nnz_local = nl;
  if (nl >= (1ull << 32)) throw StatusError{SF_ERR_UNSUPPORTED, "shard nnz must be < 2^32"};

  DevBuf keys, pos0;
  if (keys_in && pos_in && keys_in->p && pos_in->p) {  // reuse the features' sort
    keys = std::move(*keys_in);
    pos0 = std::move(*pos_in);
  } else if (n) {
    matricized_sort(t, mode, keys, pos0);
  }
  if (!t.have_features[mode]) {
    features_from_sorted(t, mode, keys.as<uint64_t>(), &t.features[mode]);
    t.have_features[mode] = true;
  }
  p.feat = t.features[mode];
  trace_mark("build: sorted");

  const int s = secondary_mode(t, mode);
  p.row_begin = p.row_end = 0;
  if (nl) {
    uint64_t kb, ke;
    {
      void* dst[2] = {&kb, &ke};
      const void* src[2] = {keys.as<uint64_t>() + lo, keys.as<uint64_t>() + hi - 1};
      const size_t nb[2] = {8, 8};
      d2h_small(t.stream, 2, dst, src, nb);
    }
    const uint64_t kmask = t.carry_kb[mode] ? (1ull << t.carry_kb[mode]) - 1 : ~0ull;
    p.row_begin = (kb & kmask) / t.dims[s];
    p.row_end = (ke & kmask) / t.dims[s] + 1;
  }
  // the caller's out block: whole Y unsharded, the touched rows of a shard
  p.out_row0 = t.nranks > 1 ? p.row_begin : 0;
  p.out_rows = t.nranks > 1 ? p.row_end - p.row_begin : t.dims[mode];
  trace_mark("build: shard range");
  const bool staged_is_secondary = launch.kernel == SF_KERNEL_FRAG && launch.staged_mask == (1u << s);
  // tiles of the other mode of a 3-way tensor from the bits its sort carried
  const int o = N == 3 ? 3 - mode - s : -1;
  const bool staged_is_carry = launch.kernel == SF_KERNEL_FRAG && o >= 0 && t.carry_kb[mode] &&
                               launch.staged_mask == (1u << o) &&
                               launch.block_rows[o] % (1u << kCarryShift) == 0;
  if (!staged_is_secondary && !staged_is_carry) keys.release();  // else kept for the tile keys

  // Kernel order (positions into the raw COO).
  const bool staged = (launch.kernel == SF_KERNEL_FRAG) && launch.staged_mask != 0;
  DevBuf perm(nl * 4 + kPadBytes), tkeys;
  if (nl) {
    if (staged) {
      TileParams tp{};
      uint64_t total_tiles = 1;
      for (int m = 0; m < N; ++m) {
        tp.ind[m] = t.ind[m].as<uint32_t>();
        if (launch.staged_mask & (1u << m)) {
          tp.block_rows[m] = launch.block_rows[m];
          tp.ntiles[m] = (t.dims[m] + launch.block_rows[m] - 1) / launch.block_rows[m];
          total_tiles *= tp.ntiles[m];
        }
      }
      tp.staged_mask = launch.staged_mask;
      tp.nmodes = N;
      DevBuf k0(nl * 8 + 16), k1(nl * 8 + 16), p1(nl * 4 + kPadBytes);
      const uint64_t kmask = t.carry_kb[mode] ? (1ull << t.carry_kb[mode]) - 1 : ~0ull;
      if (staged_is_secondary)
        tile_key_from_keys_kernel<<<grid_for(nl), 256, 0, t.stream>>>(
            keys.as<uint64_t>() + lo, pos0.as<uint32_t>() + lo, nl, Div64(t.dims[s]), kmask, launch.block_rows[s],
            k0.as<uint64_t>(), perm.as<uint32_t>());
      else if (staged_is_carry)
        tile_key_from_carry_kernel<<<grid_for(nl), 256, 0, t.stream>>>(
            keys.as<uint64_t>() + lo, pos0.as<uint32_t>() + lo, nl, t.carry_kb[mode],
            launch.block_rows[o] >> kCarryShift, k0.as<uint64_t>(), perm.as<uint32_t>());
      else
        tile_key_kernel<<<grid_for(nl), 256, 0, t.stream>>>(tp, pos0.as<uint32_t>() + lo, nl, k0.as<uint64_t>(),
                                                           perm.as<uint32_t>());
      count_launch();
      SF_CUDA(cudaGetLastError());
      pos0.release();
      keys.release();
      const int end_bit = std::max(1, bitlen(total_tiles - 1));
      cub::DoubleBuffer<uint64_t> dk(k0.as<uint64_t>(), k1.as<uint64_t>());
      cub::DoubleBuffer<uint32_t> dv(perm.as<uint32_t>(), p1.as<uint32_t>());
      size_t temp = 0;
      SF_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, temp, dk, dv, (int64_t)nl, 0, end_bit, t.stream));
      DevBuf tmp(temp + 16);
      SF_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, temp, dk, dv, (int64_t)nl, 0, end_bit, t.stream));
      count_launch((uint64_t)((end_bit + 7) / 8) * 3);
      if (dk.Current() == k0.as<uint64_t>()) tkeys = std::move(k0); else tkeys = std::move(k1);
      if (dv.Current() != perm.as<uint32_t>()) perm = std::move(p1);
    } else {
      d2d_copy(perm.p, pos0.as<uint32_t>() + lo, nl * 4, t.stream);
      pos0.release();
    }
  }

  trace_mark("build: tile order");
  // AoS record copy of the raw COO (built once per tensor, reused by every mode's plan)
  const int WR = (N + 1 <= 4) ? 4 : (N + 1 <= 8 ? 8 : 16);
  if (nl && !t.aos.p) {
    t.aos.alloc((size_t)n * WR * 4 + 64);
    AosParams a{};
    for (int m = 0; m < N; ++m) a.ind[m] = t.ind[m].as<uint32_t>();
    a.val = t.val.as<float>();
    a.aos = t.aos.as<uint32_t>();
    a.nmodes = N;
    a.W = WR;
    build_aos_kernel<<<grid_for(n), 256, 0, t.stream>>>(a, n);
    count_launch();
    SF_CUDA(cudaGetLastError());
    t.aos_words = WR;
  }
  const bool use_rec = launch.kernel == SF_KERNEL_FRAG && frag_supported(N, rank);
  p.rec_words = 0;
  if (use_rec) {
    // frag3 records in slot order [i_n, staged slots, other gathered slots, value, 0...]
    const bool packed = N >= 4 && rec_packable(t);
    const int WK = packed ? 4 : rec_words_for(N);
    p.rec_words = WK;
    p.rec_packed = packed;
    p.rec.alloc(nl * WK * 4 + kPadBytes);
    SF_CUDA(cudaMemsetAsync(p.rec.as<uint32_t>() + nl * WK, 0, kPadBytes, t.stream));
    RecParams rp{};
    for (int d = 0; d < 8; ++d) rp.fmap[d] = -1;
    int slot_mode[SF_MAX_MODES];
    const int Ssm = frag_slot_order(N, mode, smem_staged_mask(launch), slot_mode);
    rp.fmap[0] = mode;
    for (int q = 0; q < N - 1; ++q) rp.fmap[1 + q] = slot_mode[q];
    rp.fmap[N] = N;  // value word of the raw record
    rp.nfields = 0;
    // hot-row cache: eligible gathered slots are gathered from L2/HBM (not staged in shared
    // memory, not the L2-tiled mode; the selector decides whether the plan uses the cache)
    bool hot_q[SF_MAX_MODES] = {};
    std::vector<DevBuf> hcnt(SF_MAX_MODES), hslot(SF_MAX_MODES);
    const uint32_t* hcnt_ptr[SF_MAX_MODES] = {};
    p.hot_total = 0;
    for (int q = 0; q < SF_MAX_MODES; ++q) {
      p.hot_bit[q] = 0;
      p.hot_count[q] = p.hot_off[q] = 0;
      p.hot_rows[q].release();
    }
    p.hot_cache.release();
    if (launch.hot_kb > 0 && nl) {
      int bits_used = 0;
      if (packed)
        for (int f = 0; f < N; ++f) bits_used += index_bits(t.dims[rp.fmap[f]]);
      for (int q = Ssm; q < N - 1; ++q) {
        const int m = slot_mode[q];
        if (launch.staged_mask & (1u << m)) continue;
        if (t.dims[m] >= (1ull << 31)) continue;
        if (packed && bits_used + 1 > 96) continue;
        bits_used += packed ? 1 : 0;
        hot_q[q] = true;
      }
      HotCount hc{};
      for (int q = 0; q < N - 1; ++q) {
        if (!hot_q[q]) continue;
        const int m = slot_mode[q];
        // row frequencies of mode m: over this plan's nonzeros when the handle is a shard,
        // else over the whole tensor -- counted once per (handle, mode) and reused by every
        // plan that gathers mode m
        const bool whole = t.nranks == 1;
        DevBuf* cnt = whole ? &t.hot_cnt[m] : &hcnt[q];
        if (whole) {
          ensure_hot_counts(t, m);
        } else {
          cnt->alloc(t.dims[m] * 4 + 16);
          SF_CUDA(cudaMemsetAsync(cnt->p, 0, t.dims[m] * 4, t.stream));
          count_rows(t.ind[m].as<uint32_t>(), perm.as<uint32_t>(), nl, t.dims[m], cnt->as<uint32_t>(), t.stream);
        }
        hcnt_ptr[q] = cnt->as<uint32_t>();
        hc.cnt[hc.n] = cnt->as<uint32_t>();
        hc.dim[hc.n] = t.dims[m];
        ++hc.n;
      }
      trace_mark("build: hot counts");
      if (hc.n) {
        // one global threshold tau (rows with count > tau are hot) so the hot rows of every
        // slot fit the budget: the static cache of the most frequently gathered rows
        const uint64_t budget = (uint64_t)launch.hot_kb * 1024ull / ((uint64_t)rank * 4);
        const uint32_t tau = hot_threshold(t, hc, budget);
        uint64_t total = 0;
        for (int q = 0; q < N - 1; ++q) {
          if (!hot_q[q]) continue;
          const int m = slot_mode[q];
          const uint64_t I = t.dims[m];
          hslot[q].alloc(I * 4 + 16);
          hot_flag_kernel<<<grid_for(I), 256, 0, t.stream>>>(hcnt_ptr[q], I, tau, hslot[q].as<uint32_t>());
          uint32_t last_flag = 0, last_slot = 0;
          d2h_small(t.stream, &last_flag, hslot[q].as<uint32_t>() + I - 1, 4);
          size_t tb = 0;
          SF_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, hslot[q].as<uint32_t>(), hslot[q].as<uint32_t>(),
                                                (int64_t)I, t.stream));
          DevBuf tmp(tb + 16);
          SF_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tb, hslot[q].as<uint32_t>(), hslot[q].as<uint32_t>(),
                                                (int64_t)I, t.stream));
          d2h_small(t.stream, &last_slot, hslot[q].as<uint32_t>() + I - 1, 4);
          const uint64_t cnt = (uint64_t)last_slot + last_flag;
          count_launch(2);
          if (cnt == 0) continue;
          p.hot_rows[q].alloc(cnt * 4 + 16);
          p.hot_bit[q] = packed ? (1u << index_bits(I)) : 0x80000000u;
          hot_rows_kernel<<<grid_for(I), 256, 0, t.stream>>>(hcnt_ptr[q], hslot[q].as<uint32_t>(), I, tau,
                                                             p.hot_bit[q], p.hot_rows[q].as<uint32_t>());
          count_launch();
          p.hot_count[q] = cnt;
          p.hot_off[q] = total;
          total += cnt;
          rp.hmap[1 + q] = hslot[q].as<uint32_t>();
        }
        p.hot_total = total;
        trace_mark("build: hot rows");
        if (total) p.hot_cache.alloc(total * rank * 4 + 64);
        SF_CUDA(cudaGetLastError());
      }
    }
    if (packed) {  // fields in slot order, i_n at bit 0 (a hot slot's field has one more bit)
      uint32_t off = 0;
      for (int f = 0; f < N; ++f) {
        const int b = index_bits(t.dims[rp.fmap[f]]) + ((f >= 1 && p.hot_bit[f - 1]) ? 1 : 0);
        rp.boff[f] = off;
        p.rec_boff[f] = off;
        p.rec_bmask[f] = (b >= 32) ? 0xFFFFFFFFu : ((1u << b) - 1u);
        off += (uint32_t)b;
      }
      rp.nfields = N;
    }
    if (nl) {
      const uint32_t* aos = t.aos.as<uint32_t>();
      const uint32_t* pm = perm.as<uint32_t>();
      uint32_t* rec = p.rec.as<uint32_t>();
      if (WR == 4 && WK == 4) gather_rec_kernel<4, 4><<<grid_for(nl), 256, 0, t.stream>>>(aos, pm, nl, rp, rec);
      else if (WR == 8 && WK == 8) gather_rec_kernel<8, 8><<<grid_for(nl), 256, 0, t.stream>>>(aos, pm, nl, rp, rec);
      else if (WR == 8 && WK == 4 && packed)
        gather_rec_kernel<8, 8><<<grid_for(nl), 256, 0, t.stream>>>(aos, pm, nl, rp, rec);
      else throw StatusError{SF_ERR_UNSUPPORTED, "frag3 records: unsupported record width"};
      count_launch();
      SF_CUDA(cudaGetLastError());
      if (p.hot_total) SF_CUDA(cudaStreamSynchronize(t.stream));  // hcnt / hslot are freed on return
    }
  } else {
    // Gather the kernel-order SoA arrays (padded for aligned bulk copies).
    GatherParams g{};
    for (int m = 0; m < N; ++m) {
      p.ind[m].alloc(nl * 4 + kPadBytes);
      SF_CUDA(cudaMemsetAsync(p.ind[m].p, 0, nl * 4 + kPadBytes, t.stream));
      g.src[m] = t.ind[m].as<uint32_t>();
      g.dst[m] = p.ind[m].as<uint32_t>();
    }
    p.val.alloc(nl * 4 + kPadBytes);
    SF_CUDA(cudaMemsetAsync(p.val.p, 0, nl * 4 + kPadBytes, t.stream));
    g.vsrc = t.val.as<float>();
    g.vdst = p.val.as<float>();
    g.nmodes = N;
    if (nl) {
      const int W = WR;
      DevBuf dptr(sizeof(uint32_t*) * SF_MAX_MODES);
      uint32_t* hptr[SF_MAX_MODES] = {};
      for (int m = 0; m < N; ++m) hptr[m] = g.dst[m];
      h2d_small(t.stream, dptr.p, hptr, sizeof(hptr));
      uint32_t* const* dd = reinterpret_cast<uint32_t* const*>(dptr.p);
      switch (W) {
        case 4: gather_aos_kernel<4><<<grid_for(nl), 256, 0, t.stream>>>(t.aos.as<uint32_t>(), perm.as<uint32_t>(), nl, N, dd, g.vdst); break;
        case 8: gather_aos_kernel<8><<<grid_for(nl), 256, 0, t.stream>>>(t.aos.as<uint32_t>(), perm.as<uint32_t>(), nl, N, dd, g.vdst); break;
        default: gather_aos_kernel<16><<<grid_for(nl), 256, 0, t.stream>>>(t.aos.as<uint32_t>(), perm.as<uint32_t>(), nl, N, dd, g.vdst); break;
      }
      count_launch();
      SF_CUDA(cudaGetLastError());
      SF_CUDA(cudaStreamSynchronize(t.stream));  // dptr's host source must outlive the copy
    }
  }
  p.perm = std::move(perm);
  trace_mark("build: records");

  // Chunks.
  p.num_chunks = 0;
  p.num_tiles = 0;
  if (nl) {
    // Per tile (run of equal tile keys in kernel order): its start, its nonzero count and
    // ceil(count / C) chunks; chunk j of tile t begins at start_t + (j - first_chunk_t) * C.
    // O(num_tiles + num_chunks) after one run-length encode of the tile keys.
    const uint32_t C = (uint32_t)std::max(1, launch.chunk_nnz);
    if (!staged) {
      p.num_tiles = 1;
      p.num_chunks = (nl + C - 1) / C;
      p.chunk_begin.alloc((p.num_chunks + 1) * 4 + 16);
      p.chunk_tile.alloc(p.num_chunks * 8 + 16);
      chunk_fill_kernel<<<grid_for(p.num_chunks + 1), 256, 0, t.stream>>>(
          nullptr, nullptr, nullptr, nullptr, 1, C, nl, p.num_chunks, p.chunk_begin.as<uint32_t>(),
          p.chunk_tile.as<uint64_t>());
      p.tile_chunk.alloc(2 * 4 + 16);
      tile_chunk_kernel<<<1, 32, 0, t.stream>>>(nullptr, 1, p.num_chunks, p.tile_chunk.as<uint32_t>());
      count_launch(2);
    } else {
      uint64_t tiles_bound = 1;
      for (int m = 0; m < N; ++m)
        if (launch.staged_mask & (1u << m))
          tiles_bound = std::min<uint64_t>(nl, tiles_bound * ((t.dims[m] + launch.block_rows[m] - 1) / launch.block_rows[m]));
      tiles_bound = std::min<uint64_t>(tiles_bound, nl);
      DevBuf uniq(tiles_bound * 8 + 16), cnts(tiles_bound * 4 + 16), nruns(16), nch(tiles_bound * 4 + 16),
          tstart(tiles_bound * 4 + 16), coff(tiles_bound * 4 + 16);
      SF_CUDA(cudaMemsetAsync(cnts.p, 0, tiles_bound * 4 + 16, t.stream));
      size_t t1 = 0, t2 = 0;
      SF_CUDA(cub::DeviceRunLengthEncode::Encode(nullptr, t1, tkeys.as<uint64_t>(), uniq.as<uint64_t>(),
                                                 cnts.as<uint32_t>(), nruns.as<uint32_t>(), (int64_t)nl, t.stream));
      SF_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, t2, cnts.as<uint32_t>(), tstart.as<uint32_t>(),
                                            (int64_t)tiles_bound, t.stream));
      DevBuf tmp(std::max(t1, t2) + 16);
      SF_CUDA(cub::DeviceRunLengthEncode::Encode(tmp.p, t1, tkeys.as<uint64_t>(), uniq.as<uint64_t>(),
                                                 cnts.as<uint32_t>(), nruns.as<uint32_t>(), (int64_t)nl, t.stream));
      chunk_count_kernel<<<grid_for(tiles_bound), 256, 0, t.stream>>>(cnts.as<uint32_t>(), tiles_bound, C,
                                                                      nch.as<uint32_t>());
      SF_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, t2, cnts.as<uint32_t>(), tstart.as<uint32_t>(),
                                            (int64_t)tiles_bound, t.stream));
      SF_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, t2, nch.as<uint32_t>(), coff.as<uint32_t>(),
                                            (int64_t)tiles_bound, t.stream));
      count_launch(5);
      uint32_t nr = 0, last_off = 0, last_n = 0;
      {
        void* dst[3] = {&nr, &last_off, &last_n};
        const void* src[3] = {nruns.p, coff.as<uint32_t>() + tiles_bound - 1, nch.as<uint32_t>() + tiles_bound - 1};
        const size_t nb[3] = {4, 4, 4};
        d2h_small(t.stream, 3, dst, src, nb);
      }
      trace_mark("build: chunk count sync");
      p.num_tiles = nr;
      p.num_chunks = (uint64_t)last_off + last_n;
      p.chunk_begin.alloc((p.num_chunks + 1) * 4 + 16);
      p.chunk_tile.alloc(p.num_chunks * 8 + 16);
      chunk_fill_kernel<<<grid_for(p.num_chunks + 1), 256, 0, t.stream>>>(
          uniq.as<uint64_t>(), tstart.as<uint32_t>(), coff.as<uint32_t>(), nullptr, nr, C, nl, p.num_chunks,
          p.chunk_begin.as<uint32_t>(), p.chunk_tile.as<uint64_t>());
      p.tile_chunk.alloc(((uint64_t)nr + 1) * 4 + 16);
      tile_chunk_kernel<<<grid_for((uint64_t)nr + 1), 256, 0, t.stream>>>(coff.as<uint32_t>(), nr, p.num_chunks,
                                                                         p.tile_chunk.as<uint32_t>());
      count_launch(2);
    }
    SF_CUDA(cudaGetLastError());
  } else {
    p.chunk_begin.alloc(16);
    SF_CUDA(cudaMemsetAsync(p.chunk_begin.p, 0, 16, t.stream));
    p.tile_chunk.alloc(16);
    SF_CUDA(cudaMemsetAsync(p.tile_chunk.p, 0, 16, t.stream));
  }
  SF_CUDA(cudaEventRecord(ev1, t.stream));
  SF_CUDA(cudaEventSynchronize(ev1));
  float ms = 0;
  SF_CUDA(cudaEventElapsedTime(&ms, ev0, ev1));
  p.plan_ms = ms;
  cudaEventDestroy(ev0);
  cudaEventDestroy(ev1);
}

// Segment sort of the one-shot streamed path (sf_mttkrp_streamed): stable radix sort of a
// segment's i_n (the low `bits` bits) with the segment positions as payload.
size_t seg_sort_temp_bytes(uint64_t len, int bits) {
  size_t tb = 0;
  SF_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                          (const uint32_t*)nullptr, (uint32_t*)nullptr, (int64_t)len, 0,
                                          std::max(1, bits)));
  return tb;
}

void seg_sort(const uint32_t* keys_in, uint32_t* keys_out, const uint32_t* vals_in, uint32_t* vals_out, uint64_t len,
              int bits, void* temp, size_t temp_bytes, cudaStream_t s) {
  if (!len) return;
  SF_CUDA(cub::DeviceRadixSort::SortPairs(temp, temp_bytes, keys_in, keys_out, vals_in, vals_out, (int64_t)len, 0,
                                          std::max(1, bits), s));
  count_launch((uint64_t)((std::max(1, bits) + 7) / 8) + 1);
}

}  // namespace sf
