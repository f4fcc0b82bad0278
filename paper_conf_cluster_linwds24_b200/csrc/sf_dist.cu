// sf_dist.cu - distributed ingest and preprocessing (SURVEY §8(e) "v2", row F4).
//
// v1 (sf_set_shard / sf_comm_attach): every rank holds the whole raw COO and sorts all of it
// to keep its shard.  v2 (sf_tensor_create_dist): rank p holds only a contiguous slice of
// the input positions; per mode n its shard -- matricized positions [c_p, c_{p+1}),
// c_p = floor(p*nnz/P), the SAME nonzeros in the same order as v1 -- is assembled by
//   1. a histogram of i_n over the local slice, summed over ranks (allgatherv + rank-order sum)
//      -> the global start of every row in the matricized order (exclusive scan);
//   2. every local nonzero is sent to the rank(s) whose position range meets its row's range
//      (whole rows inside one shard go to that rank; a row straddling cuts goes to every rank it
//      straddles) -- one all-to-all (grouped ncclSend/ncclRecv);
//   3. the receiver sorts what it got by (i_n, i_s) -- received blocks arrive in rank order,
//      i.e. in increasing input position, so the stable sort breaks ties by input position as
//      the matricized order does -- and keeps exactly [c_p, c_{p+1}): it received complete
//      rows, so sorted slot k is global position row_start(first row) + k.
// The shard then plans like a one-rank tensor (sub[mode]); its plan is bit-identical to v1's
// (tests/test_gpu_multirank.py through tools/multirank_check.py).
#include <cuda_runtime.h>

#include <algorithm>
#include <cub/cub.cuh>
#include <thrust/iterator/counting_iterator.h>
#include <vector>

#include "sf_internal.h"

namespace sf {

constexpr int SF_MAX_RANKS_DIST = 64;

struct SegIn {
  const uint32_t* ind[SF_MAX_MODES];
  const float* val;
  int nmodes;
};

static inline int grid_of(uint64_t n) { return (int)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 148ull * 16)); }

__global__ void dist_hist_kernel(const uint32_t* __restrict__ in, uint64_t n, uint32_t* __restrict__ hist) {
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (uint64_t)gridDim.x * blockDim.x)
    atomicAdd(hist + __ldg(in + e), 1u);
}

__global__ void dist_sum_kernel(const uint32_t* __restrict__ parts, int P, uint64_t n, uint32_t* __restrict__ out) {
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t a = 0;
    for (int k = 0; k < P; ++k) a += parts[(size_t)k * n + e];
    out[e] = a;
  }
}

struct Cuts {
  uint64_t c[SF_MAX_RANKS_DIST + 1];
  int P;
};

// rank whose position range [c_q, c_{q+1}) contains global position x (c_P = nnz)
__device__ __forceinline__ int rank_of(const Cuts& k, uint64_t x) {
  int q = 0;
  while (q + 1 < k.P && k.c[q + 1] <= x) ++q;
  return q;
}

// flag[e] = 1 iff local nonzero e goes to rank q (its row's positions meet [c_q, c_{q+1}))
__global__ void dist_flag_kernel(const uint32_t* __restrict__ in, uint64_t n, const uint32_t* __restrict__ start,
                                 const uint32_t* __restrict__ cnt, Cuts k, int q, uint8_t* __restrict__ flag) {
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t r = __ldg(in + e);
    const uint64_t a = __ldg(start + r), b = a + __ldg(cnt + r);  // row r = positions [a, b)
    flag[e] = (rank_of(k, a) <= q && q <= rank_of(k, b - 1)) ? 1 : 0;
  }
}

// send record: N indices, value, global input position  (W = N + 2 words)
__global__ void dist_pack_kernel(const uint32_t* __restrict__ sel, uint64_t n, SegIn in, uint64_t pos_begin, int W,
                                 uint32_t* __restrict__ out) {
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t e = __ldg(sel + j);
    uint32_t* o = out + j * W;
    for (int m = 0; m < in.nmodes; ++m) o[m] = __ldg(in.ind[m] + e);
    o[in.nmodes] = __float_as_uint(__ldg(in.val + e));
    o[in.nmodes + 1] = (uint32_t)(pos_begin + e);
  }
}

__global__ void dist_key_kernel(const uint32_t* __restrict__ rec, uint64_t n, int W, int mode, int s, uint64_t Is,
                                uint64_t* __restrict__ key, uint32_t* __restrict__ idx) {
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (uint64_t)gridDim.x * blockDim.x) {
    key[j] = (uint64_t)rec[j * W + mode] * Is + rec[j * W + s];
    idx[j] = (uint32_t)j;
  }
}

struct SubOut {
  uint32_t* ind[SF_MAX_MODES];
  float* val;
  uint32_t* gpos;
  int nmodes;
};

__global__ void dist_unpack_kernel(const uint32_t* __restrict__ rec, const uint32_t* __restrict__ order, uint64_t first,
                                   uint64_t n, int W, SubOut o) {
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t* r = rec + (uint64_t)__ldg(order + first + j) * W;
    for (int m = 0; m < o.nmodes; ++m) o.ind[m][j] = r[m];
    o.val[j] = __uint_as_float(r[o.nmodes]);
    o.gpos[j] = r[o.nmodes + 1];
  }
}

static int bitlen64(uint64_t x) {
  int b = 0;
  while (x) { ++b; x >>= 1; }
  return b;
}

void dist_build_sub(Tensor& t, int mode) {
  if (t.sub[mode]) return;
  if (!t.comm) throw StatusError{SF_ERR_INVALID_ARG, "sf_tensor_create_dist handle: attach a comm before sf_plan"};
  const int P = t.nranks, me = t.rank, N = t.nmodes;
  if (P > SF_MAX_RANKS_DIST) throw StatusError{SF_ERR_UNSUPPORTED, "distributed ingest: too many ranks"};
  cudaStream_t s = t.stream;
  SF_CUDA(cudaSetDevice(t.device));
  const uint64_t In = t.dims[mode], n = t.nnz;
  // 0. the slices must tile [0, nnz_total) in rank order
  {
    DevBuf b((size_t)P * 16 + 16);
    uint64_t mine[2] = {t.pos_begin, n};
    std::vector<uint64_t> bytes(P, 16), displs(P);
    for (int k = 0; k < P; ++k) displs[k] = (uint64_t)k * 16;
    h2d_small(s, b.as<char>() + me * 16, mine, 16);
    t.comm->allgatherv(b.as<char>() + me * 16, b.p, bytes.data(), displs.data(), s);
    std::vector<uint64_t> all(2 * P);
    d2h_small(s, all.data(), b.p, (size_t)P * 16);
    uint64_t at = 0;
    for (int k = 0; k < P; ++k) {
      if (all[2 * k] != at) throw StatusError{SF_ERR_INVALID_ARG, "distributed slices must tile the input in rank order"};
      at += all[2 * k + 1];
    }
    if (at != t.nnz_total) throw StatusError{SF_ERR_INVALID_ARG, "distributed slices do not sum to nnz_total"};
  }
  // 1. global row histogram and row starts
  DevBuf hist(In * 4 + 16), parts((size_t)P * In * 4 + 16), gcnt(In * 4 + 16), gstart(In * 4 + 16);
  SF_CUDA(cudaMemsetAsync(hist.p, 0, In * 4, s));
  if (n) dist_hist_kernel<<<grid_of(n), 256, 0, s>>>(t.ind[mode].as<uint32_t>(), n, hist.as<uint32_t>());
  {
    std::vector<uint64_t> bytes(P, In * 4), displs(P);
    for (int k = 0; k < P; ++k) displs[k] = (uint64_t)k * In * 4;
    t.comm->allgatherv(hist.p, parts.p, bytes.data(), displs.data(), s);
  }
  dist_sum_kernel<<<grid_of(In), 256, 0, s>>>(parts.as<uint32_t>(), P, In, gcnt.as<uint32_t>());
  parts.release();
  {
    size_t tb = 0;
    SF_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, gcnt.as<uint32_t>(), gstart.as<uint32_t>(), (int64_t)In, s));
    DevBuf tmp(tb + 16);
    SF_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tb, gcnt.as<uint32_t>(), gstart.as<uint32_t>(), (int64_t)In, s));
  }
  count_launch(4);
  Cuts cuts{};
  cuts.P = P;
  for (int q = 0; q <= P; ++q) cuts.c[q] = (uint64_t)(((unsigned __int128)q * t.nnz_total) / P);
  // 2. per destination: stable selection of the local nonzeros it needs, packed as records
  const int W = N + 2;
  SegIn in{};
  for (int m = 0; m < N; ++m) in.ind[m] = t.ind[m].as<uint32_t>();
  in.val = t.val.as<float>();
  in.nmodes = N;
  std::vector<uint64_t> scnt(P), sdis(P);
  std::vector<DevBuf> sel(P);
  DevBuf flag(n + 16), nsel(16);
  uint64_t stot = 0;
  for (int q = 0; q < P; ++q) {
    sel[q].alloc(n * 4 + 16);
    if (n) {
      dist_flag_kernel<<<grid_of(n), 256, 0, s>>>(t.ind[mode].as<uint32_t>(), n, gstart.as<uint32_t>(),
                                                  gcnt.as<uint32_t>(), cuts, q, flag.as<uint8_t>());
      size_t tb = 0;
      thrust::counting_iterator<uint32_t> it(0);
      SF_CUDA(cub::DeviceSelect::Flagged(nullptr, tb, it, flag.as<uint8_t>(), sel[q].as<uint32_t>(),
                                         nsel.as<uint64_t>(), (int64_t)n, s));
      DevBuf tmp(tb + 16);
      SF_CUDA(cub::DeviceSelect::Flagged(tmp.p, tb, it, flag.as<uint8_t>(), sel[q].as<uint32_t>(),
                                         nsel.as<uint64_t>(), (int64_t)n, s));
      count_launch(2);
      uint64_t c = 0;
      d2h_small(s, &c, nsel.p, 8);
      scnt[q] = c;
    }
    sdis[q] = stot;
    stot += scnt[q];
  }
  DevBuf sendb(stot * W * 4 + 16);
  for (int q = 0; q < P; ++q)
    if (scnt[q]) {
      dist_pack_kernel<<<grid_of(scnt[q]), 256, 0, s>>>(sel[q].as<uint32_t>(), scnt[q], in, t.pos_begin, W,
                                                        sendb.as<uint32_t>() + sdis[q] * W);
      count_launch();
    }
  for (auto& b : sel) b.release();
  flag.release();
  // receive counts: everybody's send counts (P x P)
  std::vector<uint64_t> rcnt(P), rdis(P);
  {
    DevBuf b((size_t)P * P * 8 + 16);
    std::vector<uint64_t> bytes(P, (uint64_t)P * 8), displs(P);
    for (int k = 0; k < P; ++k) displs[k] = (uint64_t)k * P * 8;
    h2d_small(s, b.as<char>() + (size_t)me * P * 8, scnt.data(), (size_t)P * 8);
    t.comm->allgatherv(b.as<char>() + (size_t)me * P * 8, b.p, bytes.data(), displs.data(), s);
    std::vector<uint64_t> all((size_t)P * P);
    d2h_small(s, all.data(), b.p, (size_t)P * P * 8);
    uint64_t at = 0;
    for (int k = 0; k < P; ++k) {
      rcnt[k] = all[(size_t)k * P + me];
      rdis[k] = at;
      at += rcnt[k];
    }
  }
  uint64_t rtot = 0;
  for (int k = 0; k < P; ++k) rtot += rcnt[k];
  DevBuf recvb(rtot * W * 4 + 16);
  {
    std::vector<uint64_t> sb(P), sd(P), rb(P), rd(P);
    for (int q = 0; q < P; ++q) {
      sb[q] = scnt[q] * W * 4; sd[q] = sdis[q] * W * 4;
      rb[q] = rcnt[q] * W * 4; rd[q] = rdis[q] * W * 4;
    }
    t.comm->alltoallv(sendb.p, sb.data(), sd.data(), recvb.p, rb.data(), rd.data(), s);
  }
  sendb.release();
  // 3. sort what arrived by (i_n, i_s) (stable: arrival order = input order) and keep [c_me, c_me+1)
  const int sm = secondary_mode(t, mode);
  const uint64_t Is = t.dims[sm];
  uint64_t first = 0, keep = 0;
  DevBuf order;
  if (rtot) {
    DevBuf k0(rtot * 8 + 16), k1(rtot * 8 + 16), i0(rtot * 4 + 16), i1(rtot * 4 + 16);
    dist_key_kernel<<<grid_of(rtot), 256, 0, s>>>(recvb.as<uint32_t>(), rtot, W, mode, sm, Is, k0.as<uint64_t>(),
                                                  i0.as<uint32_t>());
    const int end_bit = std::max(1, bitlen64(In * Is - 1));
    cub::DoubleBuffer<uint64_t> dk(k0.as<uint64_t>(), k1.as<uint64_t>());
    cub::DoubleBuffer<uint32_t> dv(i0.as<uint32_t>(), i1.as<uint32_t>());
    size_t tb = 0;
    SF_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, (int64_t)rtot, 0, end_bit, s));
    DevBuf tmp(tb + 16);
    SF_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tb, dk, dv, (int64_t)rtot, 0, end_bit, s));
    count_launch((uint64_t)(end_bit + 7) / 8 + 1);
    uint64_t k_first = 0;
    d2h_small(s, &k_first, dk.Current(), 8);
    uint32_t g0 = 0;
    d2h_small(s, &g0, gstart.as<uint32_t>() + k_first / Is, 4);
    // sorted slot j is global matricized position g0 + j (complete rows were received)
    const uint64_t lo = cuts.c[me], hi = cuts.c[me + 1];
    first = lo > g0 ? lo - g0 : 0;
    keep = (hi > lo) ? hi - lo : 0;
    if (first + keep > rtot) throw StatusError{SF_ERR_CUDA, "distributed ingest: shard bookkeeping mismatch"};
    if (dv.Current() == i0.as<uint32_t>()) order = std::move(i0); else order = std::move(i1);
  }
  // 4. the shard as a one-rank tensor: raw arrays in matricized order + global positions
  Tensor* sub = new Tensor();
  try {
    sub->device = t.device;
    sub->num_sms = t.num_sms;
    sub->smem_optin = t.smem_optin;
    SF_CUDA(cudaStreamCreateWithFlags(&sub->stream, cudaStreamNonBlocking));
    sub->nmodes = N;
    sub->nnz = keep;
    for (int m = 0; m < N; ++m) {
      sub->dims[m] = t.dims[m];
      sub->ind[m].alloc(keep * 4 + kPadBytes);
    }
    sub->val.alloc(keep * 4 + kPadBytes);
    t.sub_gpos[mode].alloc(keep * 4 + 16);
    if (keep) {
      SubOut o{};
      for (int m = 0; m < N; ++m) o.ind[m] = sub->ind[m].as<uint32_t>();
      o.val = sub->val.as<float>();
      o.gpos = t.sub_gpos[mode].as<uint32_t>();
      o.nmodes = N;
      dist_unpack_kernel<<<grid_of(keep), 256, 0, s>>>(recvb.as<uint32_t>(), order.as<uint32_t>(), first, keep, W, o);
      count_launch();
    }
    SF_CUDA(cudaGetLastError());
    SF_CUDA(cudaStreamSynchronize(s));
  } catch (...) {
    delete sub;
    throw;
  }
  t.sub[mode] = sub;
}

}  // namespace sf

using namespace sf;

extern "C" sf_status sf_tensor_create_dist(int nmodes, const uint64_t* dims, uint64_t nnz_total, uint64_t pos_begin,
                                           uint64_t nnz_local, const uint32_t* const* inds, const float* vals,
                                           sf_tensor_t* out) {
  if (nnz_total > 0xFFFFFFFFull || pos_begin + nnz_local > nnz_total) {
    set_error("sf_tensor_create_dist: need pos_begin + nnz_local <= nnz_total < 2^32");
    return SF_ERR_INVALID_ARG;
  }
  const sf_status st = sf_tensor_create_ex(nmodes, dims, nnz_local, inds, vals, 0, 0, out);
  if (st != SF_OK) return st;
  Tensor* t = reinterpret_cast<Tensor*>(*out);
  t->dist = true;
  t->pos_begin = pos_begin;
  t->nnz_total = nnz_total;
  return SF_OK;
}
