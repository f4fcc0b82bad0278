// sf_comm.cu - multi-GPU boundary exchange and row-block allgather.
//
// The paper is single-GPU; the partitioning here is new.
// Rank p of P owns the matricized positions [floor(p*nnz/P), floor((p+1)*nnz/P)) of every
// mode, so its partial Y touches one contiguous row range [row_begin_p, row_end_p) and
// adjacent ranks share at most the row straddling a cut (a heavy row may straddle several).
// Owner of a row = the lowest rank touching it (it is that rank's LAST row).  Per call:
//   1. every rank allgathers the R-float partial of its first row           (one collective)
//   2. a rank whose first row is owned below zeroes its copy
//   3. the owner adds the senders' partials to its last row, in rank order  (deterministic)
// so the local blocks hold a row-sharded Y -- the layout Alg. 1 line 5's row-local update
// A_n = M V^+ consumes.  A full-Y reduce-scatter would move I_n*R*4 bytes per
// rank; this moves R*4.
//
// Transport: NCCL (dlopen'ed libnccl.so.2: ncclBroadcast per root inside a group = an
// allgatherv, grouped ncclSend/ncclRecv = an alltoallv, on the caller's stream) or the
// caller's allgatherv callback.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "sf_internal.h"

namespace sf {

// ---------------------------------------------------------------------------
// NCCL, loaded at run time (the library must load on hosts without NCCL / without a GPU)
// ---------------------------------------------------------------------------
struct NcclApi {
  bool ok = false;
  std::string err;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

static NcclApi& nccl() {
  static NcclApi api = [] {
    NcclApi a;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
      a.err = std::string("dlopen libnccl.so.2 failed: ") + dlerror();
      return a;
    }
    auto sym = [&](const char* n) { return dlsym(h, n); };
    a.GetUniqueId = reinterpret_cast<decltype(a.GetUniqueId)>(sym("ncclGetUniqueId"));
    a.CommInitRank = reinterpret_cast<decltype(a.CommInitRank)>(sym("ncclCommInitRank"));
    a.CommDestroy = reinterpret_cast<decltype(a.CommDestroy)>(sym("ncclCommDestroy"));
    a.GroupStart = reinterpret_cast<decltype(a.GroupStart)>(sym("ncclGroupStart"));
    a.GroupEnd = reinterpret_cast<decltype(a.GroupEnd)>(sym("ncclGroupEnd"));
    a.Broadcast = reinterpret_cast<decltype(a.Broadcast)>(sym("ncclBroadcast"));
    a.Send = reinterpret_cast<decltype(a.Send)>(sym("ncclSend"));
    a.Recv = reinterpret_cast<decltype(a.Recv)>(sym("ncclRecv"));
    a.GetErrorString = reinterpret_cast<decltype(a.GetErrorString)>(sym("ncclGetErrorString"));
    a.ok = a.GetUniqueId && a.CommInitRank && a.CommDestroy && a.GroupStart && a.GroupEnd && a.Broadcast && a.Send &&
           a.Recv;
    if (!a.ok) a.err = "libnccl.so.2 lacks a required symbol";
    return a;
  }();
  return api;
}

static void nccl_check(ncclResult_t r, const char* what) {
  if (r != ncclSuccess) {
    const char* d = nccl().GetErrorString ? nccl().GetErrorString(r) : "?";
    throw StatusError{SF_ERR_NCCL, std::string(what) + ": " + d};
  }
}

// NCCL communicators are shared by every handle attached with the same (unique id, nranks,
// rank, device): ncclCommInitRank is a collective costing tens to hundreds of ms, and a user
// (or bench.py's e2e leg) creates a handle per tensor.  They live until the process exits: a
// unique id may initialise a communicator only once, so re-attaching with the same id after
// the last handle is gone must find the communicator again, not re-initialise it.
struct NcclHandle {
  ncclComm_t comm = nullptr;
  ~NcclHandle() {
    if (comm && sf::nccl().ok) sf::nccl().CommDestroy(comm);
  }
};

static std::mutex g_comm_mu;
static std::map<std::string, std::shared_ptr<NcclHandle>>* g_comms =
    new std::map<std::string, std::shared_ptr<NcclHandle>>();  // never destroyed (see above)

static std::shared_ptr<NcclHandle> nccl_comm_for(const void* id128, int nranks, int rank, int device) {
  std::string key(static_cast<const char*>(id128), 128);
  key += ":" + std::to_string(nranks) + ":" + std::to_string(rank) + ":" + std::to_string(device);
  std::lock_guard<std::mutex> g(g_comm_mu);
  auto it = g_comms->find(key);
  if (it != g_comms->end()) return it->second;
  NcclApi& api = sf::nccl();
  ncclUniqueId id;
  memcpy(&id, id128, sizeof id);
  auto h = std::make_shared<NcclHandle>();
  nccl_check(api.CommInitRank(&h->comm, nranks, id, rank), "ncclCommInitRank");
  (*g_comms)[key] = h;
  return h;
}

Comm::~Comm() = default;

void Comm::allgatherv(const void* send, void* recv, const uint64_t* bytes, const uint64_t* displs, cudaStream_t s) {
  if (fn) {
    if (fn(ctx, send, recv, bytes, displs, nranks, s) != 0)
      throw StatusError{SF_ERR_NCCL, "caller transport (allgatherv) failed"};
    return;
  }
  NcclApi& api = sf::nccl();
  if (!nccl || !api.ok) throw StatusError{SF_ERR_NCCL, "no NCCL communicator"};
  // allgatherv = one broadcast per root inside a group (every rank receives every block)
  nccl_check(api.GroupStart(), "ncclGroupStart");
  for (int k = 0; k < nranks; ++k) {
    if (bytes[k] == 0) continue;
    char* dst = static_cast<char*>(recv) + displs[k];
    const void* src = (k == rank) ? send : dst;
    nccl_check(api.Broadcast(src, dst, bytes[k], ncclChar, k, static_cast<ncclComm_t>(nccl), s), "ncclBroadcast");
  }
  nccl_check(api.GroupEnd(), "ncclGroupEnd");
}

// alltoallv: block q of `send` (sbytes[q] bytes at sdispl[q]) goes to rank q; the block from
// rank k lands at recv + rdispl[k] (rbytes[k] bytes).  NCCL: grouped ncclSend / ncclRecv.
// Caller transport: emulated with allgatherv (every rank receives every send buffer and keeps
// its blocks -- a test-only cost).
void Comm::alltoallv(const void* send, const uint64_t* sbytes, const uint64_t* sdispl, void* recv,
                     const uint64_t* rbytes, const uint64_t* rdispl, cudaStream_t s) {
  if (!fn) {
    NcclApi& api = sf::nccl();
    if (!nccl || !api.ok) throw StatusError{SF_ERR_NCCL, "no NCCL communicator"};
    nccl_check(api.GroupStart(), "ncclGroupStart");
    for (int q = 0; q < nranks; ++q) {
      if (sbytes[q])
        nccl_check(api.Send(static_cast<const char*>(send) + sdispl[q], sbytes[q], ncclChar, q,
                            static_cast<ncclComm_t>(nccl), s), "ncclSend");
      if (rbytes[q])
        nccl_check(api.Recv(static_cast<char*>(recv) + rdispl[q], rbytes[q], ncclChar, q,
                            static_cast<ncclComm_t>(nccl), s), "ncclRecv");
    }
    nccl_check(api.GroupEnd(), "ncclGroupEnd");
    return;
  }
  // every rank's (sbytes, sdispl) table, then every rank's whole send buffer
  const int P = nranks;
  DevBuf tab((size_t)P * P * 16 + 16);
  std::vector<uint64_t> mine(2 * P), bytes(P, (uint64_t)P * 16), displs(P);
  for (int q = 0; q < P; ++q) { mine[2 * q] = sbytes[q]; mine[2 * q + 1] = sdispl[q]; displs[q] = (uint64_t)q * P * 16; }
  char* tsend = tab.as<char>() + (size_t)rank * P * 16;
  SF_CUDA(cudaMemcpyAsync(tsend, mine.data(), (size_t)P * 16, cudaMemcpyHostToDevice, s));
  allgatherv(tsend, tab.p, bytes.data(), displs.data(), s);
  std::vector<uint64_t> all((size_t)P * P * 2);
  SF_CUDA(cudaMemcpyAsync(all.data(), tab.p, (size_t)P * P * 16, cudaMemcpyDeviceToHost, s));
  SF_CUDA(cudaStreamSynchronize(s));
  std::vector<uint64_t> tot(P), off(P);
  uint64_t sum = 0;
  for (int k = 0; k < P; ++k) {
    uint64_t end = 0;
    for (int q = 0; q < P; ++q) end = std::max(end, all[(size_t)k * 2 * P + 2 * q] + all[(size_t)k * 2 * P + 2 * q + 1]);
    tot[k] = end;
    off[k] = sum;
    sum += end;
  }
  DevBuf big(sum + 16);
  allgatherv(send, big.p, tot.data(), off.data(), s);
  for (int k = 0; k < P; ++k) {
    const uint64_t b = all[(size_t)k * 2 * P + 2 * rank], d = all[(size_t)k * 2 * P + 2 * rank + 1];
    if (b != rbytes[k]) throw StatusError{SF_ERR_NCCL, "alltoallv: receive size mismatch"};
    if (b) SF_CUDA(cudaMemcpyAsync(static_cast<char*>(recv) + rdispl[k], big.as<char>() + off[k] + d, b,
                                   cudaMemcpyDeviceToDevice, s));
  }
  SF_CUDA(cudaStreamSynchronize(s));
}

// ---------------------------------------------------------------------------
// Exchange map (host logic; pinned by tests/test_dist_gloo.py through sf_exchange_map)
// ---------------------------------------------------------------------------
// ranges[2k..2k+1] = [begin, end) rows touched by rank k (begin == end: empty shard).
// Out: send_first[k] (its first row is owned by a lower rank) and, per owner, the ascending
// list of senders.
static void exchange_map(const std::vector<uint64_t>& ranges, int P, std::vector<int>& owner_of_first,
                         std::vector<char>& send_first) {
  owner_of_first.assign(P, -1);
  send_first.assign(P, 0);
  for (int k = 0; k < P; ++k) {
    const uint64_t b = ranges[2 * k], e = ranges[2 * k + 1];
    if (e <= b) continue;
    int o = k;
    for (int j = 0; j < k; ++j)  // lowest rank touching row b
      if (ranges[2 * j + 1] > ranges[2 * j] && ranges[2 * j] <= b && b < ranges[2 * j + 1]) { o = j; break; }
    owner_of_first[k] = o;
    send_first[k] = o != k;
  }
}

void ensure_ranges(Tensor& t, Plan& p, cudaStream_t s) {
  if (!p.ranges.empty()) return;
  const int P = t.nranks;
  if (P == 1 || !t.comm) {
    p.ranges = {p.row_begin, p.row_end};
    return;
  }
  DevBuf buf((size_t)P * 16 + 16);
  uint64_t mine[2] = {p.row_begin, p.row_end};
  std::vector<uint64_t> bytes(P, 16), displs(P);
  for (int k = 0; k < P; ++k) displs[k] = (uint64_t)k * 16;
  char* send = buf.as<char>() + (size_t)t.rank * 16;
  h2d_small(s, send, mine, 16);
  t.comm->allgatherv(send, buf.p, bytes.data(), displs.data(), s);
  std::vector<uint64_t> r(2 * P);
  d2h_small(s, r.data(), buf.p, (size_t)P * 16);
  std::vector<int> owner;
  std::vector<char> sends;
  exchange_map(r, P, owner, sends);
  p.send_first = sends[t.rank];
  p.add_srcs.clear();
  for (int k = 0; k < P; ++k)
    if (sends[k] && owner[k] == t.rank) p.add_srcs.push_back(k);
  p.ranges = std::move(r);
}

// out[row] += recv[src_k] for the senders in rank order (one CTA: R <= 4096 columns).
__global__ void owner_add_kernel(float* __restrict__ row, const float* __restrict__ recv, const int* __restrict__ srcs,
                                 int nsrc, int R) {
  for (int c = threadIdx.x; c < R; c += blockDim.x) {
    float y = row[c];
    for (int k = 0; k < nsrc; ++k) y += recv[(size_t)srcs[k] * R + c];
    row[c] = y;
  }
}

void exchange_rows(Tensor& t, Plan& p, float* out, cudaStream_t s) {
  if (!t.comm || t.nranks == 1) return;
  ensure_ranges(t, p, s);
  const int P = t.nranks, R = p.rank;
  const size_t need = (size_t)(P + 1) * R * 4 + (size_t)P * 4 + 64;
  if (p.xbuf.bytes < need) {
    p.xbuf.alloc(need);
    std::vector<int> srcs(P, 0);
    for (size_t i = 0; i < p.add_srcs.size(); ++i) srcs[i] = p.add_srcs[i];
    h2d_small(s, p.xbuf.as<char>() + (size_t)(P + 1) * R * 4, srcs.data(), (size_t)P * 4);
  }
  float* send = p.xbuf.as<float>();
  float* recv = send + R;
  const int* srcs = reinterpret_cast<const int*>(p.xbuf.as<char>() + (size_t)(P + 1) * R * 4);
  const bool nonempty = p.row_end > p.row_begin;
  if (p.send_first) d2d_copy(send, out, (size_t)R * 4, s);
  std::vector<uint64_t> bytes(P, (uint64_t)R * 4), displs(P);
  for (int k = 0; k < P; ++k) displs[k] = (uint64_t)k * R * 4;
  t.comm->allgatherv(send, recv, bytes.data(), displs.data(), s);
  if (p.send_first) SF_CUDA(cudaMemsetAsync(out, 0, (size_t)R * 4, s));
  if (!p.add_srcs.empty() && nonempty) {
    float* last = out + (p.row_end - 1 - p.row_begin) * (size_t)R;
    owner_add_kernel<<<1, 256, 0, s>>>(last, recv, srcs, (int)p.add_srcs.size(), R);
    count_launch();
    SF_CUDA(cudaGetLastError());
  }
}

void allgather_blocks(Tensor& t, const std::vector<uint64_t>& blk, const float* local, float* full, int R,
                      cudaStream_t s) {
  const int P = t.nranks;
  std::vector<uint64_t> bytes(P), displs(P);
  for (int k = 0; k < P; ++k) {
    bytes[k] = (blk[2 * k + 1] - blk[2 * k]) * (uint64_t)R * 4;
    displs[k] = blk[2 * k] * (uint64_t)R * 4;
  }
  t.comm->allgatherv(local, full, bytes.data(), displs.data(), s);
}

}  // namespace sf

using namespace sf;

template <class F>
static sf_status comm_guard(F&& f) {
  try {
    return f();
  } catch (const CudaError& e) {
    set_error(std::string(e.what) + ": " + cudaGetErrorString(e.err));
    return SF_ERR_CUDA;
  } catch (const StatusError& e) {
    set_error(e.msg);
    return e.st;
  } catch (...) {
    set_error("unknown internal error");
    return SF_ERR_NCCL;
  }
}

extern "C" {

sf_status sf_comm_unique_id(void* id128) {
  return comm_guard([&]() -> sf_status {
    if (!id128) throw StatusError{SF_ERR_INVALID_ARG, "NULL id"};
    NcclApi& api = nccl();
    if (!api.ok) throw StatusError{SF_ERR_NCCL, api.err};
    ncclUniqueId id;
    nccl_check(api.GetUniqueId(&id), "ncclGetUniqueId");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    memcpy(id128, &id, sizeof id);
    return SF_OK;
  });
}

sf_status sf_set_shard(sf_tensor_t h, int nranks, int rank);

sf_status sf_comm_attach(sf_tensor_t h, int nranks, int rank, const void* id128) {
  return comm_guard([&]() -> sf_status {
    if (!h || !id128 || nranks < 1 || rank < 0 || rank >= nranks)
      throw StatusError{SF_ERR_INVALID_ARG, "bad comm arguments"};
    Tensor* t = reinterpret_cast<Tensor*>(h);
    NcclApi& api = nccl();
    if (!api.ok) throw StatusError{SF_ERR_NCCL, api.err};
    SF_CUDA(cudaSetDevice(t->device));
    std::shared_ptr<NcclHandle> c = nccl_comm_for(id128, nranks, rank, t->device);
    const sf_status st = sf_set_shard(h, nranks, rank);
    if (st != SF_OK) return st;
    delete t->comm;
    t->comm = new Comm();
    t->comm->nranks = nranks;
    t->comm->rank = rank;
    t->comm->shared = c;
    t->comm->nccl = c->comm;
    return SF_OK;
  });
}

sf_status sf_comm_attach_transport(sf_tensor_t h, int nranks, int rank, sf_allgatherv_fn fn, void* ctx) {
  return comm_guard([&]() -> sf_status {
    if (!h || !fn || nranks < 1 || rank < 0 || rank >= nranks)
      throw StatusError{SF_ERR_INVALID_ARG, "bad transport arguments"};
    Tensor* t = reinterpret_cast<Tensor*>(h);
    const sf_status st = sf_set_shard(h, nranks, rank);
    if (st != SF_OK) return st;
    delete t->comm;
    t->comm = new Comm();
    t->comm->nranks = nranks;
    t->comm->rank = rank;
    t->comm->fn = fn;
    t->comm->ctx = ctx;
    return SF_OK;
  });
}

sf_status sf_comm_detach(sf_tensor_t h) {
  return comm_guard([&]() -> sf_status {
    if (!h) throw StatusError{SF_ERR_INVALID_ARG, "NULL handle"};
    Tensor* t = reinterpret_cast<Tensor*>(h);
    SF_CUDA(cudaSetDevice(t->device));
    SF_CUDA(cudaDeviceSynchronize());
    delete t->comm;
    t->comm = nullptr;
    for (auto& kv : t->plans) kv.second->ranges.clear();
    return SF_OK;
  });
}

sf_status sf_comm_check(sf_tensor_t h, void* stream) {
  return comm_guard([&]() -> sf_status {
    if (!h) throw StatusError{SF_ERR_INVALID_ARG, "NULL handle"};
    Tensor* t = reinterpret_cast<Tensor*>(h);
    if (!t->comm) throw StatusError{SF_ERR_INVALID_ARG, "no comm attached"};
    SF_CUDA(cudaSetDevice(t->device));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    Comm& c = *t->comm;
    const int P = c.nranks, r = c.rank;
    // allgatherv: rank k contributes k + 1 words k * 1000 + i
    std::vector<uint64_t> bytes(P), displs(P);
    uint64_t tot = 0;
    for (int k = 0; k < P; ++k) {
      bytes[k] = 4ull * (k + 1);
      displs[k] = tot;
      tot += bytes[k];
    }
    std::vector<uint32_t> mine(r + 1), got(tot / 4);
    for (int i = 0; i <= r; ++i) mine[i] = (uint32_t)(r * 1000 + i);
    DevBuf sb(bytes[r] + 16), rb(tot + 16);
    SF_CUDA(cudaMemcpyAsync(sb.p, mine.data(), bytes[r], cudaMemcpyHostToDevice, s));
    SF_CUDA(cudaMemsetAsync(rb.p, 0xff, tot, s));
    c.allgatherv(sb.p, rb.p, bytes.data(), displs.data(), s);
    SF_CUDA(cudaMemcpyAsync(got.data(), rb.p, tot, cudaMemcpyDeviceToHost, s));
    SF_CUDA(cudaStreamSynchronize(s));
    for (int k = 0; k < P; ++k)
      for (int i = 0; i <= k; ++i)
        if (got[displs[k] / 4 + i] != (uint32_t)(k * 1000 + i))
          throw StatusError{SF_ERR_NCCL, "comm check: allgatherv delivered a wrong word"};
    // alltoallv: rank a sends (a + b) % 3 + 1 words a * 1000000 + b * 1000 + i to rank b
    auto nw = [](int a, int b) { return (uint64_t)((a + b) % 3 + 1); };
    std::vector<uint64_t> sbytes(P), sdispl(P), rbytes(P), rdispl(P);
    uint64_t st = 0, rt = 0;
    for (int q = 0; q < P; ++q) {
      sbytes[q] = 4 * nw(r, q);
      sdispl[q] = st;
      st += sbytes[q];
      rbytes[q] = 4 * nw(q, r);
      rdispl[q] = rt;
      rt += rbytes[q];
    }
    std::vector<uint32_t> out(st / 4), in(rt / 4);
    for (int q = 0; q < P; ++q)
      for (uint64_t i = 0; i < nw(r, q); ++i) out[sdispl[q] / 4 + i] = (uint32_t)(r * 1000000 + q * 1000 + i);
    DevBuf sa(st + 16), ra(rt + 16);
    SF_CUDA(cudaMemcpyAsync(sa.p, out.data(), st, cudaMemcpyHostToDevice, s));
    SF_CUDA(cudaMemsetAsync(ra.p, 0xff, rt, s));
    c.alltoallv(sa.p, sbytes.data(), sdispl.data(), ra.p, rbytes.data(), rdispl.data(), s);
    SF_CUDA(cudaMemcpyAsync(in.data(), ra.p, rt, cudaMemcpyDeviceToHost, s));
    SF_CUDA(cudaStreamSynchronize(s));
    for (int k = 0; k < P; ++k)
      for (uint64_t i = 0; i < nw(k, r); ++i)
        if (in[rdispl[k] / 4 + i] != (uint32_t)(k * 1000000 + r * 1000 + i))
          throw StatusError{SF_ERR_NCCL, "comm check: alltoallv delivered a wrong word"};
    return SF_OK;
  });
}

// Host-only: the exchange map for given row ranges (tests pin it against the rule by hand).
// send_first[k] = 1 iff rank k sends its first row; owner[k] = the rank receiving it (-1: empty).
sf_status sf_exchange_map(int nranks, const uint64_t* ranges, int32_t* send_first, int32_t* owner) {
  return comm_guard([&]() -> sf_status {
    if (nranks < 1 || !ranges || !send_first || !owner) throw StatusError{SF_ERR_INVALID_ARG, "bad arguments"};
    std::vector<uint64_t> r(ranges, ranges + 2 * nranks);
    std::vector<int> o;
    std::vector<char> sf_;
    exchange_map(r, nranks, o, sf_);
    for (int k = 0; k < nranks; ++k) {
      send_first[k] = sf_[k];
      owner[k] = o[k];
    }
    return SF_OK;
  });
}

}  // extern "C"
