// sf_api.cu - the C ABI (include/scalfrag.h) and the ingest / stream pipeline.
//
// Ingest (§8(a) A1) and the stream pipeline (§8(a) A8) follow PAPER.md §IV-C
// (L201-229): the COO tensor is cut into equal-nnz contiguous segments (reading R12),
// each segment is transferred asynchronously on its own CUDA stream, and the device
// works on finished segments while later ones are still in flight (here: the index
// range check for the resident path, the nnz-parallel kernel for the one-shot
// streamed path).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <map>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "sf_internal.h"

namespace sf {

// NVTX ranges around every public entry point (visible in nsys / ncu timelines; a no-op
// without a profiler attached).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

std::atomic<uint64_t> g_launches{0};
static thread_local std::string g_err;

void set_error(const std::string& msg) { g_err = msg; }

const char* debug_opt(const char* key) {
  static thread_local std::string val;
  const char* e = std::getenv("SF_DEBUG");
  if (!e || !*e) return nullptr;
  const std::string all(e);
  const size_t klen = strlen(key);
  size_t pos = 0;
  while (pos <= all.size()) {
    size_t end = all.find(',', pos);
    if (end == std::string::npos) end = all.size();
    const std::string item = all.substr(pos, end - pos);
    if (item.compare(0, klen, key) == 0 && (item.size() == klen || item[klen] == '=')) {
      val = item.size() == klen ? std::string() : item.substr(klen + 1);
      return val.c_str();
    }
    pos = end + 1;
  }
  return nullptr;
}

void trace_mark(const char* phase) {
  if (!debug_opt("trace")) return;
  static thread_local std::chrono::steady_clock::time_point last = std::chrono::steady_clock::now();
  const auto now = std::chrono::steady_clock::now();
  fprintf(stderr, "[sf trace] %-24s +%.3f ms\n", phase, std::chrono::duration<double, std::milli>(now - last).count());
  last = now;
}

// Caching device allocator.  cudaMalloc/cudaFree of GB-sized plan arrays cost tens of ms
// each and cudaFree synchronizes the device; blocks are instead kept in a free list keyed by
// (device, size) and reused (best fit within 2x) -- a block is only ever handed back to a
// buffer on the device it was allocated on.  Reuse is stream-safe because every library
// buffer is produced and consumed on the handle's planning stream, or the device is
// synchronized first (plan replacement, sf_set_shard and handle destruction call
// cudaDeviceSynchronize).
struct BlockCache {
  std::mutex mu;
  std::multimap<std::pair<int, size_t>, void*> free_blocks;  // (device, bytes) -> block
  size_t cached = 0;
  void* get(size_t b, size_t* got) {
    int dev = 0;
    SF_CUDA(cudaGetDevice(&dev));
    {
      std::lock_guard<std::mutex> g(mu);
      auto it = free_blocks.lower_bound({dev, b});
      if (it != free_blocks.end() && it->first.first == dev && it->first.second <= 2 * b + (1u << 20)) {
        void* q = it->second;
        *got = it->first.second;
        cached -= it->first.second;
        free_blocks.erase(it);
        return q;
      }
    }
    void* q = nullptr;
    cudaError_t e = cudaMalloc(&q, b);
    if (e != cudaSuccess) {  // give the cache back to the driver and retry once
      cudaGetLastError();
      trim();
      e = cudaMalloc(&q, b);
      if (e != cudaSuccess) {
        cudaGetLastError();
        throw CudaError{e, "cudaMalloc"};
      }
    }
    *got = b;
    return q;
  }
  size_t cached_on(int dev) {
    std::lock_guard<std::mutex> g(mu);
    size_t b = 0;
    for (auto it = free_blocks.lower_bound({dev, 0}); it != free_blocks.end() && it->first.first == dev; ++it)
      b += it->first.second;
    return b;
  }
  void put(void* q, size_t b) {
    int dev = 0;
    cudaPointerAttributes a{};
    if (cudaPointerGetAttributes(&a, q) == cudaSuccess) dev = a.device;
    else cudaGetLastError();
    std::lock_guard<std::mutex> g(mu);
    free_blocks.emplace(std::make_pair(dev, b), q);
    cached += b;
  }
  void trim() {  // every block is freed on its own device, after that device is idle
    std::lock_guard<std::mutex> g(mu);
    int cur = 0;
    cudaGetDevice(&cur);
    int synced = -1;
    for (auto& kv : free_blocks) {
      if (kv.first.first != synced) {
        cudaSetDevice(kv.first.first);
        cudaDeviceSynchronize();
        synced = kv.first.first;
      }
      cudaFree(kv.second);
    }
    cudaSetDevice(cur);
    free_blocks.clear();
    cached = 0;
  }
};
static BlockCache g_cache;

size_t device_free_bytes() {
  size_t free_b = 0, total_b = 0;
  SF_CUDA(cudaMemGetInfo(&free_b, &total_b));
  int dev = 0;
  SF_CUDA(cudaGetDevice(&dev));
  return free_b + g_cache.cached_on(dev);
}

// Bytes held by live library buffers (all devices) and their high-water mark (sf_device_bytes).
static std::atomic<uint64_t> g_in_use{0}, g_peak{0};

void DevBuf::alloc(size_t b) {
  release();
  if (b == 0) b = 16;
  b = (b + 255) & ~(size_t)255;
  size_t got = 0;
  p = g_cache.get(b, &got);
  bytes = got;
  const uint64_t now = g_in_use.fetch_add(got) + got;
  uint64_t pk = g_peak.load();
  while (now > pk && !g_peak.compare_exchange_weak(pk, now)) {
  }
}

void DevBuf::release() {
  if (p) {
    g_cache.put(p, bytes);
    g_in_use.fetch_sub(bytes);
  }
  p = nullptr;
  bytes = 0;
}

// ---- small transfers through mapped pinned memory (no copy engine) ----
__global__ void copy_bytes_kernel(unsigned char* __restrict__ dst, const unsigned char* __restrict__ src, size_t n) {
  for (size_t i = threadIdx.x; i < n; i += blockDim.x) dst[i] = src[i];
}

static unsigned char* staging(size_t need) {
  static thread_local unsigned char* buf = nullptr;
  static thread_local size_t cap = 0;
  if (need > cap) {
    if (buf) cudaFreeHost(buf);
    buf = nullptr;
    cap = std::max<size_t>(need, 1 << 16);
    SF_CUDA(cudaHostAlloc(reinterpret_cast<void**>(&buf), cap, cudaHostAllocMapped | cudaHostAllocPortable));
  }
  return buf;
}

void d2h_small(cudaStream_t s, int n, void* const* dst, const void* const* src, const size_t* bytes) {
  size_t total = 0;
  for (int i = 0; i < n; ++i) total += (bytes[i] + 15) & ~(size_t)15;
  unsigned char* st = staging(total);
  size_t off = 0;
  for (int i = 0; i < n; ++i) {
    if (!bytes[i]) continue;
    copy_bytes_kernel<<<1, 256, 0, s>>>(st + off, static_cast<const unsigned char*>(src[i]), bytes[i]);
    count_launch();
    off += (bytes[i] + 15) & ~(size_t)15;
  }
  SF_CUDA(cudaGetLastError());
  SF_CUDA(cudaStreamSynchronize(s));
  off = 0;
  for (int i = 0; i < n; ++i) {
    if (!bytes[i]) continue;
    memcpy(dst[i], st + off, bytes[i]);
    off += (bytes[i] + 15) & ~(size_t)15;
  }
}

void h2d_small(cudaStream_t s, void* dst, const void* src, size_t bytes) {
  if (!bytes) return;
  unsigned char* st = staging(bytes);
  memcpy(st, src, bytes);
  copy_bytes_kernel<<<1, 256, 0, s>>>(static_cast<unsigned char*>(dst), st, bytes);
  count_launch();
  SF_CUDA(cudaGetLastError());
  SF_CUDA(cudaStreamSynchronize(s));  // the staging buffer is reused by the next call
}

__global__ void d2d_vec_kernel(uint4* __restrict__ dst, const uint4* __restrict__ src, size_t n16) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride) dst[i] = src[i];
}

__global__ void d2d_bytes_kernel(unsigned char* __restrict__ dst, const unsigned char* __restrict__ src, size_t n,
                                 int word) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  if (word) {  // 4-byte aligned
    uint32_t* d = reinterpret_cast<uint32_t*>(dst);
    const uint32_t* q = reinterpret_cast<const uint32_t*>(src);
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n / 4; i += stride) d[i] = q[i];
    for (size_t i = (n / 4) * 4 + (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) dst[i] = src[i];
  } else {
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) dst[i] = src[i];
  }
}

void d2d_copy(void* dst, const void* src, size_t bytes, cudaStream_t s) {
  if (!bytes) return;
  const uintptr_t a = reinterpret_cast<uintptr_t>(dst) | reinterpret_cast<uintptr_t>(src);
  unsigned char* d = static_cast<unsigned char*>(dst);
  const unsigned char* q = static_cast<const unsigned char*>(src);
  size_t done = 0;
  if ((a & 15) == 0 && bytes >= 16) {
    const size_t n16 = bytes / 16;
    d2d_vec_kernel<<<(int)std::max<size_t>(1, std::min<size_t>((n16 + 255) / 256, 148 * 8)), 256, 0, s>>>(
        reinterpret_cast<uint4*>(d), reinterpret_cast<const uint4*>(q), n16);
    count_launch();
    done = n16 * 16;
  }
  if (done < bytes) {
    const size_t rest = bytes - done;
    const int word = ((a & 3) == 0) ? 1 : 0;
    d2d_bytes_kernel<<<(int)std::max<size_t>(1, std::min<size_t>((rest / 4 + 255) / 256, 148 * 8)), 256, 0, s>>>(
        d + done, q + done, rest, word);
    count_launch();
  }
  SF_CUDA(cudaGetLastError());
}

size_t Plan::device_bytes() const {
  size_t b = val.bytes + rec.bytes + perm.bytes + chunk_begin.bytes + chunk_tile.bytes + tile_chunk.bytes +
             hot_cache.bytes;
  for (int m = 0; m < SF_MAX_MODES; ++m) b += ind[m].bytes + hot_rows[m].bytes;
  return b;
}

Tensor::~Tensor() {
  for (auto& kv : plans) delete kv.second;
  plans.clear();
  for (int m = 0; m < SF_MAX_MODES; ++m) {
    delete sub[m];
    sub[m] = nullptr;
  }
  delete comm;
  comm = nullptr;
  if (stream) cudaStreamDestroy(stream);
}

template <class F>
static sf_status guard(F&& f) {
  try {
    return f();
  } catch (const CudaError& e) {
    set_error(std::string(e.what) + ": " + cudaGetErrorString(e.err));
    return (e.err == cudaErrorMemoryAllocation) ? SF_ERR_OUT_OF_MEMORY : SF_ERR_CUDA;
  } catch (const StatusError& e) {
    set_error(e.msg);
    return e.st;
  } catch (const std::bad_alloc&) {
    set_error("host allocation failed");
    return SF_ERR_OUT_OF_MEMORY;
  } catch (...) {
    set_error("unknown internal error");
    return SF_ERR_CUDA;
  }
}

static bool is_device_ptr(const void* p) {
  cudaPointerAttributes a{};
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

static bool is_pinned_ptr(const void* p) {
  cudaPointerAttributes a{};
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeHost;
}

// Segmented, multi-stream upload of the (N+1) COO arrays into the tensor's device
// arrays, with the range check of each segment enqueued behind its copy.
static void upload(Tensor& t, const uint32_t* const* inds, const float* vals, int segments,
                   int nstreams, int* d_flag) {
  const int N = t.nmodes;
  const uint64_t n = t.nnz;
  if (segments <= 0) segments = 8;
  if (nstreams <= 0) nstreams = 4;
  segments = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)segments, std::max<uint64_t>(1, n)));
  nstreams = std::max(1, std::min(nstreams, segments));
  std::vector<cudaStream_t> st(nstreams);
  for (auto& s : st) SF_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  bool pageable = false;
  for (int m = 0; m < N && !pageable; ++m) pageable = !is_pinned_ptr(inds[m]);
  if (!pageable) pageable = !is_pinned_ptr(vals);
  const uint64_t seg_len = (n + segments - 1) / segments;
  // pinned staging ring for pageable input: one slot per stream
  std::vector<void*> stage(nstreams, nullptr);
  std::vector<cudaEvent_t> done(nstreams, nullptr);
  // A8: each segment's matricized keys are sorted on its stream behind its copy (presort)
  const bool presort = presort_begin(t, seg_len);
  std::vector<DevBuf> ptemp(presort ? nstreams : 0);
  size_t ptemp_bytes = 0;
  if (presort) {
    ptemp_bytes = presort_temp_bytes(t, seg_len);
    for (auto& b : ptemp) b.alloc(ptemp_bytes + 16);
  }
  const Ingest ingest = ingest_begin(t);
  try {
    if (pageable) {
      for (int s = 0; s < nstreams; ++s) {
        SF_CUDA(cudaMallocHost(&stage[s], (size_t)seg_len * 4 * (N + 1) + 64));
        SF_CUDA(cudaEventCreateWithFlags(&done[s], cudaEventDisableTiming));
      }
    }
    for (int k = 0; k < segments; ++k) {
      const uint64_t a = (uint64_t)k * seg_len;
      if (a >= n) break;
      const uint64_t b = std::min(n, a + seg_len);
      const uint64_t len = b - a;
      const int s = k % nstreams;
      uint32_t* dseg[SF_MAX_MODES];
      for (int m = 0; m < N; ++m) dseg[m] = t.ind[m].as<uint32_t>() + a;
      if (pageable) {
        if (k >= nstreams) SF_CUDA(cudaEventSynchronize(done[s]));  // slot free again
        char* h = static_cast<char*>(stage[s]);
        for (int m = 0; m < N; ++m) {
          memcpy(h + (size_t)m * len * 4, inds[m] + a, len * 4);
          SF_CUDA(cudaMemcpyAsync(dseg[m], h + (size_t)m * len * 4, len * 4, cudaMemcpyHostToDevice, st[s]));
        }
        memcpy(h + (size_t)N * len * 4, vals + a, len * 4);
        SF_CUDA(cudaMemcpyAsync(t.val.as<float>() + a, h + (size_t)N * len * 4, len * 4,
                                cudaMemcpyHostToDevice, st[s]));
        SF_CUDA(cudaEventRecord(done[s], st[s]));
      } else {
        for (int m = 0; m < N; ++m)
          SF_CUDA(cudaMemcpyAsync(dseg[m], inds[m] + a, len * 4, cudaMemcpyHostToDevice, st[s]));
        SF_CUDA(cudaMemcpyAsync(t.val.as<float>() + a, vals + a, len * 4, cudaMemcpyHostToDevice, st[s]));
      }
      validate_indices(N, t.dims, len, dseg, d_flag, st[s]);
      if (presort) presort_segment(t, a, len, st[s], ptemp[s].p, ptemp_bytes);
      ingest_segment(t, ingest, a, len, st[s]);
    }
    for (auto& s : st) SF_CUDA(cudaStreamSynchronize(s));
    t.pre_alt.release();
  } catch (...) {
    for (auto& s : st) cudaStreamSynchronize(s);
    for (auto& s : st) cudaStreamDestroy(s);
    for (auto& p : stage) if (p) cudaFreeHost(p);
    for (auto& e : done) if (e) cudaEventDestroy(e);
    throw;
  }
  for (auto& s : st) cudaStreamDestroy(s);
  for (auto& p : stage) if (p) cudaFreeHost(p);
  for (auto& e : done) if (e) cudaEventDestroy(e);
}

static Tensor* as_tensor(sf_tensor_t h) { return reinterpret_cast<Tensor*>(h); }

static void check_mode_rank(const Tensor& t, int mode, int rank) {
  if (mode < 0 || mode >= t.nmodes) throw StatusError{SF_ERR_INVALID_ARG, "mode out of range"};
  if (rank < 1 || rank > 4096) throw StatusError{SF_ERR_INVALID_ARG, "rank out of range [1, 4096]"};
}

static Plan* get_plan(Tensor& t, int mode, int rank) {
  auto it = t.plans.find({mode, rank});
  return it == t.plans.end() ? nullptr : it->second;
}

// The tensor a plan of `mode` is built from: the handle itself, or -- for a distributed
// handle (sf_tensor_create_dist) with several ranks -- this rank's shard of the mode, gathered
// from every rank (sf_dist.cu), planned as a one-rank tensor.
static Tensor& plan_source(Tensor& t, int mode) {
  if (!t.dist || t.nranks == 1) return t;
  dist_build_sub(t, mode);
  return *t.sub[mode];
}

static void make_plan(Tensor& t, int mode, int rank, const sf_launch_t* override_launch) {
  trace_mark("plan: enter");
  SF_CUDA(cudaSetDevice(t.device));
  Tensor& src = plan_source(t, mode);
  sf_features_t f;
  DevBuf keys, pos;  // the matricized order, sorted once for features + the plan
  compute_features(src, mode, &f, &keys, &pos);
  trace_mark("plan: features");
  const uint64_t lo = (uint64_t)(((unsigned __int128)src.rank * src.nnz) / src.nranks);
  const uint64_t hi = (uint64_t)(((unsigned __int128)(src.rank + 1) * src.nnz) / src.nranks);
  sf_launch_t l;
  if (override_launch && override_launch->kernel != SF_KERNEL_AUTO) {
    l = *override_launch;
    normalize_launch(src, mode, rank, l);
  } else {
    // the hot+tile rule compares how well each candidate's rows would cache (row frequencies of
    // the whole handle; for a v1 shard a proxy of its own)
    for (int m = 0; m < src.nmodes; ++m)
      if (hot_tile_candidate(src, mode, rank, m)) hot_coverage(src, m, (16ull << 20) / (4ull * rank));
    l = select_launch(src, f, mode, rank, hi - lo);
  }
  if (l.kernel == SF_KERNEL_FRAG && frag_smem_bytes(src, mode, rank, l) > src.smem_optin)
    throw StatusError{SF_ERR_INVALID_ARG, "launch needs more shared memory than the device has"};
  trace_mark("plan: select");
  Plan* p = new Plan();
  try {
    build_plan(src, *p, mode, rank, l, &keys, &pos);
    if (&src != &t) {  // a distributed shard writes its local row block like any shard
      p->out_row0 = p->row_begin;
      p->out_rows = p->row_end - p->row_begin;
    }
    trace_mark("plan: build");
  } catch (...) {
    delete p;
    throw;
  }
  Plan* old = get_plan(t, mode, rank);
  if (old) {
    SF_CUDA(cudaDeviceSynchronize());  // in-flight sf_mttkrp may still read the old plan
    delete old;
  }
  t.plans[{mode, rank}] = p;
}

}  // namespace sf

using namespace sf;

extern "C" {

sf_status sf_tensor_create_ex(int nmodes, const uint64_t* dims, uint64_t nnz,
                              const uint32_t* const* inds, const float* vals, int segments,
                              int streams, sf_tensor_t* out) {
  NvtxRange nvtx_("sf_tensor_create_ex");
  return guard([&]() -> sf_status {
    if (!out) throw StatusError{SF_ERR_INVALID_ARG, "out is NULL"};
    *out = nullptr;
    if (nmodes < 2 || nmodes > SF_MAX_MODES || !dims)
      throw StatusError{SF_ERR_INVALID_ARG, "nmodes must be in [2, 8] and dims non-NULL"};
    for (int m = 0; m < nmodes; ++m)
      if (dims[m] < 1 || dims[m] > 0xFFFFFFFFull)
        throw StatusError{SF_ERR_INVALID_ARG, "dims[m] must be in [1, 2^32-1]"};
    if (nnz > 0 && (!inds || !vals)) throw StatusError{SF_ERR_INVALID_ARG, "inds/vals NULL"};
    if (nnz > 0xFFFFFFFFull)  // plans store input positions and slots as uint32
      throw StatusError{SF_ERR_UNSUPPORTED, "nnz must be < 2^32 (input positions are uint32)"};
    if (nnz > 0)
      for (int m = 0; m < nmodes; ++m)
        if (!inds[m]) throw StatusError{SF_ERR_INVALID_ARG, "inds[m] is NULL"};
    Tensor* t = new Tensor();
    try {
      SF_CUDA(cudaGetDevice(&t->device));
      SF_CUDA(cudaDeviceGetAttribute(&t->num_sms, cudaDevAttrMultiProcessorCount, t->device));
      int optin = 0;
      SF_CUDA(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, t->device));
      t->smem_optin = (size_t)optin;
      SF_CUDA(cudaStreamCreateWithFlags(&t->stream, cudaStreamNonBlocking));
      t->nmodes = nmodes;
      t->nnz = nnz;
      for (int m = 0; m < nmodes; ++m) {
        t->dims[m] = dims[m];
        t->ind[m].alloc(nnz * 4 + kPadBytes);
      }
      t->val.alloc(nnz * 4 + kPadBytes);
      DevBuf flag(16);
      SF_CUDA(cudaMemsetAsync(flag.p, 0, 16, t->stream));
      SF_CUDA(cudaStreamSynchronize(t->stream));
      if (nnz > 0) {
        bool dev = is_device_ptr(vals);
        for (int m = 0; m < nmodes; ++m) dev = dev && is_device_ptr(inds[m]);
        if (dev) {
          for (int m = 0; m < nmodes; ++m)
            SF_CUDA(cudaMemcpyAsync(t->ind[m].p, inds[m], nnz * 4, cudaMemcpyDeviceToDevice, t->stream));
          SF_CUDA(cudaMemcpyAsync(t->val.p, vals, nnz * 4, cudaMemcpyDeviceToDevice, t->stream));
          uint32_t* di[SF_MAX_MODES];
          for (int m = 0; m < nmodes; ++m) di[m] = t->ind[m].as<uint32_t>();
          validate_indices(nmodes, t->dims, nnz, di, flag.as<int>(), t->stream);
        } else {
          upload(*t, inds, vals, segments, streams, flag.as<int>());
        }
      }
      int bad = 0;
      SF_CUDA(cudaMemcpyAsync(&bad, flag.p, 4, cudaMemcpyDeviceToHost, t->stream));
      SF_CUDA(cudaStreamSynchronize(t->stream));
      if (bad) throw StatusError{SF_ERR_INDEX_OUT_OF_RANGE, "some index is >= its dimension"};
    } catch (...) {
      delete t;
      throw;
    }
    *out = reinterpret_cast<sf_tensor_t>(t);
    return SF_OK;
  });
}

sf_status sf_tensor_create(int nmodes, const uint64_t* dims, uint64_t nnz,
                           const uint32_t* const* inds, const float* vals, sf_tensor_t* out) {
  return sf_tensor_create_ex(nmodes, dims, nnz, inds, vals, 0, 0, out);
}

sf_status sf_tensor_destroy(sf_tensor_t h) {
  return guard([&]() -> sf_status {
    if (!h) return SF_OK;
    Tensor* t = as_tensor(h);
    cudaSetDevice(t->device);
    cudaDeviceSynchronize();  // kernels on caller streams may still read the arrays
    delete t;
    return SF_OK;
  });
}

sf_status sf_set_shard(sf_tensor_t h, int nranks, int rank) {
  return guard([&]() -> sf_status {
    if (!h) throw StatusError{SF_ERR_INVALID_ARG, "NULL handle"};
    if (nranks < 1 || rank < 0 || rank >= nranks) throw StatusError{SF_ERR_INVALID_ARG, "bad shard"};
    Tensor* t = as_tensor(h);
    if (!t->plans.empty()) {  // an in-flight sf_mttkrp may still read the plans' buffers
      SF_CUDA(cudaSetDevice(t->device));
      SF_CUDA(cudaDeviceSynchronize());
    }
    for (auto& kv : t->plans) delete kv.second;
    t->plans.clear();
    for (int m = 0; m < SF_MAX_MODES; ++m) {  // distributed shards depend on (nranks, rank)
      delete t->sub[m];
      t->sub[m] = nullptr;
      t->sub_gpos[m].release();
    }
    t->nranks = nranks;
    t->rank = rank;
    return SF_OK;
  });
}

sf_status sf_plan(sf_tensor_t h, int mode, int rank) {
  NvtxRange nvtx_("sf_plan");
  return guard([&]() -> sf_status {
    if (!h) throw StatusError{SF_ERR_INVALID_ARG, "NULL handle"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    if (get_plan(*t, mode, rank)) return SF_OK;
    make_plan(*t, mode, rank, nullptr);
    return SF_OK;
  });
}

sf_status sf_plan_release(sf_tensor_t h, int mode, int rank) {
  NvtxRange nvtx_("sf_plan_release");
  return guard([&]() -> sf_status {
    if (!h) throw StatusError{SF_ERR_INVALID_ARG, "NULL handle"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    auto it = t->plans.find({mode, rank});
    if (it != t->plans.end()) {
      SF_CUDA(cudaSetDevice(t->device));
      SF_CUDA(cudaDeviceSynchronize());
      delete it->second;
      t->plans.erase(it);
    }
    return SF_OK;
  });
}

sf_status sf_trim_cache(void) {
  return guard([&]() -> sf_status {
    g_cache.trim();
    return SF_OK;
  });
}

sf_status sf_set_launch(sf_tensor_t h, int mode, int rank, const sf_launch_t* launch) {
  NvtxRange nvtx_("sf_set_launch");
  return guard([&]() -> sf_status {
    if (!h || !launch) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    make_plan(*t, mode, rank, launch);
    return SF_OK;
  });
}

sf_status sf_features(sf_tensor_t h, int mode, sf_features_t* out) {
  return guard([&]() -> sf_status {
    if (!h || !out) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, 1);
    SF_CUDA(cudaSetDevice(t->device));
    compute_features(plan_source(*t, mode), mode, out, nullptr, nullptr);
    return SF_OK;
  });
}

sf_status sf_plan_info(sf_tensor_t h, int mode, int rank, sf_plan_info_t* out) {
  return guard([&]() -> sf_status {
    if (!h || !out) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    Plan* p = get_plan(*t, mode, rank);
    if (!p) throw StatusError{SF_ERR_NOT_PLANNED, "sf_plan(mode, rank) has not been called"};
    memset(out, 0, sizeof(*out));
    out->feat = p->feat;
    out->launch = p->launch;
    out->nnz_local = p->nnz_local;
    out->num_tiles = p->num_tiles;
    out->num_chunks = p->num_chunks;
    out->row_begin = p->row_begin;
    out->row_end = p->row_end;
    out->out_row0 = p->out_row0;
    out->out_rows = p->out_rows;
    out->device_bytes = p->device_bytes();
    out->plan_ms = p->plan_ms;
    return SF_OK;
  });
}

sf_status sf_plan_export(sf_tensor_t h, int mode, int rank, uint64_t* perm_host, uint64_t* chunks_host) {
  return guard([&]() -> sf_status {
    if (!h) throw StatusError{SF_ERR_INVALID_ARG, "NULL handle"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    Plan* p = get_plan(*t, mode, rank);
    if (!p) throw StatusError{SF_ERR_NOT_PLANNED, "sf_plan(mode, rank) has not been called"};
    SF_CUDA(cudaSetDevice(t->device));
    if (perm_host && p->nnz_local) {
      std::vector<uint32_t> tmp(p->nnz_local);
      SF_CUDA(cudaMemcpy(tmp.data(), p->perm.p, p->nnz_local * 4, cudaMemcpyDeviceToHost));
      if (t->sub[mode] && t->dist && t->nranks > 1) {  // shard positions -> global input positions
        std::vector<uint32_t> g(t->sub[mode]->nnz);
        SF_CUDA(cudaMemcpy(g.data(), t->sub_gpos[mode].p, g.size() * 4, cudaMemcpyDeviceToHost));
        for (uint64_t k = 0; k < p->nnz_local; ++k) perm_host[k] = g[tmp[k]];
      } else {
        for (uint64_t k = 0; k < p->nnz_local; ++k) perm_host[k] = tmp[k];
      }
    }
    if (chunks_host && p->num_chunks) {
      std::vector<uint32_t> b(p->num_chunks + 1);
      std::vector<uint64_t> tl(p->num_chunks);
      SF_CUDA(cudaMemcpy(b.data(), p->chunk_begin.p, (p->num_chunks + 1) * 4, cudaMemcpyDeviceToHost));
      SF_CUDA(cudaMemcpy(tl.data(), p->chunk_tile.p, p->num_chunks * 8, cudaMemcpyDeviceToHost));
      for (uint64_t j = 0; j < p->num_chunks; ++j) {
        chunks_host[3 * j] = b[j];
        chunks_host[3 * j + 1] = b[j + 1];
        chunks_host[3 * j + 2] = tl[j];
      }
    }
    return SF_OK;
  });
}

sf_status sf_mttkrp(sf_tensor_t h, int mode, const float* const* factors, int rank, float* out,
                    void* stream) {
  NvtxRange nvtx_("sf_mttkrp");
  return guard([&]() -> sf_status {
    if (!h || !factors || !out) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    Plan* p = get_plan(*t, mode, rank);
    if (!p) throw StatusError{SF_ERR_NOT_PLANNED, "sf_plan(mode, rank) has not been called"};
    for (int m = 0; m < t->nmodes; ++m)
      if (m != mode && !factors[m]) throw StatusError{SF_ERR_INVALID_ARG, "factors[m] is NULL"};
    launch_mttkrp(*t, *p, factors, out, static_cast<cudaStream_t>(stream));
    exchange_rows(*t, *p, out, static_cast<cudaStream_t>(stream));
    return SF_OK;
  });
}

sf_status sf_shard_rows(sf_tensor_t h, int mode, int rank, uint64_t* row_begin, uint64_t* row_end) {
  return guard([&]() -> sf_status {
    if (!h || !row_begin || !row_end) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    Plan* p = get_plan(*t, mode, rank);
    if (!p) throw StatusError{SF_ERR_NOT_PLANNED, "sf_plan(mode, rank) has not been called"};
    *row_begin = p->out_row0;
    *row_end = p->out_row0 + p->out_rows;
    return SF_OK;
  });
}

sf_status sf_allgather_rows(sf_tensor_t h, int mode, int rank, const float* local, float* full, void* stream) {
  NvtxRange nvtx_("sf_allgather_rows");
  return guard([&]() -> sf_status {
    if (!h || !full || !local) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    Plan* p = get_plan(*t, mode, rank);
    if (!p) throw StatusError{SF_ERR_NOT_PLANNED, "sf_plan(mode, rank) has not been called"};
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    SF_CUDA(cudaMemsetAsync(full, 0, sizeof(float) * (size_t)rank * t->dims[mode], s));
    if (t->nranks == 1 || !t->comm) {
      if (t->nranks > 1) throw StatusError{SF_ERR_INVALID_ARG, "sharded handle without a comm"};
      SF_CUDA(cudaMemcpyAsync(full, local, sizeof(float) * (size_t)rank * t->dims[mode], cudaMemcpyDeviceToDevice, s));
      return SF_OK;
    }
    ensure_ranges(*t, *p, s);
    const int P = t->nranks;
    std::vector<int32_t> sendf(P), owner(P);
    sf_exchange_map(P, p->ranges.data(), sendf.data(), owner.data());
    std::vector<uint64_t> blk(2 * P);  // owned rows of every rank
    for (int k = 0; k < P; ++k) {
      const uint64_t b = p->ranges[2 * k], e = p->ranges[2 * k + 1];
      blk[2 * k] = e > b ? b + (uint64_t)sendf[k] : b;
      blk[2 * k + 1] = std::max(blk[2 * k], e);
    }
    allgather_blocks(*t, blk, local + (size_t)sendf[t->rank] * rank, full, rank, s);
    return SF_OK;
  });
}

// One-shot streamed MTTKRP of every mode n with outs[n] != NULL (A8 (ii)): each segment of the
// host COO is uploaded once and, on the same stream, range-checked, copied into AoS records,
// and for every requested mode sorted by i_n and reduced (or, other ranks, one atomic per
// nonzero); segment k+1's upload overlaps segment k's work.
static void streamed_impl(int nmodes, const uint64_t* dims, uint64_t nnz, const uint32_t* const* inds_host,
                          const float* vals_host, const float* const* factors, int rank, float* const* outs,
                          int segments, int streams, cudaStream_t after) {
  if (nmodes < 2 || nmodes > SF_MAX_MODES || !dims || !factors || !outs)
    throw StatusError{SF_ERR_INVALID_ARG, "bad arguments"};
  if (rank < 1) throw StatusError{SF_ERR_INVALID_ARG, "bad rank"};
  if (nnz > 0 && (!inds_host || !vals_host)) throw StatusError{SF_ERR_INVALID_ARG, "NULL COO"};
  uint32_t todo = 0;
  for (int n = 0; n < nmodes; ++n)
    if (outs[n]) todo |= 1u << n;
  if (!todo) throw StatusError{SF_ERR_INVALID_ARG, "no output mode"};
  for (int m = 0; m < nmodes; ++m)
    if ((todo & ~(1u << m)) && !factors[m]) throw StatusError{SF_ERR_INVALID_ARG, "factors[m] is NULL"};
  // segments <= 0: about 5 M nonzeros per segment, 2..32 (every segment costs ~5 + 4 x modes
  // launches, which dominate below ~10 M nonzeros; profiles/r02/s3/stream_study_all_modes.jsonl)
  if (segments <= 0) segments = (int)std::min<uint64_t>(32, std::max<uint64_t>(2, (nnz + 2500000) / 5000000));
  if (streams <= 0) streams = segments <= 2 ? 2 : 4;
  segments = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)segments, std::max<uint64_t>(1, nnz)));
  streams = std::max(1, std::min(streams, segments));
  const uint64_t seg_len = (nnz + segments - 1) / segments;
  // sorted segments (A8 (ii) + pre-reduction): rank 16/32/64 (nmodes <= 7) sort every segment
  // by i_n on the device and reduce runs in registers; other ranks keep one atomic per nonzero
  const bool sorted = seg_sorted_supported(rank) && nmodes <= 7;
  auto bits_of = [&](int n) {
    int kb = 1;
    for (uint64_t x = dims[n] - 1; x; x >>= 1) ++kb;
    return kb;
  };
  int kbits = 1;
  for (int n = 0; n < nmodes; ++n)
    if (todo >> n & 1) kbits = std::max(kbits, bits_of(n));
  const size_t A = 64;
  auto al = [&](size_t b) { return (b + A - 1) & ~(A - 1); };
  const size_t raw_bytes = al((size_t)seg_len * 4) * (nmodes + 1);
  const int W = seg_aos_words(nmodes);
  const size_t aos_bytes = sorted ? al((size_t)seg_len * 4 * W) : 0;
  const size_t sort_temp = sorted ? seg_sort_temp_bytes(seg_len, kbits) : 0;
  const size_t sort_bytes = sorted ? 3 * al((size_t)seg_len * 4) + sort_temp : 0;
  std::vector<cudaStream_t> st(streams);
  for (auto& s : st) SF_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  std::vector<DevBuf> ring;
  DevBuf flag(16);
  cudaEvent_t zeroed = nullptr, before = nullptr;
  try {
    ring.reserve(streams);
    for (int s = 0; s < streams; ++s) ring.emplace_back(raw_bytes + aos_bytes + sort_bytes + A);
    SF_CUDA(cudaEventCreateWithFlags(&zeroed, cudaEventDisableTiming));
    if (after) {  // work already queued on the caller's stream (e.g. the factor uploads) first
      SF_CUDA(cudaEventCreateWithFlags(&before, cudaEventDisableTiming));
      SF_CUDA(cudaEventRecord(before, after));
      SF_CUDA(cudaStreamWaitEvent(st[0], before, 0));
    }
    SF_CUDA(cudaMemsetAsync(flag.p, 0, 16, st[0]));
    for (int n = 0; n < nmodes; ++n)
      if (todo >> n & 1) SF_CUDA(cudaMemsetAsync(outs[n], 0, sizeof(float) * dims[n] * (size_t)rank, st[0]));
    SF_CUDA(cudaEventRecord(zeroed, st[0]));
    for (int s = 1; s < streams; ++s) SF_CUDA(cudaStreamWaitEvent(st[s], zeroed, 0));
    if (sorted)  // the payload of every segment sort: positions 0 .. seg_len-1
      for (int s = 0; s < streams; ++s)
        launch_iota(reinterpret_cast<uint32_t*>(ring[s].as<char>() + raw_bytes + aos_bytes + 2 * al(seg_len * 4)),
                    seg_len, st[s]);
    for (int k = 0; k < segments; ++k) {
      const uint64_t a = (uint64_t)k * seg_len;
      if (a >= nnz) break;
      const uint64_t len = std::min(nnz, a + seg_len) - a;
      const int s = k % streams;
      char* base = ring[s].as<char>();
      uint32_t* di[SF_MAX_MODES];
      for (int m = 0; m < nmodes; ++m) {
        di[m] = reinterpret_cast<uint32_t*>(base + (size_t)m * al(seg_len * 4));
        SF_CUDA(cudaMemcpyAsync(di[m], inds_host[m] + a, len * 4, cudaMemcpyHostToDevice, st[s]));
      }
      float* dv = reinterpret_cast<float*>(base + (size_t)nmodes * al(seg_len * 4));
      SF_CUDA(cudaMemcpyAsync(dv, vals_host + a, len * 4, cudaMemcpyHostToDevice, st[s]));
      validate_indices(nmodes, dims, len, di, flag.as<int>(), st[s]);
      if (sorted) {
        uint32_t* aos = reinterpret_cast<uint32_t*>(base + raw_bytes);
        char* sb = base + raw_bytes + aos_bytes;
        uint32_t* skey = reinterpret_cast<uint32_t*>(sb);
        uint32_t* spos = reinterpret_cast<uint32_t*>(sb + al(seg_len * 4));
        const uint32_t* iota = reinterpret_cast<const uint32_t*>(sb + 2 * al(seg_len * 4));
        void* temp = sb + 3 * al(seg_len * 4);
        launch_seg_aos(nmodes, len, di, dv, aos, st[s]);
        for (int n = 0; n < nmodes; ++n) {
          if (!(todo >> n & 1)) continue;
          seg_sort(di[n], skey, iota, spos, len, bits_of(n), temp, sort_temp, st[s]);
          launch_seg_sorted(nmodes, dims, len, aos, skey, spos, factors, rank, n, outs[n], st[s]);
        }
      } else {
        for (int n = 0; n < nmodes; ++n)
          if (todo >> n & 1) launch_coo(nmodes, dims, len, di, dv, factors, rank, n, outs[n], st[s]);
      }
    }
    for (auto& s : st) SF_CUDA(cudaStreamSynchronize(s));
    int bad = 0;
    SF_CUDA(cudaMemcpy(&bad, flag.p, 4, cudaMemcpyDeviceToHost));
    for (auto& s : st) cudaStreamDestroy(s);
    st.clear();  // (the handler below must not destroy them again)
    cudaEventDestroy(zeroed);
    zeroed = nullptr;
    if (before) cudaEventDestroy(before);
    before = nullptr;
    if (bad) throw StatusError{SF_ERR_INDEX_OUT_OF_RANGE, "some index is >= its dimension"};
  } catch (...) {
    for (auto& s : st) { cudaStreamSynchronize(s); cudaStreamDestroy(s); }
    if (zeroed) cudaEventDestroy(zeroed);
    if (before) cudaEventDestroy(before);
    throw;
  }
}

sf_status sf_mttkrp_streamed(int nmodes, const uint64_t* dims, uint64_t nnz,
                             const uint32_t* const* inds_host, const float* vals_host,
                             const float* const* factors, int rank, int mode, float* out,
                             int segments, int streams) {
  NvtxRange nvtx_("sf_mttkrp_streamed");
  return guard([&]() -> sf_status {
    if (nmodes < 2 || nmodes > SF_MAX_MODES || !out) throw StatusError{SF_ERR_INVALID_ARG, "bad arguments"};
    if (mode < 0 || mode >= nmodes) throw StatusError{SF_ERR_INVALID_ARG, "bad mode/rank"};
    float* outs[SF_MAX_MODES] = {};
    outs[mode] = out;
    streamed_impl(nmodes, dims, nnz, inds_host, vals_host, factors, rank, outs, segments, streams, nullptr);
    return SF_OK;
  });
}

sf_status sf_mttkrp_streamed_modes(int nmodes, const uint64_t* dims, uint64_t nnz,
                                   const uint32_t* const* inds_host, const float* vals_host,
                                   const float* const* factors, int rank, float* const* outs,
                                   int segments, int streams, void* stream) {
  NvtxRange nvtx_("sf_mttkrp_streamed_modes");
  return guard([&]() -> sf_status {
    streamed_impl(nmodes, dims, nnz, inds_host, vals_host, factors, rank, outs, segments, streams,
                  static_cast<cudaStream_t>(stream));
    return SF_OK;
  });
}

sf_status sf_rows_op(float* Y, int rank, const int64_t* rows, float* buf, int count, int op,
                     void* stream) {
  return guard([&]() -> sf_status {
    if (count < 0 || rank < 1 || op < 0 || op > 2) throw StatusError{SF_ERR_INVALID_ARG, "bad rows_op args"};
    if (count == 0) return SF_OK;
    if (!Y || !rows || (op != 2 && !buf)) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    launch_rows_op(Y, rank, rows, buf, count, op, static_cast<cudaStream_t>(stream));
    return SF_OK;
  });
}

sf_status sf_cpals(sf_tensor_t h, int rank, float* const* factors, int iters, double tol, double* fits,
                   int* iters_done, void* stream) {
  NvtxRange nvtx_("sf_cpals");
  return guard([&]() -> sf_status {
    if (!h || !factors || iters < 0) throw StatusError{SF_ERR_INVALID_ARG, "bad arguments"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, 0, rank);
    if (t->nranks != 1 && !t->comm)
      throw StatusError{SF_ERR_INVALID_ARG, "sf_cpals: a sharded handle needs sf_comm_attach*"};
    for (int m = 0; m < t->nmodes; ++m)
      if (!factors[m]) throw StatusError{SF_ERR_INVALID_ARG, "factors[m] is NULL"};
    SF_CUDA(cudaSetDevice(t->device));
    Plan* plans[SF_MAX_MODES];
    for (int m = 0; m < t->nmodes; ++m) {
      if (!get_plan(*t, m, rank)) make_plan(*t, m, rank, nullptr);
      plans[m] = get_plan(*t, m, rank);
    }
    if (iters_done) *iters_done = 0;
    cpals(*t, rank, factors, iters, tol, fits, iters_done, static_cast<cudaStream_t>(stream), plans);
    return SF_OK;
  });
}

sf_status sf_selector_features(sf_tensor_t h, int mode, int rank, double* x, int* n) {
  return guard([&]() -> sf_status {
    if (!h || !x || !n) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    SF_CUDA(cudaSetDevice(t->device));
    sf_features_t f;
    Tensor& src = plan_source(*t, mode);
    compute_features(src, mode, &f, nullptr, nullptr);
    const uint64_t lo = (uint64_t)(((unsigned __int128)src.rank * src.nnz) / src.nranks);
    const uint64_t hi = (uint64_t)(((unsigned __int128)(src.rank + 1) * src.nnz) / src.nranks);
    *n = selector_features(src, f, mode, rank, hi - lo, x);
    return SF_OK;
  });
}

sf_status sf_selector_candidates(sf_tensor_t h, int mode, int rank, sf_launch_t* out, int* n) {
  return guard([&]() -> sf_status {
    if (!h || !out || !n) throw StatusError{SF_ERR_INVALID_ARG, "NULL argument"};
    Tensor* t = as_tensor(h);
    check_mode_rank(*t, mode, rank);
    *n = selector_candidates(*t, mode, rank, out);
    return SF_OK;
  });
}

sf_status sf_set_selector_model(const int32_t* feature, const double* threshold, const int32_t* left,
                                const int32_t* right, const int32_t* value, int n_nodes, int n_features) {
  return guard([&]() -> sf_status {
    if (n_nodes < 0 || (n_nodes > 0 && (!feature || !threshold || !left || !right || !value)))
      throw StatusError{SF_ERR_INVALID_ARG, "bad model arrays"};
    for (int i = 0; i < n_nodes; ++i)
      if (left[i] >= n_nodes || right[i] >= n_nodes) throw StatusError{SF_ERR_INVALID_ARG, "bad child index"};
    set_selector_model(feature, threshold, left, right, value, n_nodes, n_features);
    return SF_OK;
  });
}

const char* sf_status_string(sf_status s) {
  switch (s) {
    case SF_OK: return "SF_OK";
    case SF_ERR_INVALID_ARG: return "SF_ERR_INVALID_ARG";
    case SF_ERR_INDEX_OUT_OF_RANGE: return "SF_ERR_INDEX_OUT_OF_RANGE";
    case SF_ERR_OUT_OF_MEMORY: return "SF_ERR_OUT_OF_MEMORY";
    case SF_ERR_NOT_PLANNED: return "SF_ERR_NOT_PLANNED";
    case SF_ERR_UNSUPPORTED: return "SF_ERR_UNSUPPORTED";
    case SF_ERR_CUDA: return "SF_ERR_CUDA";
    case SF_ERR_NCCL: return "SF_ERR_NCCL";
    default: return "SF_ERR_UNKNOWN";
  }
}

const char* sf_last_error(void) { return g_err.c_str(); }

uint64_t sf_kernel_launches(void) { return g_launches.load(); }

sf_status sf_device_bytes(uint64_t* in_use, uint64_t* peak, int reset_peak) {
  if (in_use) *in_use = g_in_use.load();
  if (peak) *peak = g_peak.load();
  if (reset_peak) g_peak.store(g_in_use.load());
  return SF_OK;
}

const char* sf_version(void) { return "scalfrag-b200 0.1 (sm_100a)"; }

}  // extern "C"
