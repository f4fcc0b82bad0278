// sf_internal.h - internal types of libscalfrag (not part of the ABI).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <map>
#include <memory>
#include <string>
#include <utility>
#include <vector>

#include "../../include/scalfrag.h"

namespace sf {

// The library's only environment input (debug / A-B aid, include/scalfrag.h "SF_DEBUG"):
// SF_DEBUG is a comma-separated list of key or key=value; debug_opt returns the value of
// `key` ("" for a bare key) or nullptr when absent.  Read at every call (in-process A/B).
const char* debug_opt(const char* key);
// SF_DEBUG=trace: host wall-clock phase marks of sf_plan on stderr (profiling aid).
void trace_mark(const char* phase);

// Thread-local error detail + status plumbing.
void set_error(const std::string& msg);
extern std::atomic<uint64_t> g_launches;
inline void count_launch(uint64_t n = 1) { g_launches.fetch_add(n, std::memory_order_relaxed); }

struct CudaError {
  cudaError_t err;
  const char* what;
};

#define SF_CUDA(call)                                                      \
  do {                                                                     \
    cudaError_t _e = (call);                                               \
    if (_e != cudaSuccess) throw ::sf::CudaError{_e, #call};               \
  } while (0)

struct StatusError {
  sf_status st;
  std::string msg;
};

// RAII device buffer.
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  DevBuf() = default;
  explicit DevBuf(size_t b) { alloc(b); }
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  DevBuf(DevBuf&& o) noexcept : p(o.p), bytes(o.bytes) { o.p = nullptr; o.bytes = 0; }
  DevBuf& operator=(DevBuf&& o) noexcept {
    if (this != &o) { release(); p = o.p; bytes = o.bytes; o.p = nullptr; o.bytes = 0; }
    return *this;
  }
  ~DevBuf() { release(); }
  void alloc(size_t b);
  void release();
  template <class T> T* as() const { return static_cast<T*>(p); }
};

// Padding (bytes) added to every streamed array so 16-byte-aligned bulk copies of
// an aligned superset of a chunk never read past the allocation.
constexpr size_t kPadBytes = 64;

struct Plan {
  int mode = -1, rank = 0;
  sf_launch_t launch{};
  sf_features_t feat{};
  uint64_t nnz_local = 0;
  uint64_t num_tiles = 0, num_chunks = 0;
  uint64_t row_begin = 0, row_end = 0;
  double plan_ms = 0;
  // kernel-order arrays (SoA): sorted indices of every mode + values + input position
  DevBuf ind[SF_MAX_MODES];
  DevBuf val;
  DevBuf rec;           // frag3 plans: kernel-order records in slot order (rec_words each)
  int rec_words = 0;    // 0: SoA arrays (ind/val) instead of records
  DevBuf perm;          // uint32 input position per sorted slot
  DevBuf chunk_begin;   // uint32[num_chunks + 1]
  DevBuf chunk_tile;    // uint64[num_chunks]
  DevBuf tile_chunk;    // uint32[num_tiles + 1]: first chunk of every tile, then num_chunks
  mutable DevBuf cta_chunk;  // uint32[grid + 1]: first chunk of every CTA of the last launch grid
  mutable int cta_grid = 0;
  mutable int occ = 0, occ_threads = 0;  // cached CTAs/SM of the kernel for (threads, smem)
  mutable size_t occ_smem = 0;
  mutable DevBuf carry; // A7 deterministic option: per-group carry slots (rows + partials)
  bool rec_packed = false;               // frag3 PK records (N >= 4, indices bit-packed)
  // Hot-row cache (launch.hot_kb > 0): per gathered slot q with hot rows, the original row of
  // every hot slot (hot_rows[q], hot_count[q] entries), the record flag bit (hot_bit[q]) and the
  // slot's first row in the dense per-call copy `hot_cache` (hot_off[q]).
  uint32_t hot_bit[SF_MAX_MODES] = {};
  uint64_t hot_count[SF_MAX_MODES] = {};
  uint64_t hot_off[SF_MAX_MODES] = {};
  DevBuf hot_rows[SF_MAX_MODES];
  mutable DevBuf hot_cache;
  uint64_t hot_total = 0;                // rows in hot_cache
  uint32_t rec_boff[SF_MAX_MODES] = {};  // PK: bit offset of field f (slot order)
  uint32_t rec_bmask[SF_MAX_MODES] = {}; // PK: width mask of field f
  // Multi-GPU exchange map (sf_comm.cu), built at the first exchange of this plan from every
  // rank's touched row range: ranges[2k], ranges[2k+1] = rows [begin, end) of rank k.
  std::vector<uint64_t> ranges;
  bool send_first = false;    // this rank's first row is owned by a lower rank
  std::vector<int> add_srcs;  // ranks whose first row is this rank's last row (ascending)
  mutable DevBuf xbuf;        // exchange buffers: send (R floats) + recv (nranks * R floats)
  // The caller's `out` block: rows [out_row0, out_row0 + out_rows) of Y (the whole Y at
  // nranks == 1, the touched row range [row_begin, row_end) of a shard otherwise).
  uint64_t out_row0 = 0, out_rows = 0;
  size_t device_bytes() const;
};

// Collective transport of a sharded handle (sf_comm.cu): NCCL (sf_comm_attach) or a caller
// callback (sf_comm_attach_transport).  allgatherv: rank k contributes bytes[k] bytes from
// `send`; every rank receives them at recv + displs[k] (device memory, stream-ordered).
struct NcclHandle;  // a shared NCCL communicator (sf_comm.cu; one per (unique id, rank, device))
struct Comm {
  int nranks = 1, rank = 0;
  void* nccl = nullptr;  // ncclComm_t (owned by `shared`)
  std::shared_ptr<NcclHandle> shared;
  sf_allgatherv_fn fn = nullptr;
  void* ctx = nullptr;
  void allgatherv(const void* send, void* recv, const uint64_t* bytes, const uint64_t* displs, cudaStream_t s);
  void alltoallv(const void* send, const uint64_t* sbytes, const uint64_t* sdispl, void* recv, const uint64_t* rbytes,
                 const uint64_t* rdispl, cudaStream_t s);
  ~Comm();
};

struct Tensor {
  int device = 0;
  int nmodes = 0;
  uint64_t dims[SF_MAX_MODES] = {};
  uint64_t nnz = 0;
  int nranks = 1, rank = 0;
  int num_sms = 148;
  size_t smem_optin = 227 * 1024;
  DevBuf ind[SF_MAX_MODES];  // raw COO (input order)
  DevBuf val;
  DevBuf aos;                // raw COO as AoS records (aos_words per nonzero), built on first plan
  int aos_words = 0;
  bool have_features[SF_MAX_MODES] = {};
  sf_features_t features[SF_MAX_MODES] = {};
  std::map<std::pair<int, int>, Plan*> plans;  // (mode, rank) -> plan
  // A8 upload || presort (sf_plan.cu presort_*): for each mode, the matricized key of every
  // uploaded segment composed with its input position, (key << pre_pb) | pos, sorted on the
  // segment's upload stream while later segments are still in flight; the first sf_plan of
  // the mode merges the sorted runs instead of sorting all nonzeros.
  DevBuf pre[SF_MAX_MODES];
  bool have_pre[SF_MAX_MODES] = {};
  // the last matricized sort of mode m carried the other mode's (i_o >> 17) above bit
  // carry_kb[m] of its keys (0 = plain keys; sf_plan.cu key_matricized_kernel)
  int carry_kb[SF_MAX_MODES] = {};
  DevBuf pre_alt;              // composed keys of a segment before its sort (upload only)
  DevBuf hot_cnt[SF_MAX_MODES];  // hot-row cache: nonzeros per row of mode m (whole handle), lazily
  double hot_cover[SF_MAX_MODES] = {-1, -1, -1, -1, -1, -1, -1, -1};  // share of nonzeros in the
                                 // hottest 2^18 rows of mode m (hot_coverage), -1 = not measured
  uint64_t pre_seg_len = 0;
  int pre_pb = 0;              // position bits
  cudaStream_t stream = nullptr;               // internal stream for planning
  Comm* comm = nullptr;                        // sharded handles: collective transport
  // Distributed ingest (sf_tensor_create_dist): this handle holds only input
  // positions [pos_begin, pos_begin + nnz) of an nnz_total-nonzero tensor; per mode, the
  // nonzeros of this rank's shard of the matricized order are fetched from every rank
  // (histogram allgather + all-to-all) into sub[mode], whose plan the handle uses.
  bool dist = false;
  uint64_t pos_begin = 0, nnz_total = 0;
  Tensor* sub[SF_MAX_MODES] = {};
  DevBuf sub_gpos[SF_MAX_MODES];               // global input position of every sub[mode] nonzero
  ~Tensor();
};

// Packed 16-byte records for N >= 4 (frag3 PK): all N indices fit 96 bits.
inline int index_bits(uint64_t dim) {  // bits to hold 0 .. dim-1 (>= 1)
  int b = 0;
  for (uint64_t x = dim > 0 ? dim - 1 : 0; x; x >>= 1) ++b;
  return b > 0 ? b : 1;
}
inline bool rec_packable(const Tensor& t) {
  if (t.nmodes < 4) return false;
  int b = 0;
  for (int m = 0; m < t.nmodes; ++m) b += index_bits(t.dims[m]);
  return b <= 96;
}
// Words per frag3 record for this tensor: 4 (N <= 3, or N >= 4 packed), else 8.
inline int tensor_rec_words(const Tensor& t) {
  return (t.nmodes + 1 <= 4 || rec_packable(t)) ? 4 : 8;
}

// Secondary sort key of mode n (reading R10): the gathered mode with the
// smallest dimension (ties: the higher mode index) -- the (i_n, i_s) fibers with the most
// reuse of A_s rows.
inline int secondary_mode(const Tensor& t, int mode) {
  int s = -1;
  for (int m = 0; m < t.nmodes; ++m) {
    if (m == mode) continue;
    if (s < 0 || t.dims[m] <= t.dims[s]) s = m;
  }
  return s;
}

// ---- frag3 layout helpers (shared by the planner, the selector and the kernel) ----
template <int N>
struct RecWords {
  static constexpr int W = (N + 1 <= 4) ? 4 : 8;
};

__host__ __device__ inline int rec_words_for(int N) { return (N + 1 <= 4) ? 4 : 8; }


// Region stride (words) of one group's K records: W*K + pad with stride/4 odd, so the
// GPW groups' record k (read in lockstep) fall into distinct 16-byte bank quads.
__host__ __device__ __forceinline__ uint32_t frag3_region_words(uint32_t K, uint32_t W) {
  const uint32_t base = K * W;
  return ((base / 4u) % 2u == 0u) ? base + 4u : base + 8u;
}

// Records per group per stage for a launch's chunk_nnz (nonzeros per warp per stage).
__host__ __device__ __forceinline__ uint32_t frag3_K(uint32_t chunk_nnz, uint32_t GPW) {
  uint32_t K = chunk_nnz / GPW;
  return K < 4u ? 4u : K;
}

// Lane groups per warp of the fragment kernels for rank R (LaneMap<R> in sf_frag.cuh).
inline int frag_groups_per_warp(int R) {
  const int lpn = R >= 32 ? R / 8 : R / 4;
  return lpn >= 1 && lpn <= 32 ? 32 / lpn : 1;
}

// Small host<->device transfers that must not queue behind bulk copies on the copy engines
// (a plan's scalar reads would otherwise wait for a caller's multi-GB D2H on another stream):
// a kernel moves the bytes through mapped pinned host memory, then the stream is synchronized.
// Each call synchronizes `s`.  `n` pairs of (host dst, device src, bytes) for the reads.
void d2h_small(cudaStream_t s, int n, void* const* dst, const void* const* src, const size_t* bytes);
inline void d2h_small(cudaStream_t s, void* dst, const void* src, size_t bytes) {
  d2h_small(s, 1, &dst, &src, &bytes);
}
void h2d_small(cudaStream_t s, void* dst, const void* src, size_t bytes);
// Device-to-device copy by a kernel (any alignment; 16-byte vectors when both pointers allow):
// keeps bulk plan copies off the copy engines a caller's H2D/D2H may be occupying.
void d2d_copy(void* dst, const void* src, size_t bytes, cudaStream_t s);

// ---- planning (sf_plan.cu) ----
// upload || presort: decide and allocate (returns false: no mode qualifies / disabled by
// SF_PRESORT=0 / not enough memory), per-segment work on the upload stream, CUB temp bytes
// one segment's sort needs.
// Free device memory of the current device: the driver's plus the library's cached blocks.
size_t device_free_bytes();
bool presort_begin(Tensor& t, uint64_t seg_len);
void presort_segment(Tensor& t, uint64_t a, uint64_t len, cudaStream_t s, void* temp, size_t temp_bytes);
size_t presort_temp_bytes(const Tensor& t, uint64_t seg_len);
// Raw-COO work every plan needs, done per segment behind its upload (A8): the AoS record copy
// (unless the presort builds it) and the whole-handle row counts of modes with >= 2^18 rows
// (the hot-row cache's input).  Skipped when device memory is short (then built at plan time).
struct Ingest {
  bool aos = false;
  uint32_t cnt_mask = 0;
};
Ingest ingest_begin(Tensor& t);
void ingest_segment(Tensor& t, const Ingest& g, uint64_t a, uint64_t len, cudaStream_t s);
// keys/pos (optional): receive the matricized order (sorted keys, input positions) when
// this call had to sort, so build_plan can reuse it instead of sorting again.
void compute_features(Tensor& t, int mode, sf_features_t* out, DevBuf* keys, DevBuf* pos);
void build_plan(Tensor& t, Plan& p, int mode, int rank, const sf_launch_t& launch, DevBuf* keys, DevBuf* pos);
// ---- selection (sf_select.cpp) ----
sf_launch_t select_launch(const Tensor& t, const sf_features_t& f, int mode, int rank,
                          uint64_t nnz_local);
void normalize_launch(const Tensor& t, int mode, int rank, sf_launch_t& l);
int selector_features(const Tensor& t, const sf_features_t& f, int mode, int rank, uint64_t nnz_local,
                      double* x);
int selector_candidates(const Tensor& t, int mode, int rank, sf_launch_t* out);
void set_selector_model(const int32_t* feature, const double* threshold, const int32_t* left,
                        const int32_t* right, const int32_t* value, int n_nodes, int n_features);
size_t frag_smem_bytes(const Tensor& t, int mode, int rank, const sf_launch_t& l);
bool hot_tile_candidate(const Tensor& t, int mode, int rank, int m);
// share of the handle's nonzeros whose mode-m index is among the hottest `rows` rows (cached in
// t.hot_cover[m]; counts in t.hot_cnt[m]) -- how well a hot-row cache would serve mode m
void hot_coverage(Tensor& t, int m, uint64_t rows);
// ---- CP-ALS (sf_cpals.cu) ----
void cpals(Tensor& t, int R, float* const* factors, int iters, double tol, double* fits, int* done,
           cudaStream_t s, Plan* const* plans);
// ---- kernels (sf_mttkrp.cu) ----
void launch_mttkrp(const Tensor& t, const Plan& p, const float* const* factors, float* out,
                   cudaStream_t s);
void launch_coo(int nmodes, const uint64_t* dims, uint64_t nnz, const uint32_t* const* inds,
                const float* vals, const float* const* factors, int rank, int mode, float* out,
                cudaStream_t s);
bool frag_supported(int nmodes, int rank);
bool seg_sorted_supported(int rank);
int seg_aos_words(int nmodes);
void launch_seg_aos(int nmodes, uint64_t len, const uint32_t* const* inds, const float* vals, uint32_t* aos,
                    cudaStream_t s);
void launch_seg_sorted(int nmodes, const uint64_t* dims, uint64_t len, const uint32_t* aos, const uint32_t* skey,
                       const uint32_t* spos, const float* const* factors, int rank, int mode, float* out,
                       cudaStream_t s);
void launch_iota(uint32_t* x, uint64_t n, cudaStream_t s);
size_t seg_sort_temp_bytes(uint64_t len, int bits);
void seg_sort(const uint32_t* keys_in, uint32_t* keys_out, const uint32_t* vals_in, uint32_t* vals_out, uint64_t len,
              int bits, void* temp, size_t temp_bytes, cudaStream_t s);
// gathered slot order of a plan: staged modes ascending, then the other gathered modes
int frag_slot_order(int nmodes, int mode, uint32_t staged_mask, int* slot_mode);
// modes whose factor blocks are copied into shared memory (L2-tiled plans stage none)
inline uint32_t smem_staged_mask(const sf_launch_t& l) {
  return (l.flags & SF_LAUNCH_L2_TILES) ? 0u : l.staged_mask;
}
void launch_rows_op(float* Y, int R, const int64_t* rows, float* buf, int count, int op, cudaStream_t s);
// ---- multi-GPU (sf_comm.cu) ----
// Boundary-row exchange of a sharded plan's local block `out` (rows [row_begin, row_end)):
// the first row goes to its owner (the lowest rank touching it) and is zeroed here; the
// owner adds the partials in rank order.  No-op without a comm or at nranks == 1.
void exchange_rows(Tensor& t, Plan& p, float* out, cudaStream_t s);
// Every rank contributes rows [blk[2k], blk[2k+1]) of an I x R matrix from `local`
// (this rank's rows starting at blk[2*rank]); full (I x R, every rank) receives them all.
void allgather_blocks(Tensor& t, const std::vector<uint64_t>& blk, const float* local, float* full, int R,
                      cudaStream_t s);
void ensure_ranges(Tensor& t, Plan& p, cudaStream_t s);
// sf_tensor_create_dist handles: build sub[mode] (this rank's shard of mode `mode`, gathered
// from every rank; sf_dist.cu).
void dist_build_sub(Tensor& t, int mode);
void validate_indices(int nmodes, const uint64_t* dims, uint64_t nnz,
                      uint32_t* const* inds, int* d_flag, cudaStream_t s);

}  // namespace sf
