/*
 * scalfrag.h - C ABI of the B200-native ScalFrag hot path: mode-n sparse MTTKRP.
 *
 * What is computed (§II-C, Eq. (4)):
 *     M = X_(n) (A^(N) ⊙ ... ⊙ A^(n+1) ⊙ A^(n-1) ⊙ ... ⊙ A^(1))
 * for an N-way COO tensor X (§II-D: entries M(i,j,k,val)),
 * i.e. elementwise  Y(i,:) = sum_{e: i_n(e)=i} v_e * ⊙_{m≠n} A_m(i_m(e),:)
 * (reading R1).  Y is OVERWRITTEN (Alg. 1 line 4, PAPER.md L111
 * "M <- ..."), rows without nonzeros are 0, duplicate coordinates are summed.
 *
 * The calls follow the north star: sf_tensor_create (ingest, §8(a) A1; the
 * paper's "pipelined to the device side"), sf_plan
 * (matricize + chunk + features + launch selection, PAPER.md L189-199;
 * §8(a) A2-A4) and sf_mttkrp (the kernel, §8(a) A5-A7).
 *
 * Conventions
 *   - All functions are extern "C", take plain pointers and sizes, never throw,
 *     and return an sf_status.  On failure no state changes; sf_last_error()
 *     returns a thread-local detail string.
 *   - 2 <= nmodes <= SF_MAX_MODES; 1 <= dims[m] <= 2^32-1; indices are 0-based
 *     uint32; values fp32; factors fp32 row-major I_m x rank (ld = rank).
 *   - nnz must be < 2^32 (plans store input positions as uint32; SF_ERR_UNSUPPORTED
 *     otherwise).  nnz = 0 is valid (Y = 0).
 *   - A handle is bound to the CUDA device current at create time; it owns all
 *     device arrays, plans and scratch.  Handles are not thread-safe; calls on
 *     different handles are independent.
 *   - Device pointers are CUDA device pointers (e.g. torch tensor .data_ptr()).
 *     `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *   - Asynchronous kernel faults surface at the caller's next synchronization
 *     (as in cuBLAS); the library itself synchronizes only where stated.
 *   - Arithmetic: fp32 products and sums; the vector reductions at run boundaries
 *     (red.global.add.v4.f32) flush subnormal results to zero, so a row whose |.|-scale
 *     S = sum |v * prod A| is itself subnormal (< 1.2e-38) may come back as 0 -- such
 *     inputs are outside the 1e-4 relative contract (reading R8).
 *   - Environment: the library reads nothing but SF_DEBUG, a debug / A-B aid that is never
 *     needed in production: a comma-separated list of trace (sf_plan phase marks on
 *     stderr), no_presort, no_l2tiles, no_hot, no_cpals_fused (disable one optimisation)
 *     and l2_revisit=<x> (calibration of the L2-tile rule).
 */
#ifndef SCALFRAG_H
#define SCALFRAG_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SF_MAX_MODES 8
#define SF_HIST_BINS 40

typedef struct sf_tensor_s* sf_tensor_t;

typedef enum {
  SF_OK = 0,
  SF_ERR_INVALID_ARG = 1,        /* bad pointer / size / mode / rank */
  SF_ERR_INDEX_OUT_OF_RANGE = 2, /* some inds[m][e] >= dims[m] */
  SF_ERR_OUT_OF_MEMORY = 3,      /* cudaMalloc / pinned allocation failed */
  SF_ERR_NOT_PLANNED = 4,        /* sf_mttkrp before sf_plan(mode, rank) */
  SF_ERR_UNSUPPORTED = 5,        /* e.g. nnz >= 2^32, rank/nmodes without a kernel */
  SF_ERR_CUDA = 6,               /* a CUDA runtime call failed (detail in sf_last_error) */
  SF_ERR_NCCL = 7                /* a collective failed (NCCL, or the caller's transport returned != 0) */
} sf_status;

/* Kernel families. */
typedef enum {
  SF_KERNEL_AUTO = 0, /* let the selector choose (sf_set_launch only) */
  SF_KERNEL_COO = 1,  /* nnz-parallel over the raw COO, one vector atomic per nonzero */
  SF_KERNEL_FRAG = 2  /* sorted fragments: register segmented reduction, factor blocks
                         staged in shared memory, atomics only at run/fragment edges */
} sf_kernel_kind;

/* Launch configuration ("combination of launch parameters"),
 * extended for the fragment kernel. */
typedef struct {
  int32_t kernel;        /* sf_kernel_kind */
  int32_t block_threads; /* threads per CTA, multiple of 32 in [64, 1024] */
  int32_t ctas_per_sm;   /* FRAG: persistent grid = ctas_per_sm * #SMs (0 = max resident) */
  int32_t chunk_nnz;     /* FRAG: C, nonzeros per chunk ("segment") */
  uint32_t staged_mask;  /* FRAG: bit m set => factor m is staged in shared memory by
                            blocks of block_rows[m] rows (a "tensor block") */
  uint32_t block_rows[SF_MAX_MODES];
  uint32_t flags;        /* FRAG: SF_LAUNCH_* bits below */
  uint32_t hot_kb;       /* FRAG: hot-row cache budget in KiB (0 = off).  The most frequent rows
                            of the gathered factors that are neither staged nor L2-tiled (by
                            nonzero count in this plan, one global threshold) are copied per
                            call into one dense block and gathered from there (DESIGN.md §5
                            "hot-row cache"); plain records need I_m < 2^31, packed records one
                            spare bit per such field (else the slot is skipped). */
} sf_launch_t;
#define SF_LAUNCH_NO_OWNER_STORES 4u /* FRAG, unstaged: memset Y + atomics only (disable A5) */
#define SF_LAUNCH_DETERMINISTIC 32u /* FRAG: A7 two-pass carry combine instead of atomics; forces an
                                       unstaged owner-store plan; Y is bitwise reproducible run to run */
#define SF_LAUNCH_L2_TILES 64u /* FRAG: the staged_mask modes are NOT copied into shared memory; they
                                 only tile the order (tile = block of block_rows[m] rows, PAPER.md L34
                                 "tensor blocks") and every CTA sweeps the tiles in the same order,
                                 taking 1/grid of each, so the factor rows gathered at any moment
                                 are one block that stays L2-resident (for factors >> L2).  Forces
                                 memset + atomics (no owner stores); ignored with DETERMINISTIC. */

/* Tensor feature vector (reading R4). Integers are exact. */
typedef struct {
  uint64_t nnz;
  uint64_t dim;               /* I_n */
  uint64_t num_slices;        /* non-empty rows of mode n */
  uint64_t num_fibers;        /* distinct (i_n, i_s) pairs, s = secondary (smallest gathered) mode */
  uint64_t max_nnz_per_slice;
  uint64_t max_nnz_per_fiber;
  uint64_t sum_sq_nnz_per_slice;
  uint64_t slice_hist[SF_HIST_BINS]; /* slices with nnz in [2^b, 2^(b+1)) */
  int32_t nmodes, mode, secondary, reserved;
  double slice_ratio;         /* num_slices / I_n */
  double fiber_ratio;         /* num_fibers / num_slices */
  double avg_nnz_per_slice, avg_nnz_per_fiber, std_nnz_per_slice;
} sf_features_t;

typedef struct {
  sf_features_t feat;   /* features of the whole tensor for this mode */
  sf_launch_t launch;   /* the launch the plan uses */
  uint64_t nnz_local;   /* nonzeros of this shard */
  uint64_t num_tiles;   /* distinct tiles present */
  uint64_t num_chunks;
  uint64_t row_begin;   /* this shard touches rows [row_begin, row_end) of Y */
  uint64_t row_end;
  uint64_t out_row0;    /* sf_mttkrp's `out` holds rows [out_row0, out_row0 + out_rows) of Y: */
  uint64_t out_rows;    /*   all of Y at nranks == 1, the local block [row_begin, row_end) else */
  uint64_t device_bytes;
  double plan_ms;       /* device time of the last sf_plan for this (mode, rank) */
} sf_plan_info_t;

/* ---- lifetime ---------------------------------------------------------- */

/* Ingest (§8(a) A1).  Copies the COO tensor to the device and validates every
 * index on the device (one synchronization).  inds: nmodes pointers, each to nnz
 * uint32; vals: nnz floats.  Pointers may be host (pageable or pinned) or device;
 * host data is uploaded in `segments` chunks through pinned staging buffers over
 * `streams` CUDA streams, overlapping copies with the device-side range check
 * (§IV-C; segments/streams <= 0 pick defaults 8/4).
 * The caller keeps ownership of its buffers (deep copy). */
sf_status sf_tensor_create(int nmodes, const uint64_t* dims, uint64_t nnz,
                           const uint32_t* const* inds, const float* vals, sf_tensor_t* out);
sf_status sf_tensor_create_ex(int nmodes, const uint64_t* dims, uint64_t nnz,
                              const uint32_t* const* inds, const float* vals, int segments,
                              int streams, sf_tensor_t* out);
sf_status sf_tensor_destroy(sf_tensor_t t);
/* Distributed ingest (SURVEY §8(e) "v2", row F4): this rank passes only input positions
 * [pos_begin, pos_begin + nnz_local) of an nnz_total-nonzero tensor (the ranks' slices must
 * tile [0, nnz_total) in rank order; nnz_total < 2^32).  After sf_comm_attach*, the first
 * sf_plan of a mode assembles this rank's shard of the matricized order -- the same nonzeros
 * as sf_set_shard on the whole tensor -- by a global i_n histogram (allgather + rank-order
 * sum) and one all-to-all, then sorts only the shard.  sf_plan_export reports global input
 * positions.  Everything else behaves as a sharded handle. */
sf_status sf_tensor_create_dist(int nmodes, const uint64_t* dims, uint64_t nnz_total, uint64_t pos_begin,
                                uint64_t nnz_local, const uint32_t* const* inds, const float* vals,
                                sf_tensor_t* out);

/* Multi-GPU (§8(e)): restrict this handle to shard `rank` of `nranks`: for every mode
 * it owns matricized positions [floor(rank*nnz/nranks), floor((rank+1)*nnz/nranks)).
 * With nranks > 1, sf_mttkrp writes only this shard's LOCAL ROW BLOCK (sf_shard_rows).
 * Drops existing plans (synchronizes the device first).  Default 1/0. */
sf_status sf_set_shard(sf_tensor_t t, int nranks, int rank);

/* Rows [*row_begin, *row_end) of Y that sf_mttkrp(mode, rank) writes into `out` (out row 0 =
 * Y row *row_begin): all of Y for an unsharded handle, this shard's local row block else
 * (the rows its nonzeros touch; adjacent shards share at most one boundary row, which the
 * exchange below assigns to the lowest rank touching it).  Needs sf_plan(mode, rank). */
sf_status sf_shard_rows(sf_tensor_t t, int mode, int rank, uint64_t* row_begin, uint64_t* row_end);

/* Collective transport for sharded handles.  With a comm attached,
 * sf_mttkrp ends with the boundary-row exchange on its stream: the partial of a shard's
 * first row, if a lower rank also touches it, is sent to that owner (and zeroed locally);
 * the owner adds the partials in rank order.  Afterwards the local blocks hold a
 * ROW-SHARDED Y: each row's value lives on its owner, the other copies are 0, rows no
 * shard touches are 0 everywhere.  One allgather of rank*4 bytes per rank per call.
 *   sf_comm_unique_id: rank 0 creates a 128-byte NCCL id (broadcast it, e.g. by torch).
 *   sf_comm_attach:    ncclCommInitRank on this handle's device + sf_set_shard(nranks, rank);
 *                      handles attached with the same (id, nranks, rank, device) share one
 *                      communicator, created once and kept until the process exits (a
 *                      unique id can initialise only one communicator).
 *   sf_comm_attach_transport: the same exchange over the caller's allgatherv (tests, or a
 *                      non-NCCL fabric); fn returns 0 on success.
 * NCCL is loaded at run time (dlopen libnccl.so.2); SF_ERR_NCCL on any collective error. */
typedef int (*sf_allgatherv_fn)(void* ctx, const void* send, void* recv, const uint64_t* bytes,
                                const uint64_t* displs, int nranks, void* stream);
sf_status sf_comm_unique_id(void* id128);
sf_status sf_comm_attach(sf_tensor_t t, int nranks, int rank, const void* id128);
sf_status sf_comm_attach_transport(sf_tensor_t t, int nranks, int rank, sf_allgatherv_fn fn, void* ctx);
sf_status sf_comm_detach(sf_tensor_t t);
/* Diagnostic (collective: every rank of the attached comm calls it): a rank-stamped
 * allgatherv (rank k sends k + 1 words) and alltoallv (rank r sends (r + q) % 3 + 1 words to
 * rank q) of device buffers through the attached transport on `stream`, checked word by word
 * on the host.  SF_OK, SF_ERR_NCCL on a wrong word or a failed collective, SF_ERR_INVALID_ARG
 * without a comm.  Synchronizes. */
sf_status sf_comm_check(sf_tensor_t t, void* stream);
/* Replicated Y from the row-sharded local blocks after sf_mttkrp (optional):
 * full (device, I_mode x rank) receives every rank's owned rows, zeros elsewhere. */
sf_status sf_allgather_rows(sf_tensor_t t, int mode, int rank, const float* local, float* full, void* stream);
/* Host-only (no GPU needed): the exchange rule for given touched row ranges
 * (ranges[2k], ranges[2k+1] = [begin, end) of rank k; begin == end: empty shard).
 * send_first[k] = 1 iff rank k's first row is owned by a lower rank; owner[k] = the owner
 * of rank k's first row (the lowest rank touching it; k itself if it owns it; -1 if empty). */
sf_status sf_exchange_map(int nranks, const uint64_t* ranges, int32_t* send_first, int32_t* owner);

/* ---- planning (§8(a) A2-A4) -------------------------------------------- */

/* Sort (matricized order, then tiles), build fragments/chunks, compute features and
 * select the launch for (mode, rank).  Idempotent; synchronizes the device. */
sf_status sf_plan(sf_tensor_t t, int mode, int rank);
/* Free the plan of (mode, rank) (device memory returns to the library's block cache);
 * a later sf_mttkrp needs sf_plan again.  Synchronizes the device. */
sf_status sf_plan_release(sf_tensor_t t, int mode, int rank);
/* Return every cached device block to the driver (cudaFree).  Synchronizes the device. */
sf_status sf_trim_cache(void);
/* Override the selector (sweeps, Fig. 4) and re-plan. */
sf_status sf_set_launch(sf_tensor_t t, int mode, int rank, const sf_launch_t* launch);
/* Features only (no plan needed). Synchronizes. */
sf_status sf_features(sf_tensor_t t, int mode, sf_features_t* out);
sf_status sf_plan_info(sf_tensor_t t, int mode, int rank, sf_plan_info_t* out);
/* Bit-exact export for tests: perm_host[k] = input position of the k-th nonzero in
 * kernel order (nnz_local entries); chunks_host: 3*num_chunks uint64 (begin, end, tile).
 * Either pointer may be NULL. Synchronizes. */
sf_status sf_plan_export(sf_tensor_t t, int mode, int rank, uint64_t* perm_host,
                         uint64_t* chunks_host);

/* ---- learned launch selector (§IV-B) ---- */

#define SF_SELECTOR_MAX_FEATURES 32
#define SF_SELECTOR_MAX_CANDIDATES 16
/* The selector's feature vector for (mode, rank) of this handle/shard (log2-scaled sizes,
 * PAPER.md L195 features); returns the count in *n (<= SF_SELECTOR_MAX_FEATURES). */
sf_status sf_selector_features(sf_tensor_t t, int mode, int rank, double* x, int* n);
/* The discrete launch classes the learned model chooses among (class id = index). */
sf_status sf_selector_candidates(sf_tensor_t t, int mode, int rank, sf_launch_t* out, int* n);
/* Install a decision tree (sklearn tree_ layout: node arrays; leaf iff left < 0; value =
 * class id).  n_nodes = 0 removes it (rule-based selection).  Process-global; later
 * sf_plan calls use it.  Copies the arrays. */
sf_status sf_set_selector_model(const int32_t* feature, const double* threshold, const int32_t* left,
                                const int32_t* right, const int32_t* value, int n_nodes, int n_features);

/* ---- the hot path (§8(a) A5-A7) ---------------------------------------- */

/* Y = mode-`mode` MTTKRP.  factors: host array of nmodes DEVICE pointers (factors[mode]
 * is ignored and may be NULL); out: device fp32, out_rows x rank (sf_shard_rows /
 * sf_plan_info: I_mode x rank unsharded, the local row block of a shard), overwritten.
 * With a comm attached the boundary-row exchange follows on the same stream.
 * Stream-ordered, returns after enqueue.  out must not alias a factor. */
sf_status sf_mttkrp(sf_tensor_t t, int mode, const float* const* factors, int rank, float* out,
                    void* stream);

/* One-shot streamed path (the paper's pipeline; §8(a) A8 (ii)):
 * host COO is uploaded in `segments` pieces over `streams` streams while finished
 * segments are computed; Y (device, I_mode x rank) is overwritten.  No handle.  For rank
 * 16/32/64 each segment is sorted by i_n on the device and reduced in registers along its
 * runs (one atomic per run piece: heavy rows keep short fp32 chains); other ranks use one
 * atomic per nonzero.  Synchronizes before returning.  On SF_ERR_INDEX_OUT_OF_RANGE the
 * offending nonzeros were skipped and Y holds the sum of the others. */
sf_status sf_mttkrp_streamed(int nmodes, const uint64_t* dims, uint64_t nnz,
                             const uint32_t* const* inds_host, const float* vals_host,
                             const float* const* factors, int rank, int mode, float* out,
                             int segments, int streams);

/* The same one-shot pipeline for several modes at once (one MTTKRP per mode n with
 * outs[n] != NULL, all with the same factors: the N MTTKRPs of a step): every segment is
 * uploaded ONCE and, behind its H2D, range-checked, copied into 16/32-byte AoS records
 * (shared by the modes) and, per requested mode, sorted by i_n and reduced along its runs
 * (compute overlaps the H2D of later segments).  outs: nmodes DEVICE
 * pointers (NULL = mode not computed), Y_n is I_n x rank row-major, overwritten.  factors:
 * nmodes device pointers; A_m may be NULL only if m is the one mode computed.  stream: the
 * work is ordered after what the caller queued on it before the call (e.g. the factor
 * uploads; NULL = no ordering).  Device footprint: O(streams x segment) + the caller's
 * arrays.  segments / streams <= 0: chosen by the library (about 5 M nonzeros per segment,
 * 2..32; 4 streams, 2 for <= 2 segments).  Synchronizes before returning; errors as
 * sf_mttkrp_streamed. */
sf_status sf_mttkrp_streamed_modes(int nmodes, const uint64_t* dims, uint64_t nnz,
                                   const uint32_t* const* inds_host, const float* vals_host,
                                   const float* const* factors, int rank, float* const* outs,
                                   int segments, int streams, void* stream);

/* Boundary-row exchange helper for multi-GPU row shards (§8(e)): for k < count with
 * rows[k] >= 0 (device int64 array):
 *   op 0 (PACK): buf[k, :] = Y[rows[k], :]      op 1 (ADD): Y[rows[k], :] += buf[k, :]
 *   op 2 (ZERO): Y[rows[k], :] = 0
 * Y, rows, buf are device pointers; Y is I x rank row-major.  Stream-ordered. */
typedef enum { SF_ROWS_PACK = 0, SF_ROWS_ADD = 1, SF_ROWS_ZERO = 2 } sf_rows_op_t;
sf_status sf_rows_op(float* Y, int rank, const int64_t* rows, float* buf, int count, int op,
                     void* stream);

/* ---- CP-ALS (Algorithm 1) ------------- */

/* Runs up to `iters` ALS sweeps over all modes on this tensor, calling the MTTKRP of the
 * hot path for line 4 of Alg. 1 (plans are built on demand with the selector).  factors:
 * nmodes DEVICE pointers, fp32 I_m x rank row-major, in/out (initial guess -> result).
 * fits: host array of >= iters doubles (may be NULL), fit after each sweep; stops early
 * when tol > 0 and |fit_k - fit_{k-1}| < tol.  rank <= 64.  Sharded handles need a comm
 * (sf_comm_attach*) and the SAME initial factors on every rank: each rank computes
 * A_n = M V^+ for its owned rows, the row blocks are allgathered (every rank ends with the
 * full, identical factors) and the Grams / fit terms are summed in rank order.
 * Stream-ordered work, synchronizes once per sweep (to read the fit). */
sf_status sf_cpals(sf_tensor_t t, int rank, float* const* factors, int iters, double tol, double* fits,
                   int* iters_done, void* stream);

/* ---- diagnostics -------------------------------------------------------- */
const char* sf_status_string(sf_status s);
const char* sf_last_error(void);
/* Number of kernels this library has launched in this process (monotone). */
uint64_t sf_kernel_launches(void);
/* Device bytes held by the library's live buffers (all handles, plans, scratch; the block
 * cache's idle blocks excluded) and their high-water mark since the last reset_peak != 0. */
sf_status sf_device_bytes(uint64_t* in_use, uint64_t* peak, int reset_peak);
/* Library version string. */
const char* sf_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SCALFRAG_H */
