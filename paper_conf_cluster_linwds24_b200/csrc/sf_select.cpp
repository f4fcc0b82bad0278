// sf_select.cpp - adaptive launch selection (§8(a) A4).
//
// PAPER.md §IV-B (L191-199): "we first extract the characteristic parameters of the
// input tensor ... input these parameters into the trained launch parameter selection
// model.  The model will output an optimal launch parameter combination".  The paper's
// model is a DecisionTree regressor trained on sweeps of its RTX 3090 kernel (L197);
// that model and its training data are prior art for another GPU and another kernel.
// Here the selector is a set of rules over the features of PAPER.md L195 plus dims /
// nnz / R / shared-memory capacity, calibrated on and validated against an exhaustive
// launch sweep (sweep.py; DESIGN.md §5 Selector).
//
// Decision: which gathered factors to stage in shared memory as blocks ("tensor
// blocks ... based on the resource constraints of hardware") and the
// block sizes; the chunk length C; threads per CTA.
#include <algorithm>
#include <cmath>
#include <cstdlib>

#include "sf_internal.h"

namespace sf {

static constexpr int kStagesHost = 2;  // must match kFragStages (sf_frag.cuh)

// Shared memory of frag3_kernel: mbarriers (2 per warp + 1), per warp a double-buffered
// stage of GPW regions of K = C / GPW records (C = chunk_nnz, nonzeros per warp per
// stage), and the staged factor blocks.
size_t frag_smem_bytes(const Tensor& t, int mode, int rank, const sf_launch_t& l) {
  (void)mode;
  const size_t nwarps = (size_t)std::max(1, l.block_threads / 32);
  size_t b = ((2 * nwarps + 1) * 8 + 127) & ~(size_t)127;
  // frag3: per warp 2 stages x GPW regions of K records
  const uint32_t gpw = (uint32_t)frag_groups_per_warp(rank);
  const uint32_t K = frag3_K((uint32_t)l.chunk_nnz, gpw);
  b += nwarps * kStagesHost * gpw * (size_t)frag3_region_words(K, (uint32_t)tensor_rec_words(t)) * 4;
  if (!(l.flags & SF_LAUNCH_L2_TILES))
    for (int m = 0; m < t.nmodes; ++m)
      if (l.staged_mask & (1u << m)) b += (size_t)l.block_rows[m] * rank * 4;
  return b;
}

void normalize_launch(const Tensor& t, int mode, int rank, sf_launch_t& l) {
  const int N = t.nmodes;
  if (l.kernel != SF_KERNEL_COO && l.kernel != SF_KERNEL_FRAG) l.kernel = SF_KERNEL_FRAG;
  if (l.kernel == SF_KERNEL_FRAG && !frag_supported(N, rank)) l.kernel = SF_KERNEL_COO;
  l.block_threads = std::min(1024, std::max(64, (l.block_threads / 32) * 32));
  if (l.ctas_per_sm < 0) l.ctas_per_sm = 0;
  if (l.chunk_nnz <= 0) l.chunk_nnz = 128;
  l.chunk_nnz = std::min(16384, std::max(16, (l.chunk_nnz + 3) / 4 * 4));
  uint32_t mask = 0;
  for (int m = 0; m < N; ++m) {
    if (m == mode || !(l.staged_mask & (1u << m))) { l.block_rows[m] = 0; continue; }
    uint32_t br = l.block_rows[m];
    if (br == 0) continue;
    br = (uint32_t)std::min<uint64_t>(br, t.dims[m]);
    l.block_rows[m] = br;
    mask |= 1u << m;
  }
  for (int m = N; m < SF_MAX_MODES; ++m) l.block_rows[m] = 0;
  l.staged_mask = (l.kernel == SF_KERNEL_FRAG) ? mask : 0u;
  if (l.flags & SF_LAUNCH_DETERMINISTIC) {  // A7 option: unstaged owner-store plan (no atomics)
    l.staged_mask = 0u;
    for (int m = 0; m < SF_MAX_MODES; ++m) l.block_rows[m] = 0;
    l.flags &= ~(SF_LAUNCH_NO_OWNER_STORES | SF_LAUNCH_L2_TILES);
  }
  if (l.staged_mask == 0u) l.flags &= ~SF_LAUNCH_L2_TILES;
  l.flags &= (SF_LAUNCH_NO_OWNER_STORES | SF_LAUNCH_DETERMINISTIC | SF_LAUNCH_L2_TILES);
  if (l.kernel != SF_KERNEL_FRAG) l.hot_kb = 0;
  l.hot_kb = std::min<uint32_t>(l.hot_kb, 4u << 20);  // 4 GiB
}

// Selector rules, calibrated on the sweeps in profiles/:
//  * a gathered mode is staged WHOLE (one tile, loaded once per CTA) when its factor
//    fits the shared-memory budget next to the stream stages;
//  * otherwise the gathered mode with the most reuse is staged in BLOCKS if every staged
//    row is reused often inside its tile: nnz / I_m >= kMinReuse
//    (hyper-sparse tensors lose to block staging by up to 1000x: each tile would be
//    staged for a handful of nonzeros);
//  * at most one block-staged mode (two block-staged modes multiply the tile count and
//    split output-row runs into short (tile,row) pieces whose flushes dominate);
//  * per-warp chunks of C = 128 nonzeros, 512 threads (sweep optima, profiles/).
static constexpr double kMinReuse = 256.0;
static constexpr uint32_t kBlockRows = 256;

static sf_launch_t select_rules(const Tensor& t, const sf_features_t& f, int mode, int rank,
                               uint64_t nnz_local) {
  (void)f;
  sf_launch_t l{};
  const int N = t.nmodes;
  l.kernel = frag_supported(N, rank) ? SF_KERNEL_FRAG : SF_KERNEL_COO;
  l.block_threads = 512;
  l.ctas_per_sm = 0;
  l.chunk_nnz = 128;
  l.staged_mask = 0;
  if (l.kernel != SF_KERNEL_FRAG || nnz_local == 0) {
    normalize_launch(t, mode, rank, l);
    return l;
  }
  const double R4 = 4.0 * rank;
  // 1) whole-mode staging of small modes (largest first that fits)
  // keep two CTAs per SM: half the shared memory per CTA
  double budget = (double)t.smem_optin / 2 - (double)frag_smem_bytes(t, mode, rank, l) - 1024.0;
  int order[SF_MAX_MODES], k = 0;
  for (int m = 0; m < N; ++m)
    if (m != mode) order[k++] = m;
  std::sort(order, order + k, [&](int a, int b) { return t.dims[a] < t.dims[b]; });
  for (int q = 0; q < k; ++q) {
    const int m = order[q];
    const double bytes = (double)t.dims[m] * R4;
    if (bytes <= budget) {
      l.staged_mask |= 1u << m;
      l.block_rows[m] = (uint32_t)t.dims[m];
      budget -= bytes;
    }
  }
  // 2) otherwise block-stage the gathered mode whose rows are reused most, if every staged
  //    row is reused >= kMinReuse times on average (nnz / I_m)
  if (l.staged_mask == 0) {
    int best = -1;
    double reuse = 0;
    for (int q = 0; q < k; ++q) {
      const int m = order[q];
      const double r = (double)nnz_local / (double)t.dims[m];
      // tiny factors (< 512 KB) stay hot in L1/L2 anyway: staging them only costs smem
      if ((double)t.dims[m] * R4 < 512.0 * 1024) continue;
      if (r >= kMinReuse && r > reuse) { best = m; reuse = r; }
    }
    if (best >= 0) {
      l.staged_mask = 1u << best;
      l.block_rows[best] = kBlockRows;
    }
  }
  normalize_launch(t, mode, rank, l);
  if (frag_smem_bytes(t, mode, rank, l) > t.smem_optin) {  // safety: drop staging
    l.staged_mask = 0;
    normalize_launch(t, mode, rank, l);
  }
  return l;
}

// ---------------------------------------------------------------------------
// Learned selector (§IV-B).  Features of the tensor
// and mode -> a DecisionTree (trained offline on sweeps of synthetic *training* tensors,
// tools/train_selector.py) -> one of kNumCandidates launch classes.  Classes are defined
// relative to the gathered modes sorted by dimension so one model serves every mode.
// ---------------------------------------------------------------------------
static int gathered_sorted(const Tensor& t, int mode, int* g) {
  int k = 0;
  for (int m = 0; m < t.nmodes; ++m)
    if (m != mode) g[k++] = m;
  std::sort(g, g + k, [&](int a, int b) { return t.dims[a] < t.dims[b] || (t.dims[a] == t.dims[b] && a < b); });
  return k;
}

static inline double lg2(double x) { return std::log2(std::max(x, 1.0)); }

int selector_features(const Tensor& t, const sf_features_t& f, int mode, int rank, uint64_t nnz_local,
                      double* x) {
  int g[SF_MAX_MODES];
  const int k = gathered_sorted(t, mode, g);
  const double nnz = (double)std::max<uint64_t>(nnz_local, 1);
  const double R4 = 4.0 * rank;
  double fac = 0;
  for (int q = 0; q < k; ++q) fac += (double)t.dims[g[q]] * R4;
  int i = 0;
  x[i++] = t.nmodes;
  x[i++] = rank;
  x[i++] = lg2(nnz);
  x[i++] = lg2((double)t.dims[mode]);
  x[i++] = lg2((double)t.dims[g[0]]);                        // smallest gathered dim
  x[i++] = k >= 3 ? lg2((double)t.dims[g[1]]) : 0.0;         // middle (4-way+)
  x[i++] = lg2((double)t.dims[g[k - 1]]);                    // largest gathered dim
  x[i++] = lg2(nnz / (double)t.dims[g[0]]);                  // reuse of the smallest
  x[i++] = lg2(nnz / (double)t.dims[g[k - 1]]);              // reuse of the largest
  x[i++] = lg2(f.avg_nnz_per_slice);
  x[i++] = lg2((double)f.max_nnz_per_slice);
  x[i++] = f.avg_nnz_per_slice > 0 ? f.std_nnz_per_slice / f.avg_nnz_per_slice : 0.0;
  x[i++] = f.slice_ratio;
  x[i++] = f.fiber_ratio;
  x[i++] = lg2(f.avg_nnz_per_fiber * 16.0);
  x[i++] = lg2(fac);                                         // gathered factor bytes
  x[i++] = lg2((double)t.dims[mode] * R4);                   // Y bytes
  x[i++] = lg2((double)t.dims[g[0]] * R4);                   // smallest factor bytes
  return i;
}

int selector_candidates(const Tensor& t, int mode, int rank, sf_launch_t* out) {
  int g[SF_MAX_MODES];
  const int k = gathered_sorted(t, mode, g);
  sf_launch_t base{};
  base.kernel = frag_supported(t.nmodes, rank) ? SF_KERNEL_FRAG : SF_KERNEL_COO;
  base.block_threads = 512;
  base.chunk_nnz = 128;
  int n = 0;
  auto add = [&](int stage_mode, uint32_t rows, uint32_t flags) {
    sf_launch_t l = base;
    l.flags |= flags;
    if (stage_mode >= 0) {
      l.staged_mask = 1u << stage_mode;
      l.block_rows[stage_mode] = rows;
    }
    normalize_launch(t, mode, rank, l);
    out[n++] = l;
  };
  add(-1, 0, 0);                          // 0 unstaged, owner stores
  add(-1, 0, SF_LAUNCH_NO_OWNER_STORES);  // 1 unstaged, memset + atomics
  add(g[0], 256, 0);                      // 2 stage smallest gathered mode, 256-row blocks
  add(g[0], 512, 0);                      // 3                              512-row blocks
  add(g[k - 1], 256, 0);                  // 4 stage largest gathered mode, 256-row blocks
  add(g[k - 1], 512, 0);                  // 5                              512-row blocks
  add(k >= 3 ? g[1] : g[0], 256, 0);      // 6 stage middle gathered mode (4-way), 256
  // L2-tiled classes (SF_LAUNCH_L2_TILES, DESIGN.md §5 "L2 tiles"): blocks of a gathered factor
  // swept by every CTA in tile order; a factor smaller than its block degenerates to class 1
  const double RB = 4.0 * rank;
  auto rows_for = [&](double bytes) { return (uint32_t)std::max(1.0, bytes / RB); };
  add(g[k - 1], rows_for(64.0 * 1024 * 1024), SF_LAUNCH_L2_TILES);              // 7 largest, 64 MB
  add(k >= 2 ? g[k - 2] : g[k - 1], rows_for(64.0 * 1024 * 1024), SF_LAUNCH_L2_TILES);  // 8 2nd largest
  add(g[k - 1], rows_for(16.0 * 1024 * 1024), SF_LAUNCH_L2_TILES);              // 9 largest, 16 MB
  return n;
}

struct TreeModel {
  std::vector<int32_t> feature, left, right, value;
  std::vector<double> threshold;
  int nfeat = 0;
  bool l2_classes = false;  // trained with the L2-tiled classes (7-9): no hand rule on top
};
static TreeModel g_model;
static bool g_have_model = false;

// The deployed model (selector_model.json) is compiled in (build/sf_selector_model.inc,
// written by _build.py) and installed when the library loads, so a C caller gets the same
// launch as the tests and the bench; sf_set_selector_model replaces it (n_nodes = 0: rules).
#include "sf_selector_model.inc"
static const bool g_default_model_installed = [] {
  set_selector_model(kModel_feature, kModel_threshold, kModel_left, kModel_right, kModel_value, kModelNodes,
                     kModelFeatures);
  return true;
}();

void set_selector_model(const int32_t* feature, const double* threshold, const int32_t* left,
                        const int32_t* right, const int32_t* value, int n_nodes, int n_features) {
  if (n_nodes <= 0) {
    g_have_model = false;
    return;
  }
  g_model.feature.assign(feature, feature + n_nodes);
  g_model.threshold.assign(threshold, threshold + n_nodes);
  g_model.left.assign(left, left + n_nodes);
  g_model.right.assign(right, right + n_nodes);
  g_model.value.assign(value, value + n_nodes);
  g_model.nfeat = n_features;
  g_model.l2_classes = false;
  for (int i = 0; i < n_nodes; ++i)
    if (left[i] < 0 && value[i] >= 7) g_model.l2_classes = true;
  g_have_model = true;
}

static int tree_predict(const double* x, int nx) {
  int node = 0;
  for (int depth = 0; depth < 64; ++depth) {
    const int l = g_model.left[node], r = g_model.right[node];
    if (l < 0 || r < 0) return g_model.value[node];
    const int fi = g_model.feature[node];
    const double v = (fi >= 0 && fi < nx) ? x[fi] : 0.0;
    node = (v <= g_model.threshold[node]) ? l : r;
    if (node < 0 || node >= (int)g_model.feature.size()) return -1;
  }
  return -1;
}

// ---------------------------------------------------------------------------
// L2-tile refinement (SF_LAUNCH_L2_TILES; DESIGN.md §5 "L2 tiles").  When the pick is an
// unstaged plan (the hyper-sparse regime: factors >> L2, gathers DRAM-latency bound), tile
// the order by 64 MB row blocks of the LARGEST gathered factor of >= 160 MB, so at any moment
// every CTA gathers that factor from one L2-resident block -- unless re-visiting Y once per
// (tile, row) costs too much: rho = T * touched(T) / nnz <= 0.25, touched(T) = the expected
// rows of Y a tile touches, sum_b slices_b (1 - exp(-1.44 * 2^b / T)) over the log2
// slice-length histogram (PAPER.md L195 features); rho = 0 when Y fits in 32 MB (its
// re-visits hit L2).  Calibrated on tools/l2tile_study.py over the BASELINE.json and Table III
// shapes (profiles/r01s3_l2tiles.jsonl) and 16 random tensors (53 modes,
// profiles/r01s3_l2tiles_random.jsonl): over the random set the rule is 1.14x over no tiling
// (geomean; best possible 1.175x), within 3.3 % of the best option on average, never worse
// than 0.98x.  The 160 MB floor comes from the random set (64 MB tiled 146 MB factors at 0.78x).
static constexpr double kL2BlockBytes = 64.0 * 1024 * 1024;
static constexpr double kL2MinFactorBytes = 160.0 * 1024 * 1024;  // ~1.3x L2: smaller factors keep their hot rows
static constexpr double kL2MaxRevisit = 0.25;
static constexpr double kL2YInCache = 32.0 * 1024 * 1024;

// expected Y revisit ratio of tiling the order by T blocks: T * touched(T) / nnz, touched(T) =
// the expected rows of Y a tile touches from the log2 slice-length histogram
static double revisit_ratio(const sf_features_t& f, double T) {
  double touched = 0;
  for (int b = 0; b < SF_HIST_BINS; ++b)
    touched += (double)f.slice_hist[b] * (1.0 - std::exp(-1.44 * std::ldexp(1.0, b) / T));
  return f.nnz ? T * touched / (double)f.nnz : 0.0;
}

static void l2_tile_refine(const Tensor& t, const sf_features_t& f, int mode, int rank, uint64_t nnz_local,
                           sf_launch_t& l) {
  if (l.kernel != SF_KERNEL_FRAG || l.staged_mask != 0 || (l.flags & SF_LAUNCH_DETERMINISTIC) || nnz_local == 0 ||
      f.nnz == 0)
    return;
  const double RB = 4.0 * rank, Yb = (double)t.dims[mode] * RB;
  const char* env = debug_opt("l2_revisit");  // SF_DEBUG calibration override of kL2MaxRevisit
  const double max_revisit = (env && *env) ? std::atof(env) : kL2MaxRevisit;
  int best = -1;
  double bestF = 0;
  for (int m = 0; m < t.nmodes; ++m) {
    if (m == mode) continue;
    const double F = (double)t.dims[m] * RB;
    if (F < kL2MinFactorBytes || F <= bestF) continue;
    const double T = std::ceil(F / kL2BlockBytes);
    const double rho = (Yb > kL2YInCache) ? revisit_ratio(f, T) : 0.0;
    if (rho > max_revisit) continue;
    best = m;
    bestF = F;
  }
  if (best < 0) return;
  sf_launch_t c = l;
  c.staged_mask = 1u << best;
  c.block_rows[best] = (uint32_t)std::max(1.0, kL2BlockBytes / RB);
  c.flags = (c.flags | SF_LAUNCH_L2_TILES) & ~SF_LAUNCH_NO_OWNER_STORES;
  normalize_launch(t, mode, rank, c);
  if (frag_smem_bytes(t, mode, rank, c) <= t.smem_optin) l = c;
}

static bool l2_refine_enabled() {
  return !debug_opt("no_l2tiles");  // SF_DEBUG A/B: keep the selector's unstaged pick
}

// ---------------------------------------------------------------------------
// Hot-row cache (launch.hot_kb; DESIGN.md §5 "hot-row cache").  Random 128-byte row gathers
// from a factor spread over hundreds of MB run at ~4.6 TB/s whether or not the rows hit L2,
// while the same gathers from a dense 32 MB block run at ~15 TB/s (tools/micro/l2_hot.cu,
// profiles/r02/micro_l2hot.txt): the scattered hot rows cost TLB reach, not DRAM bytes.
// Copying the most frequent rows into one dense block per call (a few tens of us) gave
// 1.3-1.5x on nell-1- and amazon-shaped gathers in the microbenchmark; in frag3 on nell-1
// 16-32 MB blocks are best (mode 2: 7.01 -> 4.68 ms; 128 MB 4.86, 256 MB 6.02;
// profiles/r02/hot_sweep_*.jsonl).  Enabled when the gathered factors that are neither
// staged nor L2-tiled total more than ~1.3x L2.
// ---------------------------------------------------------------------------
static constexpr double kHotMinGatheredBytes = 160.0 * 1024 * 1024;
static constexpr uint32_t kHotKB = 32 * 1024, kHotKBTiled = 16 * 1024;
// hot rows + L2 tiles: tile one gathered factor by blocks of 2^19 rows (64 MB at R = 32, 32 MB at
// R = 16; 2..32 tiles, Y revisit ratio rho <= 0.10) and hot-cache the others (16 MB) -- but only
// a factor the hot-row cache would serve badly: the share of nonzeros whose index is among its
// hottest 16 MB of rows (t.hot_cover, measured by the planner) must be < 0.8, and of several
// candidates the least-covered one is tiled.  Fitted on 70 modes (16 random hyper-sparse tensors
// + the BASELINE / Table III shapes, tools/hot_heldout.py --seed 78, tools/fit_tile_rule.py:
// best / chosen 0.988 mean) and checked on 39 held-out modes (--seed 77): 0.977 mean vs 0.938
// for hot rows alone and 0.946 for the previous 3-way-only rule (profiles/r02/hot_rule/).
static constexpr double kHotTileMaxTiles = 32, kHotTileMaxRevisit = 0.10, kHotTileMaxCover = 0.8;
static constexpr uint32_t kHotTileRows = 1u << 19;

bool hot_tile_candidate(const Tensor& t, int mode, int rank, int m) {
  (void)rank;
  if (m == mode) return false;
  const double T = std::ceil((double)t.dims[m] / kHotTileRows);
  return T >= 2 && T <= kHotTileMaxTiles;
}

static void hot_tile_refine(const Tensor& t, const sf_features_t& f, int mode, int rank, sf_launch_t& l) {
  if (l.hot_kb == 0 || l.staged_mask != 0 || f.nnz == 0) return;
  const double RB = 4.0 * rank, Yb = (double)t.dims[mode] * RB;
  int best = -1;
  double bestCover = kHotTileMaxCover;
  for (int m = 0; m < t.nmodes; ++m) {
    if (!hot_tile_candidate(t, mode, rank, m) || t.hot_cover[m] < 0) continue;
    const double T = std::ceil((double)t.dims[m] / kHotTileRows);
    if ((Yb > kL2YInCache ? revisit_ratio(f, T) : 0.0) > kHotTileMaxRevisit) continue;
    if (t.hot_cover[m] < bestCover) {
      best = m;
      bestCover = t.hot_cover[m];
    }
  }
  if (best < 0) return;
  sf_launch_t c = l;
  c.staged_mask = 1u << best;
  c.block_rows[best] = kHotTileRows;
  c.flags = (c.flags | SF_LAUNCH_L2_TILES) & ~SF_LAUNCH_NO_OWNER_STORES;
  c.hot_kb = kHotKBTiled;
  c.chunk_nnz = 128;
  normalize_launch(t, mode, rank, c);
  if (frag_smem_bytes(t, mode, rank, c) <= t.smem_optin) l = c;
}

static void hot_refine(const Tensor& t, int mode, int rank, sf_launch_t& l) {
  if (l.kernel != SF_KERNEL_FRAG || (l.flags & SF_LAUNCH_DETERMINISTIC) || (l.flags & SF_LAUNCH_L2_TILES)) return;
  double gathered = 0;
  for (int m = 0; m < t.nmodes; ++m) {
    if (m == mode || (l.staged_mask & (1u << m))) continue;
    const double F = (double)t.dims[m] * rank * 4.0;
    if (F >= 16.0 * 1024 * 1024) gathered += F;
  }
  if (gathered < kHotMinGatheredBytes || debug_opt("no_hot")) return;  // SF_DEBUG A/B
  // a shared-memory-staged pick of a small factor next to >= 160 MB of gathered factors is
  // replaced by the (unstaged) hot-row class: staging + hot rows measured no better than hot
  // rows alone on deli-4d, and a held-out 4-way tensor ran 1.7x faster unstaged with hot rows
  l.staged_mask = 0;
  for (int m = 0; m < SF_MAX_MODES; ++m) l.block_rows[m] = 0;
  // the hot-row class: owner stores, 1024 threads (one CTA per SM), 32 MB of hot rows, no L2
  // tiles, and stages of 4 register batches per lane group (chunk = 8 groups x 4 x U nonzeros:
  // 64 at R >= 32 where U = 2, 128 at R = 16 where U = 4) -- the best fixed class over the
  // exhaustive sparse sweeps (sweep.py --sparse, 143-283 launches per mode, nell-1, deli-4d,
  // flickr-3d, deli-3d, flickr-4d: profiles/r02/sweeps/); L2 tiles on top of the hot rows won
  // only 1-7 % on 6 of 17 modes and lost up to 20 % on others
  l.hot_kb = (l.flags & SF_LAUNCH_L2_TILES) ? kHotKBTiled : kHotKB;
  l.block_threads = 1024;
  l.chunk_nnz = rank >= 32 ? 64 : 128;
  l.ctas_per_sm = 0;
  l.flags &= ~SF_LAUNCH_NO_OWNER_STORES;
  normalize_launch(t, mode, rank, l);
  if (frag_smem_bytes(t, mode, rank, l) > t.smem_optin) l.hot_kb = 0;
}

sf_launch_t select_launch(const Tensor& t, const sf_features_t& f, int mode, int rank, uint64_t nnz_local) {
  sf_launch_t l{};
  bool picked = false;
  // the tree was trained on 1e6..3e7-nonzero tensors; below 2^20 nonzeros the launch is latency-
  // bound (~10 us) and the rule selector (stage every small factor whole) is within 5 % of the
  // sweep best on configs[0] (profiles/r02/sweeps/sweep_tiny.jsonl), the tree's picks 0.55-0.87
  if (g_have_model && frag_supported(t.nmodes, rank) && nnz_local >= (1u << 20)) {
    double x[32];
    const int nx = selector_features(t, f, mode, rank, nnz_local, x);
    if (nx == g_model.nfeat) {
      const int c = tree_predict(x, nx);
      sf_launch_t cand[16];
      const int nc = selector_candidates(t, mode, rank, cand);
      if (c >= 0 && c < nc && frag_smem_bytes(t, mode, rank, cand[c]) <= t.smem_optin) {
        l = cand[c];
        picked = true;
      }
    }
  }
  if (!picked) l = select_rules(t, f, mode, rank, nnz_local);
  // hot-row cache first: where it applies it beats L2 tiles alone (deli-4d 1.2-1.8x, flickr-3d
  // 1.2x per mode) or ties them (nell-1), profiles/r02/hot_sweep_g06.jsonl; then L2 tiles of one
  // poorly-cached factor on top (hot_tile_refine): amazon 0.81x / nell-1 0.96-0.99x the
  // hot-only time, profiles/r02/sweeps/ and profiles/r02/hot_rule/
  hot_refine(t, mode, rank, l);
  if (l.hot_kb != 0) {
    if (l2_refine_enabled()) hot_tile_refine(t, f, mode, rank, l);
  } else if (l2_refine_enabled() && !(picked && g_model.l2_classes)) {
    // the hand rule refines picks of a selector that cannot choose L2 tiles itself
    l2_tile_refine(t, f, mode, rank, nnz_local, l);
  }
  return l;
}

}  // namespace sf
