// sf_select.cpp - adaptive launch selection (§8(a) A4).
//
// PAPER.md §IV-B (L191-199): "we first extract the characteristic parameters of the
// input tensor ... input these parameters into the trained launch parameter selection
// model.  The model will output an optimal launch parameter combination".  The paper's
// model is a DecisionTree regressor trained on sweeps of its RTX 3090 kernel (L197);
// that model and its training data are prior art for another GPU and another kernel.
// Here the selector is an analytic cost model over the features of PAPER.md L195 plus
// dims / nnz / R / shared-memory capacity, and it is validated against an exhaustive
// launch sweep (tests/test_gpu_select.py, bench.py --sweep).
//
// Decision: which gathered factors to stage in shared memory as blocks ("tensor
// blocks ... based on the resource constraints of hardware") and the
// block sizes; the chunk length C; threads per CTA.
#include <algorithm>
#include <cmath>

#include "sf_internal.h"

namespace sf {

static constexpr int kStagesHost = 2;  // must match frag_kernel's kStages

size_t frag_smem_bytes(const Tensor& t, int mode, int rank, const sf_launch_t& l) {
  (void)mode;
  size_t b = 128 + (size_t)kStagesHost * (t.nmodes + 1) * ((size_t)l.chunk_nnz + 8) * 4;
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
  if (l.chunk_nnz <= 0) l.chunk_nnz = 1024;
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
}

// Rough per-nonzero cost model in "on-chip bytes".
struct Cand {
  uint32_t mask;
  uint32_t rows[SF_MAX_MODES];
  double cost;
};

sf_launch_t select_launch(const Tensor& t, const sf_features_t& f, int mode, int rank,
                          uint64_t nnz_local) {
  sf_launch_t l{};
  const int N = t.nmodes;
  l.kernel = frag_supported(N, rank) ? SF_KERNEL_FRAG : SF_KERNEL_COO;
  l.block_threads = 512;
  l.ctas_per_sm = 0;
  l.chunk_nnz = 1024;
  l.staged_mask = 0;
  if (l.kernel != SF_KERNEL_FRAG || nnz_local == 0) {
    normalize_launch(t, mode, rank, l);
    return l;
  }
  const double R4 = 4.0 * rank;
  const double L2 = 96.0 * 1024 * 1024;  // usable L2 for factors (of ~126 MB)
  const size_t base_smem = frag_smem_bytes(t, mode, rank, l);
  const double budget_rows =
      std::floor(((double)t.smem_optin - (double)base_smem - 1024.0) / R4);
  double total_fac = 0;
  for (int m = 0; m < N; ++m)
    if (m != mode) total_fac += (double)t.dims[m] * R4;
  const double nnz = (double)nnz_local;
  const double slices = std::max<double>(1.0, (double)f.num_slices);
  Cand best{0, {}, 1e300};
  const int G = N - 1;
  int gm[SF_MAX_MODES], k = 0;
  for (int m = 0; m < N; ++m)
    if (m != mode) gm[k++] = m;
  for (uint32_t sub = 0; sub < (1u << G); ++sub) {
    Cand c{0, {}, 0};
    int ns = 0;
    for (int q = 0; q < G; ++q)
      if (sub & (1u << q)) { c.mask |= 1u << gm[q]; ++ns; }
    // block rows: small modes whole, the rest share the remaining budget equally
    double rows_left = budget_rows;
    int left = ns;
    bool ok = true;
    std::vector<int> order;
    for (int q = 0; q < G; ++q)
      if (sub & (1u << q)) order.push_back(gm[q]);
    std::sort(order.begin(), order.end(), [&](int a, int b) { return t.dims[a] < t.dims[b]; });
    for (int m : order) {
      const double share = std::floor(rows_left / left);
      if (share < 64) { ok = false; break; }
      const double r = std::min<double>((double)t.dims[m], share);
      c.rows[m] = (uint32_t)r;
      rows_left -= r;
      --left;
    }
    if (!ok) continue;
    double T = 1;
    double staged_rows = 0;
    for (int m : order) {
      T *= std::ceil((double)t.dims[m] / c.rows[m]);
      staged_rows += c.rows[m];
    }
    double cost = 4.0 * (N + 1);  // stream bytes (HBM)
    // gathers of non-staged modes: L2 hits ~1.0 per byte; misses to HBM much worse
    double unstaged_fac = 0;
    for (int q = 0; q < G; ++q)
      if (!(sub & (1u << q))) unstaged_fac += (double)t.dims[gm[q]] * R4;
    const double l2_w = unstaged_fac <= L2 ? 1.0 : 1.0 + 2.0 * (1.0 - L2 / unstaged_fac);
    for (int q = 0; q < G; ++q)
      if (!(sub & (1u << q))) cost += R4 * l2_w;
    cost += ns * R4 * 0.35;                                   // shared-memory gathers
    const double tiles_touched = std::min(T, nnz);
    const double ctas = (double)t.num_sms;
    cost += (staged_rows * R4) * (tiles_touched + ctas) / nnz;  // block staging traffic
    const double pairs = std::min(nnz, tiles_touched * slices);  // (tile,row) runs
    cost += R4 * 1.5 * (pairs / nnz + 0.05);                     // flush atomics
    c.cost = cost;
    if (c.cost < best.cost) best = c;
  }
  l.staged_mask = best.mask;
  for (int m = 0; m < N; ++m) l.block_rows[m] = (best.mask & (1u << m)) ? best.rows[m] : 0;
  (void)total_fac;
  normalize_launch(t, mode, rank, l);
  return l;
}

}  // namespace sf
