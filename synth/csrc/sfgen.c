/*
 * sfgen.c - host batch generator over sfgen_core.h (OpenMP over elements).
 * Holds none of the method's arithmetic; see sfgen_core.h for the recipe.
 */
#include "sfgen_core.h"
#include <stddef.h>

/* Fill inds[m][e - lo] and vals[e - lo] for e in [lo, hi).
 * nb[m], edges[m], thr[m] describe the per-mode power-law table (nb[m]==0: uniform).
 * inds[m] may be NULL to skip a mode; vals may be NULL. */
void sfgen_coo(int nmodes, const uint64_t* dims, uint64_t seed, uint64_t lo, uint64_t hi,
               const int* nb, const uint64_t* const* edges, const uint64_t* const* thr,
               int relabel, int val_kind, uint32_t* const* inds, float* vals) {
  for (int m = 0; m < nmodes; ++m) {
    if (!inds[m]) continue;
    const uint64_t I = dims[m];
    const int half = sfg_feistel_half(I);
    const uint64_t key = sfg_fmix64(seed ^ (SFG_KEY_SALT * (uint64_t)(m + 1)));
    uint32_t* out = inds[m];
    const int nbm = nb ? nb[m] : 0;
    const uint64_t* em = nbm ? edges[m] : NULL;
    const uint64_t* tm = nbm ? thr[m] : NULL;
#pragma omp parallel for schedule(static)
    for (int64_t e = (int64_t)lo; e < (int64_t)hi; ++e)
      out[e - (int64_t)lo] =
          (uint32_t)sfg_index(seed, m, (uint64_t)e, I, nbm, em, tm, relabel, half, key);
  }
  if (vals) {
#pragma omp parallel for schedule(static)
    for (int64_t e = (int64_t)lo; e < (int64_t)hi; ++e)
      vals[e - (int64_t)lo] = sfg_value(sfg_hash(seed, SFG_STREAM_VALUE, (uint64_t)e), val_kind);
  }
}

/* Factor matrix A (rows x rank, row-major): A[i*rank + r] from counter (seed, stream, i*rank+r). */
void sfgen_factor(uint64_t seed, uint64_t stream, uint64_t rows, int rank, int kind, float* out) {
  const int64_t n = (int64_t)(rows * (uint64_t)rank);
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) out[t] = sfg_factor(sfg_hash(seed, stream, (uint64_t)t), kind);
}

/* Exposed for tests: the relabel bijection. */
void sfgen_permute_many(uint64_t I, uint64_t seed, int m, uint64_t n, const uint64_t* in, uint64_t* out) {
  const int half = sfg_feistel_half(I);
  const uint64_t key = sfg_fmix64(seed ^ (SFG_KEY_SALT * (uint64_t)(m + 1)));
  for (uint64_t t = 0; t < n; ++t) out[t] = sfg_permute(in[t], I, half, key);
}

uint64_t sfgen_hash(uint64_t seed, uint64_t stream, uint64_t ctr) { return sfg_hash(seed, stream, ctr); }
