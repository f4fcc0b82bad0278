/*
 * oracle.c - TEST INFRASTRUCTURE ONLY.  Plain, slow, single-threaded fp64 CPU
 * implementation of what ScalFrag's hot path computes.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load it.  It shares no code with the CUDA path
 * (paper_conf_cluster_linwds24_b200/csrc) and neither includes the other.
 *
 * or_mttkrp follows the plain definition of mode-n MTTKRP
 * (§II-C, Eq. (4)):  M = X_(n) (A^(N) ⊙ ... ⊙ A^(n+1) ⊙ A^(n-1) ⊙ ... ⊙ A^(1)),
 * written elementwise for a COO tensor (§II-D):
 *
 *     Y(i, r) = sum_{e : i_n(e) = i}  v_e * prod_{m != n} A_m(i_m(e), r)
 *
 * (the column of X_(n) that holds element e meets the Khatri-Rao row that is the
 * product of the matching factor rows; reading R1).  Rows with no
 * nonzero are 0 ("M <-", Alg. 1 line 4: overwrite; reading R6).
 * Duplicated coordinates are summed (MTTKRP is linear in X; reading R5).
 * Alongside Y it returns the scale S(i,r) = sum |v_e * prod A_m(i_m(e), r)| that the
 * acceptance test divides by (north_star: "max |Δ|/(|v|·∏|A| row-scale) ≤ 1e-4").
 *
 * Steps, in input order:
 *   1. Y = 0, S = 0   (I_n x R, fp64)
 *   2. for e = 0..nnz-1:  i = i_n(e);  for r: p = (double)v_e;
 *        for m = 0..N-1, m != n, ascending: p *= (double)A_m(i_m(e), r);
 *        Y(i,r) += p;  S(i,r) += |p|
 * fp32 inputs convert to fp64 exactly.
 *
 * Pins: tests/test_oracle.py (brute force vs dense unfolding x explicit
 * Khatri-Rao product, rank-1 closed form, slice sums, exact integers, SpMM,
 * invariants, hand-computed golden fixture).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* Returns 0 on success, -1 on invalid arguments, -2 on an out-of-range index. */
int or_mttkrp(int nmodes, const uint64_t* dims, uint64_t nnz, const uint32_t* const* inds,
              const float* vals, const float* const* factors, int rank, int mode, double* Y,
              double* S) {
  if (nmodes < 1 || rank < 1 || mode < 0 || mode >= nmodes) return -1;
  const uint64_t In = dims[mode];
  memset(Y, 0, sizeof(double) * In * (uint64_t)rank);
  if (S) memset(S, 0, sizeof(double) * In * (uint64_t)rank);
  for (uint64_t e = 0; e < nnz; ++e) {
    for (int m = 0; m < nmodes; ++m)
      if ((uint64_t)inds[m][e] >= dims[m]) return -2;
    const uint64_t i = inds[mode][e];
    for (int r = 0; r < rank; ++r) {
      double p = (double)vals[e];
      for (int m = 0; m < nmodes; ++m) {
        if (m == mode) continue;
        p *= (double)factors[m][(uint64_t)inds[m][e] * (uint64_t)rank + (uint64_t)r];
      }
      Y[i * (uint64_t)rank + (uint64_t)r] += p;
      if (S) S[i * (uint64_t)rank + (uint64_t)r] += fabs(p);
    }
  }
  return 0;
}

/* Same definition restricted to sampled rows: slot[i] >= 0 selects row i and names
 * its output row in Y/S (nslots x R).  One streaming pass over the nonzeros, so the
 * full-size configs can be checked row by row without an I_n x R fp64 buffer. */
int or_mttkrp_rows(int nmodes, const uint64_t* dims, uint64_t nnz, const uint32_t* const* inds,
                   const float* vals, const float* const* factors, int rank, int mode,
                   const int32_t* slot, int64_t nslots, double* Y, double* S) {
  if (nmodes < 1 || rank < 1 || mode < 0 || mode >= nmodes) return -1;
  memset(Y, 0, sizeof(double) * (uint64_t)nslots * (uint64_t)rank);
  if (S) memset(S, 0, sizeof(double) * (uint64_t)nslots * (uint64_t)rank);
  for (uint64_t e = 0; e < nnz; ++e) {
    const uint64_t i = inds[mode][e];
    if (i >= dims[mode]) return -2;
    const int32_t s = slot[i];
    if (s < 0) continue;
    for (int r = 0; r < rank; ++r) {
      double p = (double)vals[e];
      for (int m = 0; m < nmodes; ++m) {
        if (m == mode) continue;
        p *= (double)factors[m][(uint64_t)inds[m][e] * (uint64_t)rank + (uint64_t)r];
      }
      Y[(uint64_t)s * (uint64_t)rank + (uint64_t)r] += p;
      if (S) S[(uint64_t)s * (uint64_t)rank + (uint64_t)r] += fabs(p);
    }
  }
  return 0;
}
