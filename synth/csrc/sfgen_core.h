/*
 * sfgen_core.h - counter-based synthetic-input generator core (integer only).
 *
 * This module is the ONLY code shared between the oracle side and the CUDA
 * side (rule: "only the seeded input generators serve both").  It holds none
 * of the MTTKRP arithmetic: it maps (seed, stream, counter) to 64-bit random
 * words and turns them into COO indices / values / factor entries.  Every
 * draw is a pure function of its coordinates, so generation is chunkable and
 * thread-count independent, and a host and a device build are bit-identical.
 *
 * Recipe:
 *   x = sfg_hash(seed, stream, ctr)        splitmix64-finalizer mixing
 *   uniform index in [0,I)                 mulhi64(x, I)
 *   power-law index (Zipf exponent s)      geometric bucket table: bucket k with
 *                                          probability  ∫_{e_k}^{e_{k+1}} (x+1)^-s dx,
 *                                          uniform inside the bucket; thresholds
 *                                          (uint64) are computed once on the host
 *                                          and passed in as data
 *   relabel                                keyed 4-round Feistel bijection on an
 *                                          even number of bits + cycle walking, so
 *                                          heavy ids are scattered over [0,I)
 */
#ifndef SFGEN_CORE_H
#define SFGEN_CORE_H
#include <stdint.h>

#ifdef __CUDACC__
#define SFG_HD __host__ __device__ __forceinline__
#else
#define SFG_HD static inline
#endif

SFG_HD uint64_t sfg_fmix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

SFG_HD uint64_t sfg_hash(uint64_t seed, uint64_t stream, uint64_t ctr) {
  uint64_t z = sfg_fmix64(seed + 0x9E3779B97F4A7C15ULL * (stream + 1ULL));
  return sfg_fmix64(z ^ (ctr * 0xD6E8FEB86659FD93ULL + 0x632BE59BD9B4E019ULL));
}

SFG_HD uint64_t sfg_mulhi(uint64_t a, uint64_t b) {
#ifdef __CUDA_ARCH__
  return __umul64hi(a, b);
#else
  return (uint64_t)(((unsigned __int128)a * (unsigned __int128)b) >> 64);
#endif
}

/* Number of bits h such that 2^(2h) >= I (even-width Feistel domain). */
SFG_HD int sfg_feistel_half(uint64_t I) {
  int b = 0;
  while (b < 63 && (1ULL << b) < I) ++b;
  return (b + 1) / 2;
}

SFG_HD uint64_t sfg_feistel(uint64_t x, int half, uint64_t key) {
  const uint64_t mask = (half >= 32) ? 0xFFFFFFFFULL : ((1ULL << half) - 1ULL);
  uint64_t L = x >> half, R = x & mask;
  for (int r = 0; r < 4; ++r) {
    uint64_t F = sfg_fmix64(R ^ (key + 0x9E3779B97F4A7C15ULL * (uint64_t)(r + 1))) & mask;
    uint64_t nL = R;
    R = L ^ F;
    L = nL;
  }
  return (L << half) | R;
}

/* Bijection on [0, I): Feistel on [0, 2^(2*half)) with cycle walking. */
SFG_HD uint64_t sfg_permute(uint64_t i, uint64_t I, int half, uint64_t key) {
  if (I <= 1) return 0;
  do { i = sfg_feistel(i, half, key); } while (i >= I);
  return i;
}

/* Draw the mode-m index of element e.
 * nb == 0: uniform.  Otherwise edges[0..nb] (edges[0]=0, edges[nb]=I, strictly
 * increasing) and thr[0..nb-2] (non-decreasing uint64 CDF thresholds). */
SFG_HD uint64_t sfg_index(uint64_t seed, int m, uint64_t e, uint64_t I,
                          int nb, const uint64_t* edges, const uint64_t* thr,
                          int relabel, int half, uint64_t key) {
  uint64_t x1 = sfg_hash(seed, 2ULL * (uint64_t)m, e);
  uint64_t i;
  if (nb <= 0) {
    i = sfg_mulhi(x1, I);
  } else {
    int lo = 0, hi = nb - 1;  /* k = #{ j : thr[j] <= x1 } */
    while (lo < hi) {
      int mid = (lo + hi) >> 1;
      if (thr[mid] <= x1) lo = mid + 1; else hi = mid;
    }
    int k = lo;
    uint64_t x2 = sfg_hash(seed, 2ULL * (uint64_t)m + 1ULL, e);
    i = edges[k] + sfg_mulhi(x2, edges[k + 1] - edges[k]);
  }
  if (relabel) i = sfg_permute(i, I, half, key);
  return i;
}

/* Value kinds. */
enum { SFG_VAL_UNIT = 0,   /* ((x>>40)+1) * 2^-24 in (0,1], exact in fp32 */
       SFG_VAL_SIGNED = 1, /* ((x>>40) - 2^23) * 2^-23 in [-1,1) */
       SFG_VAL_INT = 2,    /* {1,2,3,4} */
       SFG_VAL_ONES = 3,   /* 1 */
       SFG_VAL_BIN = 4 };  /* {0,1} */

SFG_HD float sfg_value(uint64_t x, int kind) {
  switch (kind) {
    case SFG_VAL_UNIT: return (float)((x >> 40) + 1ULL) * (1.0f / 16777216.0f);
    case SFG_VAL_SIGNED: return (float)((int64_t)(x >> 40) - 8388608LL) * (1.0f / 8388608.0f);
    case SFG_VAL_INT: return (float)(1ULL + (x >> 62));
    case SFG_VAL_ONES: return 1.0f;
    default: return (float)(x >> 63);
  }
}

/* Factor kinds reuse the value codes except INT -> {-2..2}, UNIT -> [0,1). */
SFG_HD float sfg_factor(uint64_t x, int kind) {
  switch (kind) {
    case SFG_VAL_UNIT: return (float)(x >> 40) * (1.0f / 16777216.0f);
    case SFG_VAL_SIGNED: return (float)((int64_t)(x >> 40) - 8388608LL) * (1.0f / 8388608.0f);
    case SFG_VAL_INT: return (float)((int64_t)sfg_mulhi(x, 5ULL) - 2LL);
    case SFG_VAL_ONES: return 1.0f;
    default: return (float)(x >> 63);
  }
}

#define SFG_STREAM_VALUE 1000ULL
#define SFG_KEY_SALT 0xA0761D6478BD642FULL

#endif
