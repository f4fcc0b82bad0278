// sf_cpals.cu - CP-ALS driver, the consumer of the hot path.
//
// Algorithm 1 of the paper (§II-B):
//   repeat: for n = 1..N:
//     V    <- Hadamard product of the Grams A_m^T A_m, m != n          (line 3)
//     M    <- X_(n) (A(N) ⊙ ... ⊙ A(1)), i.e. sf_mttkrp(mode n)       (line 4)
//     A(n) <- M V^†                                                     (line 5)
// The Grams are kept in fp64 and only G_n is recomputed after A(n) changes.  V^† is
// computed by Gauss-Jordan elimination with partial pivoting in fp64 in one CTA; pivots
// below 1e-12 of the largest diagonal entry are dropped (their row/column of V^† is zero),
// which equals the pseudo-inverse for full-rank V and approximates it otherwise
// (reading R16).  No column normalisation (Alg. 1 has none).  The fit uses the
// identity ||X - [[A]]||^2 = ||X||^2 + sum_rs prod_m G_m(r,s) - 2 <M_N, A_N>.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <vector>

#include "sf_internal.h"

namespace sf {

// G += A^T A (fp64), A is I x R row-major.  Tiles of 64 rows staged in shared memory;
// each thread owns R*R/blockDim entries, sums a tile in fp32 then folds into fp64.
__global__ void gram_kernel(const float* __restrict__ A, uint64_t I, int R, double* __restrict__ G) {
  extern __shared__ float tile[];  // 64 x R
  constexpr int TR = 64;
  const int RR = R * R;
  double acc[16];
  for (int q = 0; q < 16; ++q) acc[q] = 0.0;
  const uint64_t ntiles = (I + TR - 1) / TR;
  for (uint64_t tb = blockIdx.x; tb < ntiles; tb += gridDim.x) {
    const uint64_t r0 = tb * TR;
    const int rows = (I - r0 < (uint64_t)TR) ? (int)(I - r0) : TR;
    for (int e = threadIdx.x; e < TR * R; e += blockDim.x) {
      const int rr = e / R;
      tile[e] = rr < rows ? A[(r0 + rr) * R + (e - rr * R)] : 0.f;
    }
    __syncthreads();
    for (int q = 0; q < 16; ++q) {
      const int e = threadIdx.x + q * blockDim.x;
      if (e >= RR) break;
      const int a = e / R, b = e - a * R;
      float s = 0.f;
      for (int rr = 0; rr < TR; ++rr) s = fmaf(tile[rr * R + a], tile[rr * R + b], s);
      acc[q] += (double)s;
    }
    __syncthreads();
  }
  for (int q = 0; q < 16; ++q) {
    const int e = threadIdx.x + q * blockDim.x;
    if (e >= RR) break;
    atomicAdd(&G[e], acc[q]);
  }
}

// Register-tiled Gram for R in {16, 32, 64}: the R x R output is cut into 4 x 4 blocks, one
// per thread of a "row group" of (R/4)^2 threads; the 256 / (R/4)^2 row groups of a CTA split
// each staged tile of TR rows.  Per row a thread does two LDS.128 and 16 FMAs (compute-bound,
// unlike the scalar kernel above); fp32 inside a tile, folded into fp64 per tile, row groups
// reduced in shared memory, one fp64 atomic per entry per CTA.
template <int R>
__global__ void __launch_bounds__(256) gram_rt_kernel(const float* __restrict__ A, uint64_t I,
                                                      double* __restrict__ G) {
  constexpr int TR = 4096 / R, NB = R / 4, TPG = NB * NB, NG = 256 / TPG;
  // two 16 KB tiles (the next one streams in with cp.async while this one is used), then
  // reused for the row-group partials (NG * 16 * TPG doubles <= 32 KB)
  __shared__ __align__(16) unsigned char sbuf[2 * TR * R * 4];
  static_assert(NG * 16 * TPG * 8 <= 2 * TR * R * 4, "partials must fit the tile buffers");
  float* const tiles = reinterpret_cast<float*>(sbuf);
  const int tid = threadIdx.x, g = tid / TPG, l = tid % TPG, bi = l / NB, bj = l % NB;
  double acc[16];
#pragma unroll
  for (int q = 0; q < 16; ++q) acc[q] = 0.0;
  const uint64_t ntiles = (I + TR - 1) / TR;
  auto prefetch = [&](uint64_t tb, int b) {  // rows past I are zero-filled
    if (tb < ntiles) {
      const uint64_t r0 = tb * TR;
      const int rows = (I - r0 < (uint64_t)TR) ? (int)(I - r0) : TR;
      const float4* src = reinterpret_cast<const float4*>(A + r0 * R);
      float* dst = tiles + b * TR * R;
      for (int e = tid; e < TR * R / 4; e += 256) {
        const bool ok = e < rows * R / 4;
        const uint32_t d = (uint32_t)__cvta_generic_to_shared(dst + 4 * e);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(d), "l"(ok ? src + e : src),
                     "r"(ok ? 16 : 0) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  int buf = 0;
  prefetch(blockIdx.x, 0);
  for (uint64_t tb = blockIdx.x; tb < ntiles; tb += gridDim.x, buf ^= 1) {
    __syncthreads();  // everyone is done with the other buffer
    prefetch(tb + gridDim.x, buf ^ 1);
    asm volatile("cp.async.wait_group 1;" ::: "memory");
    __syncthreads();
    const float* tile = tiles + buf * TR * R;
    float s[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) s[q] = 0.f;
    for (int rr = g; rr < TR; rr += NG) {
      const float4 a = *reinterpret_cast<const float4*>(tile + rr * R + 4 * bi);
      const float4 b = *reinterpret_cast<const float4*>(tile + rr * R + 4 * bj);
      const float av[4] = {a.x, a.y, a.z, a.w}, bv[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 4; ++y) s[x * 4 + y] = fmaf(av[x], bv[y], s[x * 4 + y]);
    }
#pragma unroll
    for (int q = 0; q < 16; ++q) acc[q] += (double)s[q];
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
  __syncthreads();
  double* red = reinterpret_cast<double*>(sbuf);
  if constexpr (NG > 1) {
#pragma unroll
    for (int q = 0; q < 16; ++q) red[(g * 16 + q) * TPG + l] = acc[q];
    __syncthreads();
  }
  if (g == 0) {
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      double v = acc[q];
      if constexpr (NG > 1)
        for (int h = 1; h < NG; ++h) v += red[(h * 16 + q) * TPG + l];
      const int x = q / 4, y = q % 4;
      atomicAdd(&G[(4 * bi + x) * R + 4 * bj + y], v);
    }
  }
}

// A = M x Vinv for R in {16, 32, 64}: one thread per row, its R outputs in registers, Vinv
// broadcast from shared memory (R / 4 LDS.128 per k for R FMAs).
template <int R>
__global__ void __launch_bounds__(256) rowmat_rt_kernel(const float* __restrict__ M, uint64_t I,
                                                        const float* __restrict__ Vinv, float* __restrict__ A) {
  __shared__ __align__(16) float V[R * R];
  for (int e = threadIdx.x; e < R * R; e += blockDim.x) V[e] = Vinv[e];
  __syncthreads();
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < I; i += stride) {
    const float4* m4 = reinterpret_cast<const float4*>(M + i * R);
    float acc[R];
#pragma unroll
    for (int r = 0; r < R; ++r) acc[r] = 0.f;
#pragma unroll 2
    for (int k4 = 0; k4 < R / 4; ++k4) {
      const float4 mv = __ldg(m4 + k4);
      const float mk[4] = {mv.x, mv.y, mv.z, mv.w};
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const float4* v4 = reinterpret_cast<const float4*>(V + (4 * k4 + kk) * R);
#pragma unroll
        for (int c = 0; c < R / 4; ++c) {
          const float4 v = v4[c];
          acc[4 * c] = fmaf(mk[kk], v.x, acc[4 * c]);
          acc[4 * c + 1] = fmaf(mk[kk], v.y, acc[4 * c + 1]);
          acc[4 * c + 2] = fmaf(mk[kk], v.z, acc[4 * c + 2]);
          acc[4 * c + 3] = fmaf(mk[kk], v.w, acc[4 * c + 3]);
        }
      }
    }
    float4* a4 = reinterpret_cast<float4*>(A + i * R);
#pragma unroll
    for (int c = 0; c < R / 4; ++c) a4[c] = make_float4(acc[4 * c], acc[4 * c + 1], acc[4 * c + 2], acc[4 * c + 3]);
  }
}

// Alg. 1 line 5 and the Gram refresh fused (R in {16, 32, 64}): per tile of TR = 4096 / R
// rows, M is read once into shared memory (cp.async, the next tile in flight while this one
// is computed: the synchronous load left every tile's DRAM latency exposed), A = M Vinv is formed in registers (4 rows x 4
// columns per thread, rows strided by NRB so a quarter-warp's LDS.128 hit distinct banks),
// written back through shared memory with coalesced stores, and G_n += A^T A (fp32 per
// tile, fp64 across tiles) plus, for the fit, <M, A> are taken from the same tile: M is
// read once and A written once (the separate kernels read A again for the Gram and M and A
// again for the fit).
template <int R>
__global__ void __launch_bounds__(256, 2) update_rt_kernel(const float* __restrict__ M, uint64_t I,
                                                           const float* __restrict__ Vinv, float* __restrict__ A,
                                                           double* __restrict__ G, double* __restrict__ dot) {
  constexpr int NCB = R / 4, NRB = 256 / NCB, TR = 4 * NRB, LD = R + 4;  // padded row stride
  // Gram: only the upper-triangular 4 x 4 blocks (G is symmetric), one per thread of a row
  // group; NG row groups split each tile's rows (threads past NG * TPG skip the Gram)
  constexpr int TPG = NCB * (NCB + 1) / 2, NG = 256 / TPG;
  extern __shared__ __align__(16) float sm[];
  float* Mbuf = sm;               // 2 x TR x LD: the M tile being used and the next one in flight
  float* As = Mbuf + 2 * TR * LD; // TR x LD
  float* Vs = As + TR * LD;       // R x R
  const int tid = threadIdx.x;
  for (int e = tid; e < R * R; e += 256) Vs[e] = Vinv[e];
  const int rs = tid % NRB, cb = tid / NRB;            // A-block: rows rs + NRB*x, cols 4cb..4cb+3
  const int g = tid / TPG, l = tid % TPG;  // Gram block (bi <= bj) number l of row group g
  int bi = 0, rem = l;
  while (rem >= NCB - bi) {
    rem -= NCB - bi;
    ++bi;
  }
  const int bj = bi + rem;
  double gacc[16];
#pragma unroll
  for (int q = 0; q < 16; ++q) gacc[q] = 0.0;
  double dacc = 0.0;
  const uint64_t ntiles = (I + TR - 1) / TR;
  // M tile tb -> buffer b with cp.async (16 B per copy, rows past I zero-filled): the next
  // tile's copies are in flight while this one is computed
  auto prefetch = [&](uint64_t tb, int b) {
    if (tb < ntiles) {
      const uint64_t r0 = tb * TR;
      const int rows = (I - r0 < (uint64_t)TR) ? (int)(I - r0) : TR;
      const float4* src = reinterpret_cast<const float4*>(M + r0 * R);
      float* dstb = Mbuf + b * TR * LD;
      for (int e = tid; e < TR * NCB; e += 256) {
        const int r = e / NCB, c = e % NCB;
        const uint32_t d = (uint32_t)__cvta_generic_to_shared(dstb + r * LD + 4 * c);
        const bool ok = r < rows;
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(d), "l"(ok ? src + e : src),
                     "r"(ok ? 16 : 0) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  int buf = 0;
  prefetch(blockIdx.x, 0);
  for (uint64_t tb = blockIdx.x; tb < ntiles; tb += gridDim.x, buf ^= 1) {
    const uint64_t r0 = tb * TR;
    const int rows = (I - r0 < (uint64_t)TR) ? (int)(I - r0) : TR;
    __syncthreads();  // the previous tile's reads of the other buffer and of As are done
    prefetch(tb + gridDim.x, buf ^ 1);
    asm volatile("cp.async.wait_group 1;" ::: "memory");
    __syncthreads();  // every thread's copies of this tile have landed
    const float* Ms = Mbuf + buf * TR * LD;
    float a[4][4];
#pragma unroll
    for (int x = 0; x < 4; ++x)
#pragma unroll
      for (int y = 0; y < 4; ++y) a[x][y] = 0.f;
#pragma unroll 2
    for (int k4 = 0; k4 < NCB; ++k4) {
      float4 m[4], v[4];
#pragma unroll
      for (int x = 0; x < 4; ++x) m[x] = *reinterpret_cast<const float4*>(Ms + (rs + NRB * x) * LD + 4 * k4);
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) v[kk] = *reinterpret_cast<const float4*>(Vs + (4 * k4 + kk) * R + 4 * cb);
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        const float mk[4] = {m[x].x, m[x].y, m[x].z, m[x].w};
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
          a[x][0] = fmaf(mk[kk], v[kk].x, a[x][0]);
          a[x][1] = fmaf(mk[kk], v[kk].y, a[x][1]);
          a[x][2] = fmaf(mk[kk], v[kk].z, a[x][2]);
          a[x][3] = fmaf(mk[kk], v[kk].w, a[x][3]);
        }
      }
    }
    float dpart = 0.f;
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      const int r = rs + NRB * x;
      *reinterpret_cast<float4*>(As + r * LD + 4 * cb) = make_float4(a[x][0], a[x][1], a[x][2], a[x][3]);
      if (dot) {
        const float4 mm = *reinterpret_cast<const float4*>(Ms + r * LD + 4 * cb);
        dpart = fmaf(mm.x, a[x][0], fmaf(mm.y, a[x][1], fmaf(mm.z, a[x][2], fmaf(mm.w, a[x][3], dpart))));
      }
    }
    dacc += (double)dpart;
    __syncthreads();
    float4* dst = reinterpret_cast<float4*>(A + r0 * R);
    for (int e = tid; e < rows * NCB; e += 256) {
      const int r = e / NCB, c = e % NCB;
      dst[e] = *reinterpret_cast<const float4*>(As + r * LD + 4 * c);
    }
    float s4[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) s4[q] = 0.f;
    for (int rr = g; g < NG && rr < rows; rr += NG) {
      const float4 x4 = *reinterpret_cast<const float4*>(As + rr * LD + 4 * bi);
      const float4 y4 = *reinterpret_cast<const float4*>(As + rr * LD + 4 * bj);
      const float av[4] = {x4.x, x4.y, x4.z, x4.w}, bv[4] = {y4.x, y4.y, y4.z, y4.w};
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 4; ++y) s4[x * 4 + y] = fmaf(av[x], bv[y], s4[x * 4 + y]);
    }
#pragma unroll
    for (int q = 0; q < 16; ++q) gacc[q] += (double)s4[q];
  }
  // reduce the NG row groups' Gram partials (shared memory reused) and the fit dot
  asm volatile("cp.async.wait_all;" ::: "memory");
  __syncthreads();
  double* red = reinterpret_cast<double*>(sm);
  static_assert((size_t)NG * 16 * TPG * 8 <= (size_t)3 * TR * LD * 4, "Gram partials must fit the tile buffers");
  if constexpr (NG > 1) {
    if (g < NG) {
#pragma unroll
      for (int q = 0; q < 16; ++q) red[(g * 16 + q) * TPG + l] = gacc[q];
    }
  }
  __syncthreads();
  if (g == 0) {
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      double v = gacc[q];
      if constexpr (NG > 1)
        for (int h = 1; h < NG; ++h) v += red[(h * 16 + q) * TPG + l];
      const int x = q / 4, y = q % 4;
      atomicAdd(&G[(4 * bi + x) * R + 4 * bj + y], v);
      if (bi != bj) atomicAdd(&G[(4 * bj + y) * R + 4 * bi + x], v);
    }
  }
  if (dot) {
    for (int o = 16; o > 0; o >>= 1) dacc += __shfl_xor_sync(0xffffffffu, dacc, o);
    if ((tid & 31) == 0) atomicAdd(dot, dacc);
  }
}

template <int R>
static size_t update_rt_smem() {
  constexpr int NCB = R / 4, NRB = 256 / NCB, TR = 4 * NRB, LD = R + 4;
  return (size_t)(3 * TR * LD + R * R) * sizeof(float);
}

// Vinv = (Hadamard_{m != n} G_m)^†, one CTA, fp64 Gauss-Jordan on [V | I].
__global__ void pinv_kernel(const double* __restrict__ G, int N, int n, int R, double* __restrict__ Vinv64,
                            float* __restrict__ Vinv32) {
  extern __shared__ double W[];  // R x 2R
  __shared__ int piv;
  __shared__ double dmax;
  const int C = 2 * R;
  for (int e = threadIdx.x; e < R * R; e += blockDim.x) {
    double v = 1.0;
    for (int m = 0; m < N; ++m)
      if (m != n) v *= G[(size_t)m * R * R + e];
    const int r = e / R, c = e - r * R;
    W[r * C + c] = v;
    W[r * C + R + c] = (r == c) ? 1.0 : 0.0;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double d = 0;
    for (int r = 0; r < R; ++r) d = fmax(d, fabs(W[r * C + r]));
    dmax = d;
  }
  __syncthreads();
  const double eps = 1e-12 * dmax;
  for (int c = 0; c < R; ++c) {
    if (threadIdx.x == 0) {
      int p = c;
      double best = fabs(W[c * C + c]);
      for (int r = c + 1; r < R; ++r)
        if (fabs(W[r * C + c]) > best) { best = fabs(W[r * C + c]); p = r; }
      piv = (best > eps) ? p : -1;
    }
    __syncthreads();
    const int p = piv;
    if (p < 0) {  // rank-deficient column: drop it from the inverse
      for (int e = threadIdx.x; e < C; e += blockDim.x) W[c * C + e] = 0.0;
      __syncthreads();
      continue;
    }
    if (p != c)
      for (int e = threadIdx.x; e < C; e += blockDim.x) {
        const double t = W[c * C + e];
        W[c * C + e] = W[p * C + e];
        W[p * C + e] = t;
      }
    __syncthreads();
    const double inv = 1.0 / W[c * C + c];
    __syncthreads();
    for (int e = threadIdx.x; e < C; e += blockDim.x) W[c * C + e] *= inv;
    __syncthreads();
    for (int e = threadIdx.x; e < R * C; e += blockDim.x) {
      const int r = e / C, k = e - r * C;
      if (r == c) continue;
      const double f = W[r * C + c];
      if (k != c) W[e] -= f * W[c * C + k];
    }
    __syncthreads();
    for (int r = threadIdx.x; r < R; r += blockDim.x)
      if (r != c) W[r * C + c] = 0.0;
    __syncthreads();
  }
  for (int e = threadIdx.x; e < R * R; e += blockDim.x) {
    const int r = e / R, k = e - r * R;
    const double v = W[r * C + R + k];
    Vinv64[e] = v;
    Vinv32[e] = (float)v;
  }
}

// A = M x Vinv (I x R times R x R), Vinv staged in shared memory; one thread per output.
__global__ void rowmat_kernel(const float* __restrict__ M, uint64_t I, int R, const float* __restrict__ Vinv,
                              float* __restrict__ A) {
  extern __shared__ float V[];
  for (int e = threadIdx.x; e < R * R; e += blockDim.x) V[e] = Vinv[e];
  __syncthreads();
  const uint64_t total = I * (uint64_t)R;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
    const uint64_t i = t / R;
    const int r = (int)(t - i * R);
    const float* m = M + i * R;
    float s = 0.f;
    for (int k = 0; k < R; ++k) s = fmaf(__ldg(m + k), V[k * R + r], s);
    A[t] = s;
  }
}

// out[0] += sum_e a[e] * b[e] (fp64), out[1] += sum_e a[e]^2 when b == nullptr
__global__ void dot_kernel(const float* __restrict__ a, const float* __restrict__ b, uint64_t n,
                           double* __restrict__ out) {
  double s = 0.0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += stride) {
    const double x = a[e];
    s += x * (b ? (double)b[e] : x);
  }
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  __shared__ double ws[32];
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += ws[w];
    atomicAdd(out, t);
  }
}

// out = sum_{r,s} prod_m G_m(r,s)
__global__ void model_norm_kernel(const double* __restrict__ G, int N, int R, double* __restrict__ out) {
  double s = 0;
  for (int e = threadIdx.x; e < R * R; e += blockDim.x) {
    double v = 1.0;
    for (int m = 0; m < N; ++m) v *= G[(size_t)m * R * R + e];
    s += v;
  }
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  __shared__ double ws[32];
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += ws[w];
    *out = t;
  }
}

static int grid_of(uint64_t n, int threads) {
  return (int)std::max<uint64_t>(1, std::min<uint64_t>((n + threads - 1) / threads, 148ull * 16));
}

static void gram(const float* A, uint64_t I, int R, double* G, cudaStream_t s) {
  SF_CUDA(cudaMemsetAsync(G, 0, sizeof(double) * R * R, s));
  const int rt_grid = (int)std::max<uint64_t>(1, std::min<uint64_t>((I + 4096 / R - 1) / (4096 / R), 148ull * 4));
  switch (R) {  // register-tiled kernels; the scalar one for other ranks
    case 16: gram_rt_kernel<16><<<rt_grid, 256, 0, s>>>(A, I, G); break;
    case 32: gram_rt_kernel<32><<<rt_grid, 256, 0, s>>>(A, I, G); break;
    case 64: gram_rt_kernel<64><<<rt_grid, 256, 0, s>>>(A, I, G); break;
    default: {
      const uint64_t tiles = (I + 63) / 64;
      gram_kernel<<<grid_of(tiles, 1), 256, 64 * R * sizeof(float), s>>>(A, I, R, G);
    }
  }
  count_launch();
  SF_CUDA(cudaGetLastError());
}

// A = M Vinv, G = A^T A, and (dot != nullptr) *dot += <M, A>; false: rank not specialised.
template <int R>
static void update_one(const float* M, uint64_t I, const float* Vinv, float* A, double* G, double* dot,
                       cudaStream_t s) {
  const size_t smem = update_rt_smem<R>();
  SF_CUDA(cudaFuncSetAttribute(update_rt_kernel<R>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  constexpr uint64_t TR = 4096 / R;
  const int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>((I + TR - 1) / TR, 148ull * 2));
  update_rt_kernel<R><<<grid, 256, smem, s>>>(M, I, Vinv, A, G, dot);
}

static bool update_fused(const float* M, uint64_t I, int R, const float* Vinv, float* A, double* G, double* dot,
                         cudaStream_t s) {
  if (debug_opt("no_cpals_fused")) return false;  // SF_DEBUG A/B: separate kernels
  SF_CUDA(cudaMemsetAsync(G, 0, sizeof(double) * R * R, s));
  switch (R) {
    case 16: update_one<16>(M, I, Vinv, A, G, dot, s); break;
    case 32: update_one<32>(M, I, Vinv, A, G, dot, s); break;
    case 64: update_one<64>(M, I, Vinv, A, G, dot, s); break;
    default: return false;
  }
  count_launch();
  SF_CUDA(cudaGetLastError());
  return true;
}

static void rowmat(const float* M, uint64_t I, int R, const float* Vinv, float* A, cudaStream_t s) {
  const int g = (int)std::max<uint64_t>(1, std::min<uint64_t>((I + 255) / 256, 148ull * 8));
  switch (R) {
    case 16: rowmat_rt_kernel<16><<<g, 256, 0, s>>>(M, I, Vinv, A); break;
    case 32: rowmat_rt_kernel<32><<<g, 256, 0, s>>>(M, I, Vinv, A); break;
    case 64: rowmat_rt_kernel<64><<<g, 256, 0, s>>>(M, I, Vinv, A); break;
    default:
      rowmat_kernel<<<grid_of(I * (uint64_t)R, 256), 256, (size_t)R * R * sizeof(float), s>>>(M, I, R, Vinv, A);
  }
  count_launch();
  SF_CUDA(cudaGetLastError());
}

// out[e] = sum_k parts[k][e] in rank order (identical on every rank)
__global__ void sum_parts_kernel(const double* __restrict__ parts, int P, int n, double* __restrict__ out) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < n; e += gridDim.x * blockDim.x) {
    double acc = 0.0;
    for (int k = 0; k < P; ++k) acc += parts[(size_t)k * n + e];
    out[e] = acc;
  }
}

// Rows of Y assigned to each rank of a sharded plan for the row-local update A_n = M V^+:
// rank k owns [row_begin_k + send_first_k, row_end_k) (sf_comm.cu exchange rule); the
// assignment extends each owned block over the empty rows up to the next owned block, so
// the blocks partition [0, I_n) (blk[2k], blk[2k+1]).
static std::vector<uint64_t> assigned_blocks(const Plan& p, int P, uint64_t I) {
  std::vector<int32_t> sendf(P), owner(P);
  sf_exchange_map(P, p.ranges.data(), sendf.data(), owner.data());
  std::vector<uint64_t> ob(P), nonempty(P);
  for (int k = 0; k < P; ++k) {
    const uint64_t b = p.ranges[2 * k], e = p.ranges[2 * k + 1];
    ob[k] = b + (uint64_t)sendf[k];
    nonempty[k] = e > ob[k];
  }
  std::vector<uint64_t> blk(2 * P);
  uint64_t next = I;  // begin of the next non-empty owned block, scanning from the right
  for (int k = P - 1; k >= 0; --k) {
    if (nonempty[k]) next = ob[k];
    blk[2 * k] = (k == 0) ? 0 : next;
  }
  for (int k = 0; k < P; ++k) blk[2 * k + 1] = (k + 1 < P) ? blk[2 * (k + 1)] : I;
  return blk;
}

void cpals(Tensor& t, int R, float* const* factors, int iters, double tol, double* fits, int* done,
           cudaStream_t s, Plan* const* plans) {
  const int N = t.nmodes;
  if (R > 64) throw StatusError{SF_ERR_UNSUPPORTED, "sf_cpals: rank must be <= 64"};
  const bool sharded = t.nranks > 1;
  if (sharded && !t.comm) throw StatusError{SF_ERR_INVALID_ARG, "sf_cpals: a sharded handle needs a comm"};
  const int P = t.nranks;
  uint64_t maxI = 0;
  for (int m = 0; m < N; ++m) maxI = std::max<uint64_t>(maxI, t.dims[m]);
  DevBuf M(maxI * R * sizeof(float)), G((size_t)N * R * R * sizeof(double)), Vinv64(R * R * sizeof(double)),
      Vinv32(R * R * sizeof(float)), scal(4 * sizeof(double)),
      parts(sharded ? (size_t)P * R * R * sizeof(double) + 64 : 16);
  double* dG = G.as<double>();
  for (int m = 0; m < N; ++m) gram(factors[m], t.dims[m], R, dG + (size_t)m * R * R, s);
  // ||X||^2 (whole tensor: every rank holds the full raw COO; distributed handles sum slices)
  SF_CUDA(cudaMemsetAsync(scal.p, 0, 4 * sizeof(double), s));
  dot_kernel<<<grid_of(t.nnz, 256), 256, 0, s>>>(t.val.as<float>(), nullptr, t.nnz, scal.as<double>());
  count_launch();
  double normX2 = 0;
  if (sharded && t.dist) {  // a distributed handle holds only its slice of the values
    std::vector<uint64_t> bytes(P, 8), displs(P);
    for (int k = 0; k < P; ++k) displs[k] = (uint64_t)k * 8;
    t.comm->allgatherv(scal.p, parts.p, bytes.data(), displs.data(), s);
    sum_parts_kernel<<<1, 32, 0, s>>>(parts.as<double>(), P, 1, scal.as<double>());
    count_launch();
  }
  d2h_small(s, &normX2, scal.p, sizeof(double));
  const float* const* cf = const_cast<const float* const*>(factors);
  // [V | I] in fp64: 64 KB at R = 64, above the 48 KB default dynamic shared-memory limit
  const size_t pinv_smem = (size_t)R * 2 * R * sizeof(double);
  SF_CUDA(cudaFuncSetAttribute(pinv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pinv_smem));
  // sharded: per mode, the rows this rank updates (Alg. 1 line 5 is row-local)
  std::vector<std::vector<uint64_t>> blk(N);
  if (sharded)
    for (int n = 0; n < N; ++n) {
      ensure_ranges(t, *plans[n], s);
      blk[n] = assigned_blocks(*plans[n], P, t.dims[n]);
    }
  // sum a per-rank partial (count doubles at dst) over the ranks, in rank order
  auto allreduce_parts = [&](double* dst, int count) {
    std::vector<uint64_t> bytes(P, (uint64_t)count * 8), displs(P);
    for (int k = 0; k < P; ++k) displs[k] = (uint64_t)k * count * 8;
    t.comm->allgatherv(dst, parts.p, bytes.data(), displs.data(), s);
    sum_parts_kernel<<<grid_of((uint64_t)count, 256), 256, 0, s>>>(parts.as<double>(), P, count, dst);
    count_launch();
  };
  double prev = -1.0;
  int k = 0;
  for (; k < iters; ++k) {
    for (int n = 0; n < N; ++n) {
      pinv_kernel<<<1, 256, pinv_smem, s>>>(dG, N, n, R, Vinv64.as<double>(), Vinv32.as<float>());
      count_launch();
      SF_CUDA(cudaGetLastError());
      const Plan& p = *plans[n];
      // M holds Y rows [a0, a1) for the update (all of Y unsharded); the plan's out block
      // [out_row0, out_row0 + out_rows) lies inside [a0 - 1, a1) (a shared first row is sent
      // to its owner and zeroed by the exchange)
      uint64_t a0 = 0, a1 = t.dims[n];
      if (sharded) {
        a0 = blk[n][2 * t.rank];
        a1 = blk[n][2 * t.rank + 1];
        SF_CUDA(cudaMemsetAsync(M.as<float>() + a0 * R, 0, (a1 - a0) * R * sizeof(float), s));
      }
      float* Mblk = M.as<float>() + p.out_row0 * R;
      launch_mttkrp(t, p, cf, Mblk, s);
      exchange_rows(t, *plans[n], Mblk, s);
      const uint64_t I = a1 - a0;
      const float* Mown = M.as<float>() + a0 * R;
      float* Aown = factors[n] + a0 * R;
      // fit after the sweep needs <M_N, A_N> of the last mode
      double* dot = (n == N - 1) ? scal.as<double>() + 1 : nullptr;
      if (n == N - 1) SF_CUDA(cudaMemsetAsync(scal.as<double>() + 1, 0, 2 * sizeof(double), s));
      double* Gn = dG + (size_t)n * R * R;
      if (!update_fused(Mown, I, R, Vinv32.as<float>(), Aown, Gn, dot, s)) {
        rowmat(Mown, I, R, Vinv32.as<float>(), Aown, s);
        gram(Aown, I, R, Gn, s);
        if (dot) {
          const uint64_t nl = I * (uint64_t)R;
          dot_kernel<<<grid_of(nl, 256), 256, 0, s>>>(Mown, Aown, nl, dot);
          count_launch();
        }
      }
      SF_CUDA(cudaGetLastError());
      if (sharded) {  // every rank ends with the full A_n, G_n and <M_N, A_N>
        allgather_blocks(t, blk[n], Aown, factors[n], R, s);
        allreduce_parts(Gn, R * R);
        if (dot) allreduce_parts(dot, 1);
      }
    }
    model_norm_kernel<<<1, 256, 0, s>>>(dG, N, R, scal.as<double>() + 2);
    count_launch();
    double h[3];
    d2h_small(s, h, scal.p, 3 * sizeof(double));
    const double res2 = std::max(normX2 + h[2] - 2.0 * h[1], 0.0);
    const double fit = normX2 > 0 ? 1.0 - std::sqrt(res2) / std::sqrt(normX2) : 0.0;
    if (fits) fits[k] = fit;
    if (tol > 0 && prev >= 0 && std::fabs(fit - prev) < tol) {
      ++k;
      break;
    }
    prev = fit;
  }
  if (done) *done = k;
}

}  // namespace sf
