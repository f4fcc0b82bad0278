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
  const uint64_t tiles = (I + 63) / 64;
  gram_kernel<<<grid_of(tiles, 1), 256, 64 * R * sizeof(float), s>>>(A, I, R, G);
  count_launch();
  SF_CUDA(cudaGetLastError());
}

void cpals(Tensor& t, int R, float* const* factors, int iters, double tol, double* fits, int* done,
           cudaStream_t s, Plan* const* plans) {
  const int N = t.nmodes;
  if (R > 64) throw StatusError{SF_ERR_UNSUPPORTED, "sf_cpals: rank must be <= 64"};
  uint64_t maxI = 0;
  for (int m = 0; m < N; ++m) maxI = std::max<uint64_t>(maxI, t.dims[m]);
  DevBuf M(maxI * R * sizeof(float)), G((size_t)N * R * R * sizeof(double)), Vinv64(R * R * sizeof(double)),
      Vinv32(R * R * sizeof(float)), scal(4 * sizeof(double));
  double* dG = G.as<double>();
  for (int m = 0; m < N; ++m) gram(factors[m], t.dims[m], R, dG + (size_t)m * R * R, s);
  // ||X||^2 (whole tensor; this handle holds the full COO)
  SF_CUDA(cudaMemsetAsync(scal.p, 0, 4 * sizeof(double), s));
  dot_kernel<<<grid_of(t.nnz, 256), 256, 0, s>>>(t.val.as<float>(), nullptr, t.nnz, scal.as<double>());
  count_launch();
  double normX2 = 0;
  SF_CUDA(cudaMemcpyAsync(&normX2, scal.p, sizeof(double), cudaMemcpyDeviceToHost, s));
  SF_CUDA(cudaStreamSynchronize(s));
  const float* const* cf = const_cast<const float* const*>(factors);
  double prev = -1.0;
  int k = 0;
  for (; k < iters; ++k) {
    for (int n = 0; n < N; ++n) {
      pinv_kernel<<<1, 256, (size_t)R * 2 * R * sizeof(double), s>>>(dG, N, n, R, Vinv64.as<double>(),
                                                                    Vinv32.as<float>());
      count_launch();
      launch_mttkrp(t, *plans[n], cf, M.as<float>(), s);
      rowmat_kernel<<<grid_of(t.dims[n] * (uint64_t)R, 256), 256, (size_t)R * R * sizeof(float), s>>>(
          M.as<float>(), t.dims[n], R, Vinv32.as<float>(), factors[n]);
      count_launch();
      gram(factors[n], t.dims[n], R, dG + (size_t)n * R * R, s);
      SF_CUDA(cudaGetLastError());
    }
    // fit after the sweep: M holds the last mode's MTTKRP, factors[N-1] its update
    SF_CUDA(cudaMemsetAsync(scal.as<double>() + 1, 0, 2 * sizeof(double), s));
    const uint64_t nl = t.dims[N - 1] * (uint64_t)R;
    dot_kernel<<<grid_of(nl, 256), 256, 0, s>>>(M.as<float>(), factors[N - 1], nl, scal.as<double>() + 1);
    model_norm_kernel<<<1, 256, 0, s>>>(dG, N, R, scal.as<double>() + 2);
    count_launch(2);
    double h[3];
    SF_CUDA(cudaMemcpyAsync(h, scal.p, 3 * sizeof(double), cudaMemcpyDeviceToHost, s));
    SF_CUDA(cudaStreamSynchronize(s));
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
