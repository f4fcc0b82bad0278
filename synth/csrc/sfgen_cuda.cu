// sfgen_cuda.cu - device twin of sfgen.c over the same sfgen_core.h (bit-identical draws).
// Holds none of the method's arithmetic; used by tests / bench / selector training to
// create large synthetic tensors directly in HBM.
#include <cuda_runtime.h>

#include "sfgen_core.h"

namespace {

struct ModeTab {
  const uint64_t* edges;
  const uint64_t* thr;
  int nb;
};

__global__ void gen_kernel(int nmodes, const uint64_t* __restrict__ dims, uint64_t seed, uint64_t lo, uint64_t n,
                           const uint64_t* __restrict__ edges, const uint64_t* __restrict__ thr,
                           const int* __restrict__ nb, const int* __restrict__ eoff, const int* __restrict__ toff,
                           int relabel, int val_kind, uint32_t* const* __restrict__ inds, float* __restrict__ vals) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += stride) {
    const uint64_t e = lo + k;
    for (int m = 0; m < nmodes; ++m) {
      if (!inds[m]) continue;
      const uint64_t I = dims[m];
      const int half = sfg_feistel_half(I);
      const uint64_t key = sfg_fmix64(seed ^ (SFG_KEY_SALT * (uint64_t)(m + 1)));
      inds[m][k] = (uint32_t)sfg_index(seed, m, e, I, nb[m], edges + eoff[m], thr + toff[m], relabel, half, key);
    }
    if (vals) vals[k] = sfg_value(sfg_hash(seed, SFG_STREAM_VALUE, e), val_kind);
  }
}

__global__ void factor_kernel(uint64_t seed, uint64_t stream, uint64_t n, int kind, float* __restrict__ out) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n; t += stride)
    out[t] = sfg_factor(sfg_hash(seed, stream, t), kind);
}

}  // namespace

extern "C" {

// All pointers are device pointers; edges/thr are the concatenated per-mode tables with
// offsets eoff/toff (device int arrays), nb per mode (device).  inds: device array of nmodes
// device pointers.  Returns a cudaError_t code.
int sfgen_coo_device(int nmodes, const uint64_t* dims, uint64_t seed, uint64_t lo, uint64_t hi,
                     const uint64_t* edges, const uint64_t* thr, const int* nb, const int* eoff, const int* toff,
                     int relabel, int val_kind, uint32_t* const* inds, float* vals, void* stream) {
  const uint64_t n = hi - lo;
  if (n == 0) return 0;
  int blocks = (int)((n + 255) / 256);
  if (blocks > 148 * 32) blocks = 148 * 32;
  gen_kernel<<<blocks, 256, 0, (cudaStream_t)stream>>>(nmodes, dims, seed, lo, n, edges, thr, nb, eoff, toff,
                                                        relabel, val_kind, inds, vals);
  return (int)cudaGetLastError();
}

int sfgen_factor_device(uint64_t seed, uint64_t stream_id, uint64_t rows, int rank, int kind, float* out,
                        void* stream) {
  const uint64_t n = rows * (uint64_t)rank;
  if (n == 0) return 0;
  int blocks = (int)((n + 255) / 256);
  if (blocks > 148 * 32) blocks = 148 * 32;
  factor_kernel<<<blocks, 256, 0, (cudaStream_t)stream>>>(seed, stream_id, n, kind, out);
  return (int)cudaGetLastError();
}

}  // extern "C"
