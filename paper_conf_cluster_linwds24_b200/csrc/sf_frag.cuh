// sf_frag.cuh - device helpers shared by the fragment MTTKRP kernel (sf_frag3.cuh):
// PTX wrappers (256-bit global loads/stores, vector reductions, mbarrier, 1-D TMA bulk
// copies), the lane map (which rank slice each lane owns) and the (N, S) instantiation
// switch.  The round-1 SoA chunk-stretch kernel that lived here was replaced by
// frag3_kernel (measured 0.98 -> 0.74 ms per mode on nell-2, profiles/r01_frag3/).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "sf_internal.h"

namespace sf {

constexpr int kFragStages = 2;  // double-buffered record stages (sf_select.cpp kStagesHost)
constexpr int kFragUnroll = 4;

namespace detail {

__device__ __forceinline__ void st256(float* p, const float4& a, const float4& b) {
  asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "f"(a.x), "f"(a.y), "f"(a.z),
               "f"(a.w), "f"(b.x), "f"(b.y), "f"(b.z), "f"(b.w));
}
__device__ __forceinline__ void st128(float* p, const float4& a) {
  asm volatile("st.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(a.x), "f"(a.y), "f"(a.z), "f"(a.w));
}

__device__ __forceinline__ void red_add_v4_nomem(float* addr, const float4& v) {
  asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(addr), "f"(v.x), "f"(v.y), "f"(v.z),
               "f"(v.w));
}

__device__ __forceinline__ uint32_t su32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// 128-bit gathers (R = 16) allocate in L1: bypassing it made amazon 1.4-1.7x slower
// (session 3) -- its hot 64-byte rows hit there
__device__ __forceinline__ float4 ldg128(const float4* p) { return __ldg(p); }

__device__ __forceinline__ void ldg256_na(const float4* p, float4& a, float4& b) {
  asm("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w), "=f"(b.x), "=f"(b.y), "=f"(b.z), "=f"(b.w)
      : "l"(p));
}
// L1-allocating 256-bit gather: the hot-row plans' gathers (session 3 A/B: deli-4d +2.3 %,
// nell-1 unchanged; on the L2-resident nell-2 plans allocation cost 1.5 %, so those keep
// ldg256_na)
__device__ __forceinline__ void ldg256_l1(const float4* p, float4& a, float4& b) {
  asm("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w), "=f"(b.x), "=f"(b.y), "=f"(b.z), "=f"(b.w)
      : "l"(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(dst)),
      "l"(src), "r"(bytes), "r"(su32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  const uint32_t a = su32(bar);
  do {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  } while (!done);
}

}  // namespace detail

// Lane mapping.  VEC = floats per lane (4 for R <= 16, else 8), LPN = R / VEC lanes per
// nonzero.  VEC = 8: lane t owns the 32 contiguous bytes of 16-byte chunks 2t, 2t+1 of a
// factor row: a global gather is ONE 256-bit load (ld.global.nc.v8.f32, sm_100), and a
// shared-memory gather is two 128-bit loads issued in parity order (quarter-warp
// half p = (lane>>2)&1 reads chunk 2t+p first), so the 8 lanes of a quarter-warp touch
// all 32 banks exactly once per load; the pair is swapped back into (2t, 2t+1).
// VEC = 4: lane t owns chunk t.
template <int R>
struct LaneMap {
  static constexpr int VEC = (R >= 32) ? 8 : 4;  // R = 16 with VEC = 8: 15-30 % slower (profiles/r01_frag3)
  static constexpr int LPN = R / VEC;
};

struct F8 {
  float4 a, b;
};

__device__ __forceinline__ void f4mul_(float4& x, const float4& y) {
  x.x *= y.x; x.y *= y.y; x.z *= y.z; x.w *= y.w;
}
__device__ __forceinline__ void f4fma_(float4& acc, const float4& x, const float4& y) {
  acc.x = fmaf(x.x, y.x, acc.x);
  acc.y = fmaf(x.y, y.y, acc.y);
  acc.z = fmaf(x.z, y.z, acc.z);
  acc.w = fmaf(x.w, y.w, acc.w);
}

// (N, S) -> instantiation, for one R.
#define SF_FRAG_NS_SWITCH(R, FN, ...)                  \
  switch (N * 10 + S) {                                \
    case 20: return FN<2, R, 0>(__VA_ARGS__);          \
    case 21: return FN<2, R, 1>(__VA_ARGS__);          \
    case 30: return FN<3, R, 0>(__VA_ARGS__);          \
    case 31: return FN<3, R, 1>(__VA_ARGS__);          \
    case 32: return FN<3, R, 2>(__VA_ARGS__);          \
    case 40: return FN<4, R, 0>(__VA_ARGS__);          \
    case 41: return FN<4, R, 1>(__VA_ARGS__);          \
    case 42: return FN<4, R, 2>(__VA_ARGS__);          \
    case 43: return FN<4, R, 3>(__VA_ARGS__);          \
    case 50: return FN<5, R, 0>(__VA_ARGS__);          \
    case 51: return FN<5, R, 1>(__VA_ARGS__);          \
    case 52: return FN<5, R, 2>(__VA_ARGS__);          \
    case 53: return FN<5, R, 3>(__VA_ARGS__);          \
    case 54: return FN<5, R, 4>(__VA_ARGS__);          \
    default: break;                                    \
  }

}  // namespace sf
