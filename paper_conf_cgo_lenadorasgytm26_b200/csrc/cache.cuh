// cache.cuh -- L2 residency control for the gather kernels: per-access L2
// eviction priorities through `createpolicy` cache-policy operands.
//   keep   : the gathered operand (a K slice of X, er / dinv, Θ rows): L2::evict_last, so the
//            streamed arrays cannot push it out of L2 while it is being re-read;
//   stream : data read or written exactly once per launch (col_idx, edge values, output rows):
//            L2::evict_first (+ L1::no_allocate), so it leaves L2 first.
// `on == 0` gives L2::evict_normal for both (the default allocation policy), for A/B runs
// (GRANII_L2HINT=0).  The policy is a 64-bit operand held in a uniform register (SASS: the
// desc[UR] of the LDG / STG), so `on` must be warp-uniform -- it is a kernel argument.
#pragma once
#include <cstdint>

namespace granii {

struct L2Pol {
  uint64_t keep, stream;
};

__device__ __forceinline__ L2Pol make_l2pol(int on) {
  L2Pol p;
  if (on) {
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p.keep));
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p.stream));
  } else {
    asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p.keep));
    p.stream = p.keep;
  }
  return p;
}

// read-only gathers (non-coherent path, as __ldg), with an L2 policy
__device__ __forceinline__ float4 ldg_pol(const float4* p, uint64_t pol) {
  float4 v;
  asm("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
      : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
      : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float ldg_pol(const float* p, uint64_t pol) {
  float v;
  asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}
// streamed once: no L1 allocation either
__device__ __forceinline__ int32_t ldg_stream(const int32_t* p, uint64_t pol) {
  int32_t v;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ int4 ldg_stream(const int4* p, uint64_t pol) {
  int4 v;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
      : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
      : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float ldg_stream(const float* p, uint64_t pol) {
  float v;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void st_pol(float4* p, float4 v, uint64_t pol) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.f32 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p), "f"(v.x),
               "f"(v.y), "f"(v.z), "f"(v.w), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void st_pol(float* p, float v, uint64_t pol) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(p), "f"(v), "l"(pol) : "memory");
}

// GRANII_L2HINT (default on): host-side switch for the A/B measurement
int l2hint_enabled();

}  // namespace granii
