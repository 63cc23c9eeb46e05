// np_le_acc.cuh -- one LE slave's accumulation order for item-major rows,
// shared by the register / global placements (np_le.cu, LeSlaveV) and the
// shared-memory placement (np_le_tma.cu), so all three stay bit-identical.
//
// A slave's elements come as head scalars (up to the row's 16-byte boundary),
// 128-bit body units and tail scalars.  Loops 2 and 3 of Fig 5/6d (P:232-247,
// P:299-324) accumulate head and tail in scalars and the body in a pair of
// lanes (x,y) / (z,w) with sm_100's packed fp32 instructions (FADD2 / FFMA2,
// __fadd2_rn / __ffma2_rn): half the issue slots for the body's arithmetic,
// which ncu found the LE kernel bound by.  The results are the paper's sums
// reassociated (reading R12): fp32 within tolerance of the oracle.
#pragma once
#include <cuda_runtime.h>

#include "np_team.cuh"

namespace cudanp {

// Loop 2: sum of the slave's elements.
struct LeSum {
  float hs = 0.f, ts = 0.f;
  float2 b = make_float2(0.f, 0.f);
  __device__ __forceinline__ void head(float v) { hs += v; }
  __device__ __forceinline__ void tail(float v) { ts += v; }
  __device__ __forceinline__ void body(V4<float> v) {
    b = __fadd2_rn(b, make_float2(v.x, v.y));
    b = __fadd2_rn(b, make_float2(v.z, v.w));
  }
  __device__ __forceinline__ float result() const { return (hs + (b.x + b.y)) + ts; }
};

// Loop 3: t = Grad - ave; var += t*t; ep += t.
struct LeVarEp {
  float hv = 0.f, he = 0.f, tv = 0.f, te = 0.f;
  float2 v2 = make_float2(0.f, 0.f), e2 = make_float2(0.f, 0.f), na;
  __device__ __forceinline__ explicit LeVarEp(float ave) : na(make_float2(-ave, -ave)) {}
  __device__ __forceinline__ void head(float g) {
    const float t = g + na.x;
    hv = fmaf(t, t, hv);
    he += t;
  }
  __device__ __forceinline__ void tail(float g) {
    const float t = g + na.x;
    tv = fmaf(t, t, tv);
    te += t;
  }
  __device__ __forceinline__ void body(V4<float> g) {
    const float2 t0 = __fadd2_rn(make_float2(g.x, g.y), na);
    const float2 t1 = __fadd2_rn(make_float2(g.z, g.w), na);
    v2 = __ffma2_rn(t0, t0, v2);
    e2 = __fadd2_rn(e2, t0);
    v2 = __ffma2_rn(t1, t1, v2);
    e2 = __fadd2_rn(e2, t1);
  }
  __device__ __forceinline__ float var() const { return (hv + (v2.x + v2.y)) + tv; }
  __device__ __forceinline__ float ep() const { return (he + (e2.x + e2.y)) + te; }
};

}  // namespace cudanp
