// agent_update.cuh -- steering (Listings 5.1, 5.3-5.5) and the modification
// substage (Q10-Q13) for ONE agent, given
// its neighbour list.  Shared by the standalone update kernel and the fused
// epilogue.  Appendix A arithmetic (device_math.cuh).
#pragma once
#include "device_math.cuh"
#include "internal.h"

namespace boids {

// Diagnostics (BOIDS_OPT_PHASES): the span of a whole launch in slot `slot` of
// the phase buffer -- [0] = ~(earliest CTA start), [1] = latest CTA end
// (%globaltimer, ns), both by atomicMax so the buffer's zero fill is neutral.
constexpr int SPAN_SLOT0 = 1000;
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void span_begin(const StepArgs& a, int slot) {
  if (a.phase && threadIdx.x == 0) atomicMax(a.phase + slot * 8, ~gtimer());
}
__device__ __forceinline__ void span_end(const StepArgs& a, int slot) {  // every thread of the CTA
  if (a.phase) {
    __syncthreads();
    if (threadIdx.x == 0) atomicMax(a.phase + slot * 8 + 1, gtimer());
  }
}

__device__ __forceinline__ void prefetch_l1(const void* p) {
  asm volatile("prefetch.global.L1 [%0];" ::"l"(p));
}

// Steering vector of agent g from its <=7 neighbours (in key order, Q8).  The
// neighbours' lines are prefetched into L1 up front and the loop is kept
// rolled: this code runs once per agent per step, so at small n its
// instruction-fetch latency, not its arithmetic, is what the warps wait on.
__device__ __forceinline__ V3 steer_agent(const StepArgs& a, V3 me, V3 fme, const int* nb,
                                          int cnt) {
#pragma unroll
  for (int k = 0; k < 7; ++k)
    if (k < cnt) {
      prefetch_l1(pos_of(a.full, a.m, a.sdiv, nb[k]));
      prefetch_l1(fwd_of(a.full, a.m, a.sdiv, nb[k]));
    }
  int q0 = nb[0], q1 = nb[1], q2 = nb[2], q3 = nb[3], q4 = nb[4], q5 = nb[5], q6 = nb[6];
  V3 sep = v3(0.f, 0.f, 0.f), coh = v3(0.f, 0.f, 0.f), ali = v3(0.f, 0.f, 0.f);
#pragma unroll 1
  for (int k = 0; k < cnt; ++k) {
    const int64_t j = q0;  // nb[k]: the list shifts down one slot per iteration
    q0 = q1; q1 = q2; q2 = q3; q3 = q4; q4 = q5; q5 = q6;
    float4 pj = __ldg(pos_of(a.full, a.m, a.sdiv, j));
    float4 fj = __ldg(fwd_of(a.full, a.m, a.sdiv, j));
    V3 o = sub(v3(pj), me);  // A.position - me.position (Listing 5.3 line 7)
    float L = len(o);
    if (L > 0.0f) sep = sub(sep, divs(divs(o, L), L));  // 1/d fall-off (Listing 5.3 line 10)
    coh = add(coh, o);                                  // Listing 5.4 line 8
    ali = add(ali, v3(fj));                             // Listing 5.5 line 7
  }
  ali = sub(ali, scale(fme, (float)cnt));  // Listing 5.5 line 10
  V3 sw = scale(normalize(sep), a.p.w_separation);
  V3 aw = scale(normalize(ali), a.p.w_alignment);
  V3 cw = scale(normalize(coh), a.p.w_cohesion);
  return add(add(sw, aw), cw);  // Listing 5.1 line 5
}

// Modification substage for local agent i (global g = lo + i); writes the new state.
__device__ __forceinline__ void modify_agent(const StepArgs& a, int64_t i, V3 pos, float4 f4, V3 F) {
  const boids_params& p = a.p;
  V3 f = v3(f4);
  float speed = f4.w;
  float4 u4 = a.up4[i];
  float4 s4 = a.side4[i];
  V3 u = v3(u4), s = v3(s4);
  V3 Fc = trunc_len(F, p.max_force);
  V3 acc = divs(Fc, p.mass);
  V3 v = scale(f, speed);
  V3 v1 = add(v, scale(acc, a.dt));
  V3 v2 = trunc_len(v1, p.max_speed);
  float sp = len(v2);
  V3 p1 = add(pos, scale(v2, a.dt));
  if (sp > 0.0f) {
    f = divs(v2, sp);
    s = normalize(cross(f, u));
    u = cross(s, f);
  }
  float L = len(p1);
  if (L > p.world_radius) p1 = add(p1, scale(scale(divs(p1, L), p.world_radius), -2.0f));
  a.out[i] = make_float4(p1.x, p1.y, p1.z, 0.0f);
  a.out[a.m + i] = make_float4(f.x, f.y, f.z, sp);
  a.up4[i] = make_float4(u.x, u.y, u.z, 0.0f);
  a.side4[i] = make_float4(s.x, s.y, s.z, 0.0f);
  if (a.force4) a.force4[i] = make_float4(F.x, F.y, F.z, 0.0f);
}

}  // namespace boids
