// step_common.cuh -- per-query pieces shared by the warm-step kernels (k_warm.cu,
// k_grid.cu): the warm search bound, the shared-memory top-7 insert, and the
// per-agent finish (neighbour list, steering, modification).
#pragma once
#include "agent_update.cuh"

namespace boids {

// t0 of local query qi: an upper bound on its 7th smallest d2 this step, from
// agents that exist -- the previous step's 7 neighbours and, when known, the
// 8th nearest: t0 = 7th smallest of their d2 at the CURRENT positions, i.e. the
// max of the 7 or the second largest of the 8 (one neighbour that wrapped to
// the far side of the world then does not spoil the bound).  Valid for any
// positions (the agents are real and distinct); +inf without 7 previous
// neighbours.  All loads are issued before any is used.
__device__ __forceinline__ float warm_bound(const StepArgs& a, int64_t qi, float4 me) {
  if (qi >= a.nloc) return __int_as_float(0x7f800000);
  int nb[8];
#pragma unroll
  for (int k = 0; k < 7; ++k) nb[k] = __ldg(a.nbr + qi * 7 + k);
  nb[7] = a.nbr8 ? __ldg(a.nbr8 + qi) : -1;
  const int c = __ldg(a.cnt + qi);
  float4 p[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) p[k] = __ldg(pos_of(a.full, a.m, a.sdiv, nb[k] < 0 ? 0 : nb[k]));
  float m1 = 0.f, m2 = 0.f;  // largest and second largest
  bool absent = false;        // a previous neighbour whose position this handle does not hold
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const float d = (k < 7 || nb[7] >= 0) ? dist2(me.x, me.y, me.z, p[k]) : 0.f;  // no 8th: ignore
    absent |= !(d == d);
    m2 = fmaxf(m2, fminf(m1, d));
    m1 = fmaxf(m1, d);
  }
  // a spatial shard holds only its own agents and its halo (NaN elsewhere): a
  // bound over fewer than the 7-8 real agents would not be one
  if (c < 7 || absent) return __int_as_float(0x7f800000);
  return nb[7] >= 0 ? m2 : m1;
}

// Insert key k into a sorted 7-list in shared memory (stride between entries);
// returns the new worst d2 (+inf while fewer than 7 are held).  Out of line: it
// runs rarely and one copy keeps the hot loops small in the instruction cache.
static __device__ __noinline__ float insert_smem7(key_t* L7, int stride, key_t k) {
  key_t L[7];
#pragma unroll
  for (int s = 0; s < 7; ++s) L[s] = L7[s * stride];
  insert7(L, k);
#pragma unroll
  for (int s = 0; s < 7; ++s) L7[s * stride] = L[s];
  return key_d2(L[6]);
}

// Final list of local agent qi -> neighbour list + count, steering, modification.
__device__ __forceinline__ void finish_agent(const StepArgs& a, int64_t qi, const key_t (&A)[7]) {
  if (qi >= a.nloc) return;
  int nb[7], cnt = 0;
#pragma unroll
  for (int s = 0; s < 7; ++s) {
    nb[s] = A[s] == KEY_EMPTY ? -1 : key_idx(A[s]);
    cnt += A[s] == KEY_EMPTY ? 0 : 1;
  }
#pragma unroll
  for (int s = 0; s < 7; ++s) a.nbr[qi * 7 + s] = nb[s];
  a.cnt[qi] = cnt;
  const float4 p4 = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi));
  const float4 f4 = __ldg(fwd_of(a.full, a.m, a.sdiv, a.lo + qi));
  const V3 F = steer_agent(a, v3(p4), v3(f4), nb, cnt);
  // store_only 1: think mode, k_apply/k_select modifies later; 2: store and modify
  if (a.store_only) a.fstore[qi] = make_float4(F.x, F.y, F.z, 0.f);
  if (a.store_only != 1) modify_agent(a, qi, v3(p4), f4, F);
}

}  // namespace boids
