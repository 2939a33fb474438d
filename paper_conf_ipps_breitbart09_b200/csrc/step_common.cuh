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

// The finish of one query by the P lanes of its group (P divides 32; every lane
// of the warp calls this -- it shuffles with the full mask): A = the query's
// exact top-8 in every lane of the group, me = its position.  OpenSteer's
// behaviours: the serial finish_agent in the first lane.  The thesis's (Listings
// 5.3-5.5, reading Q10): lane `part` < cnt computes neighbour `part`'s offset o,
// its separation term (o / L) / L (L > 0) and forward -- the square root and the
// divisions, the long part -- and the group's first lane sums them IN KEY ORDER
// (reading Q8), so every rounding is the serial steer_agent's; then it writes
// the lists and modifies.  Not for think mode (no stored steering).
template <int P>
__device__ __forceinline__ void finish_group(const StepArgs& a, int64_t qi, bool valid, int part, const key_t (&A)[8],
                                             float4 me) {
  if (a.p.steer_mode != BOIDS_STEER_THESIS) {  // OpenSteer's behaviours: the serial per-agent finish
    if (!valid || part != 0) return;
    a.nbr8[qi] = A[7] == KEY_EMPTY ? -1 : key_idx(A[7]);
    key_t L[7];
#pragma unroll
    for (int s = 0; s < 7; ++s) L[s] = A[s];
    finish_agent(a, qi, L);
    return;
  }
  int cnt = 0, nbk = -1;
#pragma unroll
  for (int s = 0; s < 7; ++s) {
    cnt += A[s] == KEY_EMPTY ? 0 : 1;
    if (s == part) nbk = A[s] == KEY_EMPTY ? -1 : key_idx(A[s]);
  }
  const V3 me3 = v3(me);
  V3 o = v3(0.f, 0.f, 0.f), term = o, fj = o;
  int use = 0;
  if (valid && nbk >= 0) {
    const float4 pj = __ldg(pos_of(a.full, a.m, a.sdiv, nbk));
    const float4 fj4 = __ldg(fwd_of(a.full, a.m, a.sdiv, nbk));
    o = sub(v3(pj), me3);  // A.position - me.position (Listing 5.3)
    const float L = len(o);
    if (L > 0.0f) {
      term = divs(divs(o, L), L);  // 1/d fall-off
      use = 1;
    }
    fj = v3(fj4);
  }
  const int lane = threadIdx.x & 31, base = lane - part;
  V3 sep = v3(0.f, 0.f, 0.f), coh = sep, ali = sep;
#pragma unroll
  for (int k = 0; k < 7; ++k) {  // all lanes shuffle; the first lane of each group accumulates
    const int src = base + k;
    const V3 ok = v3(__shfl_sync(0xffffffffu, o.x, src), __shfl_sync(0xffffffffu, o.y, src),
                     __shfl_sync(0xffffffffu, o.z, src));
    const V3 tk = v3(__shfl_sync(0xffffffffu, term.x, src), __shfl_sync(0xffffffffu, term.y, src),
                     __shfl_sync(0xffffffffu, term.z, src));
    const V3 fk = v3(__shfl_sync(0xffffffffu, fj.x, src), __shfl_sync(0xffffffffu, fj.y, src),
                     __shfl_sync(0xffffffffu, fj.z, src));
    const int uk = __shfl_sync(0xffffffffu, use, src);
    if (k < cnt) {
      if (uk) sep = sub(sep, tk);  // Listing 5.3 line 10
      coh = add(coh, ok);          // Listing 5.4 line 8
      ali = add(ali, fk);          // Listing 5.5 line 7
    }
  }
  if (!valid || part != 0) return;
  a.nbr8[qi] = A[7] == KEY_EMPTY ? -1 : key_idx(A[7]);
#pragma unroll
  for (int s = 0; s < 7; ++s) a.nbr[qi * 7 + s] = A[s] == KEY_EMPTY ? -1 : key_idx(A[s]);
  a.cnt[qi] = cnt;
  const float4 f4 = __ldg(fwd_of(a.full, a.m, a.sdiv, a.lo + qi));
  ali = sub(ali, scale(v3(f4), (float)cnt));  // Listing 5.5 line 10
  const V3 sw = scale(normalize(sep), a.p.w_separation);
  const V3 aw = scale(normalize(ali), a.p.w_alignment);
  const V3 cw = scale(normalize(coh), a.p.w_cohesion);
  const V3 F = add(add(sw, aw), cw);  // Listing 5.1 line 5
  modify_agent(a, qi, me3, f4, F);
}

}  // namespace boids
