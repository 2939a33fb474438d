// k_basic.cu -- initial state, phantom fill, the two-kernel step
// (tiled search -> neighbour lists; update from lists).
//
// The two-kernel step mirrors the thesis's own structure (search kernel with a
// shared-memory position cache, Listing 6.2; separate modification
// kernel) and doubles as the standalone HBM-bound update kernel of
// SURVEY.md B5.  The default step is the fused kernel in k_fused.cu.
#include <algorithm>
#include "agent_update.cuh"

namespace boids {

// ---------------------------------------------------------------- init ----
// DESIGN.md Appendix B; agent g's stream depends only on (seed, g).
__device__ __forceinline__ float draw_coord(uint64_t& s) {
  s += SM64_GAMMA;
  uint64_t out = sm64_mix(s);
  float u = __fmul_rn((float)(uint32_t)(out >> 40), 5.9604644775390625e-08f);  // exact
  return __fsub_rn(__fmul_rn(u, 2.0f), 1.0f);
}
__device__ __forceinline__ V3 draw_ball(uint64_t& s) {
  for (;;) {
    float x = draw_coord(s), y = draw_coord(s), z = draw_coord(s);
    V3 v = v3(x, y, z);
    if (dot(v, v) < 1.0f) return v;
  }
}

__global__ void k_init(float4* out, float4* up4, float4* side4, int64_t m, int64_t lo,
                       int64_t nloc, boids_params p, uint64_t seed) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nloc) return;
  uint64_t g = (uint64_t)(lo + i);
  uint64_t s = sm64(seed ^ sm64(g));
  float R = p.init_mode == BOIDS_INIT_WORLD ? p.world_radius : p.init_radius;
  V3 pos = scale(draw_ball(s), R);
  V3 f = normalize(draw_ball(s));
  V3 side = normalize(cross(f, v3(0.f, 1.f, 0.f)));
  V3 up = cross(side, f);
  float sp = __fmul_rn(p.init_speed_frac, p.max_speed);
  out[i] = make_float4(pos.x, pos.y, pos.z, 0.f);
  out[m + i] = make_float4(f.x, f.y, f.z, sp);
  up4[i] = make_float4(up.x, up.y, up.z, 0.f);
  side4[i] = make_float4(side.x, side.y, side.z, 0.f);
}

cudaError_t launch_init(float4* out, float4* up4, float4* side4, int64_t m, int64_t lo,
                        int64_t nloc, const boids_params& p, uint64_t seed, cudaStream_t s) {
  if (nloc <= 0) return cudaSuccess;
  int64_t blocks = (nloc + 255) / 256;
  k_init<<<(unsigned)blocks, 256, 0, s>>>(out, up4, side4, m, lo, nloc, p, seed);
  return cudaGetLastError();
}

// Phantom agents [nloc, m) of each segment: NaN position (d2 = NaN is never < r2), zero fwd.
__global__ void k_fill_phantoms(float4* base, int64_t m, int64_t nloc, int64_t segments) {
  int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  int64_t per = m - nloc;
  if (k >= per * segments) return;
  int64_t seg = k / per, i = nloc + k % per;
  float nan = __int_as_float(0x7fc00000);
  base[seg * 2 * m + i] = make_float4(nan, nan, nan, 0.f);
  base[seg * 2 * m + m + i] = make_float4(0.f, 0.f, 0.f, 0.f);
}

cudaError_t launch_fill_phantoms(float4* base, int64_t m, int64_t nloc, int64_t segments,
                                 cudaStream_t s) {
  int64_t total = (m - nloc) * segments;
  if (total <= 0) return cudaSuccess;
  k_fill_phantoms<<<(unsigned)((total + 255) / 256), 256, 0, s>>>(base, m, nloc, segments);
  return cudaGetLastError();
}

__global__ void k_fill_nan(float4* p, int64_t count) {
  int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= count) return;
  float nan = __int_as_float(0x7fc00000);
  p[k] = make_float4(nan, nan, nan, __int_as_float(-1));
}

cudaError_t launch_fill_nan(float4* p, int64_t count, cudaStream_t s) {
  if (count <= 0) return cudaSuccess;
  k_fill_nan<<<(unsigned)((count + 255) / 256), 256, 0, s>>>(p, count);
  return cudaGetLastError();
}

// Host-transfer staging: [pos3 | fwd3 | up3 | side3 | speed] (k agents each) <-> float4 state.
__global__ void k_state_in(const float* __restrict__ st, int has_side, int64_t k, float4* local, int64_t m,
                           float4* up4, float4* side4) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= k) return;
  const float* p = st + 3 * i;
  const float* f = st + 3 * k + 3 * i;
  const float* u = st + 6 * k + 3 * i;
  const float* s = st + 9 * k + 3 * i;
  local[i] = make_float4(p[0], p[1], p[2], 0.f);
  local[m + i] = make_float4(f[0], f[1], f[2], st[12 * k + i]);
  up4[i] = make_float4(u[0], u[1], u[2], 0.f);
  side4[i] = has_side ? make_float4(s[0], s[1], s[2], 0.f) : make_float4(0.f, 0.f, 0.f, 0.f);
}

__global__ void k_state_out(const float4* __restrict__ local, int64_t m, const float4* __restrict__ up4,
                            const float4* __restrict__ side4, int64_t k, float* st) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= k) return;
  const float4 p = local[i], f = local[m + i], u = up4[i], s = side4[i];
  float* P = st + 3 * i;
  float* F = st + 3 * k + 3 * i;
  float* Uu = st + 6 * k + 3 * i;
  float* S = st + 9 * k + 3 * i;
  P[0] = p.x, P[1] = p.y, P[2] = p.z;
  F[0] = f.x, F[1] = f.y, F[2] = f.z;
  Uu[0] = u.x, Uu[1] = u.y, Uu[2] = u.z;
  S[0] = s.x, S[1] = s.y, S[2] = s.z;
  st[12 * k + i] = f.w;
}

cudaError_t launch_state_in(const float* stage, bool has_side, int64_t k, float4* local, int64_t m, float4* up4,
                            float4* side4, cudaStream_t s) {
  if (k <= 0) return cudaSuccess;
  k_state_in<<<(unsigned)((k + 255) / 256), 256, 0, s>>>(stage, has_side ? 1 : 0, k, local, m, up4, side4);
  return cudaGetLastError();
}

cudaError_t launch_state_out(const float4* local, int64_t m, const float4* up4, const float4* side4, int64_t k,
                             float* stage, cudaStream_t s) {
  if (k <= 0) return cudaSuccess;
  k_state_out<<<(unsigned)((k + 255) / 256), 256, 0, s>>>(local, m, up4, side4, k, stage);
  return cudaGetLastError();
}

// boids_set_state's locality check (only a performance decision, never a
// result): does the spatial query order qperm still group nearby agents in the
// uploaded positions?  Up to 256 strided pairs of consecutive qperm entries;
// out[0] = valid pairs, out[1] = pairs still within the search radius.  Reads
// the positions from the staging buffer (AoS pos3 = stage[0 .. 3k)).
__global__ void k_order_check(const float* __restrict__ pos3, const int32_t* __restrict__ qperm, int64_t k,
                              int64_t stride, int64_t cnt, float r2, int* __restrict__ out) {
  __shared__ int sv, sn;
  if (threadIdx.x == 0) sv = sn = 0;
  __syncthreads();
  const int64_t t = threadIdx.x;
  if (t < cnt) {
    const int64_t a = qperm[t * stride], b = qperm[t * stride + 1];
    if (a >= 0 && a < k && b >= 0 && b < k) {
      float d2 = 0.f;
      for (int d = 0; d < 3; ++d) {
        const float x = __fsub_rn(pos3[3 * a + d], pos3[3 * b + d]);
        d2 = __fadd_rn(d2, __fmul_rn(x, x));
      }
      atomicAdd(&sv, 1);
      if (d2 <= r2) atomicAdd(&sn, 1);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    out[0] = sv;
    out[1] = sn;
  }
}

cudaError_t launch_order_check(const float* pos3, const int32_t* qperm, int64_t k, float r2, int* out,
                               cudaStream_t s) {
  if (k < 2) return cudaMemsetAsync(out, 0, 2 * sizeof(int), s);
  const int64_t stride = std::max<int64_t>(1, (k - 1) / 256);
  const int64_t cnt = std::min<int64_t>(256, (k - 1) / stride);
  k_order_check<<<1, 256, 0, s>>>(pos3, qperm, k, stride, cnt, r2, out);
  return cudaGetLastError();
}

// Draw data of the double-buffered readback: the 4x4 local-space matrix per agent
// (rows side, up, forward, position), 64 B, packed contiguously.
__global__ void k_pack_draw(const float4* __restrict__ local, int64_t m, const float4* __restrict__ up4,
                            const float4* __restrict__ side4, int64_t k, float4* __restrict__ draw) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= k) return;
  const float4 s = side4[i], u = up4[i], f = local[m + i], p = local[i];
  draw[4 * i + 0] = make_float4(s.x, s.y, s.z, 0.f);
  draw[4 * i + 1] = make_float4(u.x, u.y, u.z, 0.f);
  draw[4 * i + 2] = make_float4(f.x, f.y, f.z, 0.f);
  draw[4 * i + 3] = make_float4(p.x, p.y, p.z, 1.f);
}

cudaError_t launch_pack_draw(const float4* local, int64_t m, const float4* up4, const float4* side4, int64_t k,
                             float4* draw, cudaStream_t s) {
  if (k <= 0) return cudaSuccess;
  k_pack_draw<<<(unsigned)((k + 255) / 256), 256, 0, s>>>(local, m, up4, side4, k, draw);
  return cudaGetLastError();
}

// ------------------------------------------------------- simple search ----
// One thread per owned agent; candidate positions staged through shared memory
// one TILE at a time (the thesis's version-2 structure, Listing 6.2), register
// top-7 of (d2, idx) keys.  Candidates are scanned in increasing index order, so
// the strict d2 < worst test realises the index tie-break of reading Q4.
__global__ void __launch_bounds__(TILE) k_search_simple(StepArgs a) {
  __shared__ float4 tile[TILE];
  int64_t i = (int64_t)blockIdx.x * TILE + threadIdx.x;
  bool active = i < a.nloc;
  int64_t g = a.lo + i;
  float4 me = active ? *pos_of(a.full, a.m, a.sdiv, g) : make_float4(0.f, 0.f, 0.f, 0.f);
  float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  key_t L[7];
#pragma unroll
  for (int s = 0; s < 7; ++s) L[s] = KEY_EMPTY;
  float lim = r2;
  int cnt = 0;
  int64_t total = (int64_t)a.world * a.m;
  for (int64_t base = 0; base < total; base += TILE) {
    tile[threadIdx.x] = *pos_of(a.full, a.m, a.sdiv, base + threadIdx.x);
    __syncthreads();
    for (int k = 0; k < TILE; ++k) {
      float d2 = dist2(me.x, me.y, me.z, tile[k]);
      int64_t j = base + k;
      if (d2 < lim && j != g) {
        insert7(L, make_key(d2, (int)j));
        cnt = cnt < 7 ? cnt + 1 : 7;
        if (cnt == 7) lim = fminf(r2, key_d2(L[6]));
      }
    }
    __syncthreads();
  }
  if (!active) return;
#pragma unroll
  for (int s = 0; s < 7; ++s) a.nbr[i * 7 + s] = s < cnt ? key_idx(L[s]) : -1;
  a.cnt[i] = cnt;
}

cudaError_t launch_search_simple(const StepArgs& a, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  k_search_simple<<<(unsigned)((a.nloc + TILE - 1) / TILE), TILE, 0, s>>>(a);
  return cudaGetLastError();
}

// -------------------------------------------------------------- update ----
// Steering + modification from the neighbour lists: one thread per owned agent.
__global__ void __launch_bounds__(256) k_update(StepArgs a) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= a.nloc) return;
  int64_t g = a.lo + i;
  float4 p4 = __ldg(pos_of(a.full, a.m, a.sdiv, g));
  float4 f4 = __ldg(fwd_of(a.full, a.m, a.sdiv, g));
  int cnt = a.cnt[i];
  int nb[7];
#pragma unroll
  for (int s = 0; s < 7; ++s) nb[s] = a.nbr[i * 7 + s];
  V3 F = steer_agent(a, v3(p4), v3(f4), nb, cnt);
  modify_agent(a, i, v3(p4), f4, F);
}

// Think mode: the modification substage of every owned agent with its stored
// steering vector (written this step by the searching kernel for thinkers,
// kept from an earlier step for the others).  HBM-bound: ~64 B in, 64 B out.
__global__ void __launch_bounds__(256) k_apply(StepArgs a) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= a.nloc) return;
  const float4 p4 = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + i));
  const float4 f4 = __ldg(fwd_of(a.full, a.m, a.sdiv, a.lo + i));
  const float4 F = a.fstore[i];
  modify_agent(a, i, v3(p4), f4, v3(F));
}

cudaError_t launch_apply(const StepArgs& a, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  BOIDS_PREFER_SMEM(k_apply);
  k_apply<<<(unsigned)((a.nloc + 255) / 256), 256, 0, s>>>(a);
  return cudaGetLastError();
}

// Think mode: split the thinking agents, in qperm (spatial) order, into those
// never searched (cnt < 0 -> k_fused) and the rest (-> warm scan).  Block-wide
// compaction keeps 1024 / k consecutive -- spatially coherent -- agents together.
__global__ void __launch_bounds__(1024) k_think_compact(StepArgs a, const int32_t* __restrict__ qperm,
                                                        int32_t* cold, int32_t* ncold, int32_t* warm,
                                                        int32_t* nwarm) {
  __shared__ int wsum[2][32];
  __shared__ int base[2];
  const int64_t s = (int64_t)blockIdx.x * 1024 + threadIdx.x;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int qi = -1;
  bool th = false, c = false;
  if (s < a.nloc) {
    qi = qperm[s];
    th = thinks(a.lo + qi, a.step_t, a.think_k);
    c = th && a.cnt[qi] < 0;
    if (th) a.routed[qi] = c ? 1 : 0;
    if (c) a.nbr8[qi] = -1;
  }
  const unsigned bc = __ballot_sync(0xffffffffu, c), bw = __ballot_sync(0xffffffffu, th && !c);
  if (lane == 0) {
    wsum[0][w] = __popc(bc);
    wsum[1][w] = __popc(bw);
  }
  __syncthreads();
  if (threadIdx.x < 64) {  // warp 0: cold scan, warp 1: warm scan (exclusive over warps)
    const int k = threadIdx.x >> 5;
    int v = wsum[k][lane], x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    wsum[k][lane] = x - v;
    if (lane == 31) base[k] = atomicAdd(k ? nwarm : ncold, x);
  }
  __syncthreads();
  const unsigned below = (1u << lane) - 1u;
  if (c) cold[base[0] + wsum[0][w] + __popc(bc & below)] = qi;
  if (th && !c) warm[base[1] + wsum[1][w] + __popc(bw & below)] = qi;
}

cudaError_t launch_think_compact(const StepArgs& a, const int32_t* qperm, int32_t* cold, int32_t* ncold,
                                 int32_t* warm, int32_t* nwarm, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  BOIDS_PREFER_SMEM(k_think_compact);
  k_think_compact<<<(unsigned)((a.nloc + 1023) / 1024), 1024, 0, s>>>(a, qperm, cold, ncold, warm, nwarm);
  return cudaGetLastError();
}

cudaError_t launch_update(const StepArgs& a, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  BOIDS_PREFER_SMEM(k_update);
  k_update<<<(unsigned)((a.nloc + 255) / 256), 256, 0, s>>>(a);
  return cudaGetLastError();
}

}  // namespace boids
