// k_small.cu -- the whole warm brute-force step in ONE kernel for small flocks
// (single-rank handles, n < SMALL_MAX: C1 and C2).
//
// At n = 1024..8191 a step is latency-bound: round 1 ran it as k_bound ->
// k_scan -> k_select1 -> k_route (+ the Morton binning every 8 steps), and the
// kernel chain -- not the 1-67M pair evaluations -- set the step time (C1 33 us,
// C2 48 us behind a cold L2).  Here P threads share one query: thread `part`
// scans the candidates 4c .. 4c+3 for c = part, part + P, ... (the warp's query
// groups read the same shared-memory slots at once; one minimum of the four
// distances decides whether they are offered one by one), keeps an exact
// running top-8 of (d2, index) keys in registers (reading Q4; the 8th nearest
// seeds the next step's warm bound), limited by the warm bound (steps with
// lists) and by its own 8th key; the P partial lists are merged by a shuffle
// butterfly (exact: every key of the global top-8 is in some part's top-8), and
// the query's first thread writes the list, steers and modifies (Listings
// 5.1-5.5, reading Q10) into the other ping-pong buffer.  Candidates stream
// through shared memory in 1024-agent chunks (round 2's first version read them
// from L1/L2 per thread: 59 % of its stall samples were load latency).  Every pair (i, j),
// j != i, is still tested (Listing 5.2's brute force); only the execution is
// one kernel.  d2 is the exact no-FMA expression of reading Q3 in k_sym's
// packed form (differences and squares of two candidates per FADD2 / FMUL2,
// the sums scalar): round 2's scalar loop spent 27 instructions per pair.
#include <cstdlib>

#include "step_common.cuh"

namespace boids {
namespace {

constexpr int NT = 256;
constexpr int CH = 1024;  // candidates per shared-memory chunk (16 KB)

template <int P>
__global__ void __launch_bounds__(NT) k_small(StepArgs a) {
  const int64_t t = (int64_t)blockIdx.x * NT + threadIdx.x;
  const int part = (int)(t % P);
  const int64_t qi = t / P;
  const bool valid = qi < a.nloc;
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  const float r2_in = __uint_as_float(__float_as_uint(r2) - 1u);  // d2 < r2  <=>  d2 <= r2_in
  const float4 me = valid ? __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi))
                          : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
  const int64_t nc = (a.n + CH - 1) / CH * CH;  // slots beyond m load as NaN phantoms
  // the next chunk's candidates, loaded into registers while the current one
  // computes (the first chunk's loads are in flight during the warm bound)
  float4 v[CH / NT];
  auto load_chunk = [&](int64_t base) {
#pragma unroll
    for (int k = 0; k < CH / NT; ++k) {
      const int64_t j = base + k * NT + threadIdx.x;
      v[k] = j < a.m ? __ldg(a.full + j) : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
    }
  };
  load_chunk(0);
  // inclusive limit: d2 <= min(prev(r2), warm bound) -- every key of the top-7 (and the 8th) passes
  float lim = fminf(r2_in, (valid && a.warm) ? warm_bound(a, qi, me) : __int_as_float(0x7f800000));
  key_t A[8];
#pragma unroll
  for (int s = 0; s < 8; ++s) A[s] = KEY_EMPTY;
  const int64_t g = a.lo + qi;
  // candidates stream through shared memory in chunks of CH as structure of
  // arrays (one coalesced float4 load per thread and CH / NT rounds); the
  // padded slots up to m hold NaN phantoms, which never pass a limit, so the
  // chunks need no guards.  Thread `part` takes the float4 groups part, part +
  // P, ... of each array: four candidates per 16-byte load, and the P threads of
  // a query read consecutive groups (no bank conflicts).
  __shared__ __align__(16) float tx[CH], ty[CH], tz[CH];
  const float4* X4 = reinterpret_cast<const float4*>(tx);
  const float4* Y4 = reinterpret_cast<const float4*>(ty);
  const float4* Z4 = reinterpret_cast<const float4*>(tz);
  // d2 of the query to candidates (2h, 2h+1) of a group: reading Q3 in k_sym's
  // packed form -- x, y, z differences of two candidates per FADD2 (the query's
  // coordinate broadcast), squares per FMUL2, the two sums scalar (no FFMA2)
  auto dist_pair = [&](float4 X, float4 Y, float4 Z, int hi, float& d0, float& d1) {
    const float2 cx = hi ? make_float2(X.z, X.w) : make_float2(X.x, X.y);
    const float2 cy = hi ? make_float2(Y.z, Y.w) : make_float2(Y.x, Y.y);
    const float2 cz = hi ? make_float2(Z.z, Z.w) : make_float2(Z.x, Z.y);
    const float2 dx = __fadd2_rn(make_float2(me.x, me.x), make_float2(-cx.x, -cx.y));
    const float2 dy = __fadd2_rn(make_float2(me.y, me.y), make_float2(-cy.x, -cy.y));
    const float2 dz = __fadd2_rn(make_float2(me.z, me.z), make_float2(-cz.x, -cz.y));
    const float2 x2 = __fmul2_rn(dx, dx), y2 = __fmul2_rn(dy, dy), z2 = __fmul2_rn(dz, dz);
    d0 = __fadd_rn(__fadd_rn(x2.x, y2.x), z2.x);
    d1 = __fadd_rn(__fadd_rn(x2.y, y2.y), z2.y);
  };
  auto offer = [&](float d, int j) {  // exact test of one candidate (rare)
    if (d <= lim && j != (int)g) {
      const key_t k = make_key(d, j);
      if (k < A[7]) {
        insert8(A, k);
        if (A[7] != KEY_EMPTY) lim = fminf(lim, key_d2(A[7]));
      }
    }
  };
  for (int64_t base = 0; base < nc; base += CH) {
    __syncthreads();  // the previous chunk is consumed
#pragma unroll
    for (int k = 0; k < CH / NT; ++k) {
      tx[k * NT + threadIdx.x] = v[k].x;
      ty[k * NT + threadIdx.x] = v[k].y;
      tz[k * NT + threadIdx.x] = v[k].z;
    }
    __syncthreads();
    if (base + CH < nc) load_chunk(base + CH);
#pragma unroll 4
    for (int c4 = part; c4 < CH / 4; c4 += P) {
      const float4 X = X4[c4], Y = Y4[c4], Z = Z4[c4];
      float d0, d1, d2, d3;
      dist_pair(X, Y, Z, 0, d0, d1);
      dist_pair(X, Y, Z, 1, d2, d3);
      if (fminf(fminf(d0, d1), fminf(d2, d3)) <= lim) {  // rare once the list holds 8 (NaN phantoms never)
        const int j0 = (int)base + 4 * c4;
        offer(d0, j0);
        offer(d1, j0 + 1);
        offer(d2, j0 + 2);
        offer(d3, j0 + 3);
      }
    }
  }
  // merge the P partial top-8 lists of the query (lanes t .. t+P-1 of one warp)
#pragma unroll
  for (int o = 1; o < P; o <<= 1) {
    key_t B[8];
#pragma unroll
    for (int s = 0; s < 8; ++s) B[s] = __shfl_xor_sync(0xffffffffu, A[s], o);
    merge8(A, B);
  }
  finish_group<P>(a, qi, valid, part, A, me);
}

}  // namespace

int small_max() { return 8192; }

cudaError_t launch_small(const StepArgs& a, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  // threads per query: enough warps in flight at every size (BOIDS_SMALL_P overrides: 8, 16 or 32)
  static const int force = [] {
    const char* e = getenv("BOIDS_SMALL_P");
    return e ? atoi(e) : 0;
  }();
  const int P = force ? force : (a.nloc <= 2048 ? 32 : 16);
  const int64_t threads = a.nloc * P;
  const unsigned blocks = (unsigned)((threads + NT - 1) / NT);
  if (P == 32) {
    BOIDS_PREFER_SMEM(k_small<32>);
    k_small<32><<<blocks, NT, 0, s>>>(a);
  } else if (P == 16) {
    BOIDS_PREFER_SMEM(k_small<16>);
    k_small<16><<<blocks, NT, 0, s>>>(a);
  } else {
    BOIDS_PREFER_SMEM(k_small<8>);
    k_small<8><<<blocks, NT, 0, s>>>(a);
  }
  return cudaGetLastError();
}

}  // namespace boids
