// k_small.cu -- the whole warm brute-force step in ONE kernel for small flocks
// (single-rank handles, n < SMALL_MAX: C1 and C2).
//
// At n = 1024..8191 a step is latency-bound: round 1 ran it as k_bound ->
// k_scan -> k_select1 -> k_route (+ the Morton binning every 8 steps), and the
// kernel chain -- not the 1-67M pair evaluations -- set the step time (C1 33 us,
// C2 48 us behind a cold L2).  Here P threads share one query: thread `part`
// scans candidates j = part, part + P, ... (the warp's query groups read the
// same shared-memory slots at once), keeps an exact
// running top-8 of (d2, index) keys in registers (reading Q4; the 8th nearest
// seeds the next step's warm bound), limited by the warm bound (steps with
// lists) and by its own 8th key; the P partial lists are merged by a shuffle
// butterfly (exact: every key of the global top-8 is in some part's top-8), and
// the query's first thread writes the list, steers and modifies (Listings
// 5.1-5.5, reading Q10) into the other ping-pong buffer.  Candidates stream
// through shared memory in 1024-agent chunks (round 2's first version read them
// from L1/L2 per thread: 59 % of its stall samples were load latency).  Every pair (i, j),
// j != i, is still tested (Listing 5.2's brute force); only the execution is
// one kernel.  d2 is the exact no-FMA expression of reading Q3 (dist2).
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
  // inclusive limit: d2 <= min(prev(r2), warm bound) -- every key of the top-7 (and the 8th) passes
  float lim = fminf(r2_in, (valid && a.warm) ? warm_bound(a, qi, me) : __int_as_float(0x7f800000));
  key_t A[8];
#pragma unroll
  for (int s = 0; s < 8; ++s) A[s] = KEY_EMPTY;
  const int64_t g = a.lo + qi;
  // candidates stream through shared memory in chunks of CH (one coalesced
  // float4 load per thread and CH / NT rounds); the padded slots up to m hold
  // NaN phantoms, which never pass a limit, so the chunks need no guards
  __shared__ float4 tile[CH];
  const int64_t nc = (a.n + CH - 1) / CH * CH;  // slots beyond m load as NaN phantoms
  for (int64_t base = 0; base < nc; base += CH) {
    __syncthreads();  // the previous chunk is consumed
#pragma unroll
    for (int k = 0; k < CH / NT; ++k) {
      const int64_t j = base + k * NT + threadIdx.x;
      tile[k * NT + threadIdx.x] = j < a.m ? __ldg(a.full + j) : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
    }
    __syncthreads();
#pragma unroll 8
    for (int c = part; c < CH; c += P) {
      const float4 cc = tile[c];
      const float d = dist2(me.x, me.y, me.z, cc);
      const int64_t j = base + c;
      if (d <= lim && j != g) {  // rare once the list holds 8: the limit follows its 8th key
        const key_t k = make_key(d, (int)j);
        if (k < A[7]) {
          insert8(A, k);
          if (A[7] != KEY_EMPTY) lim = fminf(lim, key_d2(A[7]));
        }
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
