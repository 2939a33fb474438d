// k_warm.cu -- the warm-start Boids step: k_scan (all pairs, stream-K balanced)
// + k_select (top-7, steering, modification).  Used for every step whose
// previous step left neighbour lists for all owned agents (only the cold step --
// the very first one, before any lists exist -- runs k_fused; boids_set_state
// keeps the lists as bound seeds, so the step after an upload is warm too).
//
// Why a second design.  With the warm threshold t0_i = max over the previous
// step's 7 neighbours j of d2(i, j) at the CURRENT positions, the true 7th key
// of agent i is <= t0_i (those 7 agents still exist), so the result is the top-7
// of the set {j != i : d2 <= min(prev(r2), t0_i)}, which holds only ~8-12 agents.
// The scan therefore needs no running top-7: it APPENDS every passing (d2, j)
// key to a per-agent hit buffer, and the selection happens once, afterwards.
// Without per-query lists the candidate range can be split any way at all, so
//   k_scan   a persistent grid (SMs x occupancy CTAs) walks the item space
//            (query block of 512 agents) x (256-candidate tile) in equal
//            contiguous ranges (stream-K): every CTA gets the same number of
//            items +-1 whatever n is -- no clusters, no wave quantisation.  The
//            hot loop is k_fused's (TMA ring, packed FADD2/FMUL2 distance,
//            FMNMX-tree vote); passing pairs go to a per-warp shared-memory
//            record buffer that is flushed with one global atomic per record.
//   k_select one thread per agent: sort its <= H hits into the top-7 (exact
//            (d2, index) order, reading Q4), then steering + modification.
//            Agents without a warm bound (t0 >= r2: the agent wrapped to the far
//            side of the world, or fewer than 7 previous neighbours) keep an
//            exact running top-7 in k_scan's shared memory instead, flushed as
//            partial lists that k_select merges.  A buffer that still overflows
//            is searched again by its warp, all 32 lanes scanning all
//            candidates (brute force, Listing 5.2).
// Every pair (i, j) is evaluated exactly once by k_scan: brute force as the
// thesis defines it, with the thesis's own re-use of shared memory for
// candidate positions (Listing 6.2).
#include "agent_update.cuh"
#include "tma.cuh"

namespace boids {
namespace {

constexpr int Q = 4;        // queries per thread
constexpr int CT = 128;     // candidates per tile (one TMA bulk copy of 2 KB; fine stream-K granularity)
constexpr int STAGES = 4;   // TMA ring depth
constexpr int U = 4;        // candidates per warp vote
// k_scan CTA shapes: 512 threads (one CTA per SM; its 16 warps share the TMA
// ring, so a warp that runs ahead waits on the ring instead of leaving the SM
// to a lone straggler -- measured 1.7-2x per-CTA spread with 3 small CTAs per
// SM) for large n, 128 threads when there are too few items for 148 CTAs.
constexpr int WB = Q * U * 32;  // records per warp buffer (8 KB): one vote group's maximum
constexpr int UBW = 8;         // per warp: running top-7 lists for unbounded queries

struct __align__(8) Rec {
  int qi;  // local query index
  int pad;
  key_t key;
};

template <int NT>
struct __align__(16) ScanSmem {
  float4 ring[STAGES][CT];
  Rec rec[NT / 32][WB];
  key_t ulist[NT / 32][UBW][7];  // sorted top-7 of unbounded queries (t0 >= r2)
  uint64_t full[STAGES];
  uint64_t empty[STAGES];
};


__device__ __forceinline__ int64_t query_of(const StepArgs& a, int64_t qs) {
  if (qs >= a.nq) return a.nloc;
  return a.qperm ? (int64_t)__ldg(a.qperm + qs) : qs;
}

// t0 of local query qi: an upper bound on its 7th smallest d2 this step, from
// agents that exist -- the previous step's 7 neighbours and, when known, the
// 8th nearest: t0 = 7th smallest of their d2 at the CURRENT positions, i.e. the
// max of the 7 or the second largest of the 8 (so one neighbour that wrapped
// to the far side of the world does not spoil the bound).  +inf without a full
// previous list.  All loads are issued before any is used.
__device__ __forceinline__ float warm_t0(const StepArgs& a, int64_t qi, float4 me) {
  if (qi >= a.nloc) return __int_as_float(0x7f800000);
  int nb[8];
#pragma unroll
  for (int k = 0; k < 7; ++k) nb[k] = __ldg(a.nbr + qi * 7 + k);
  nb[7] = __ldg(a.nbr8 + qi);
  const int c = __ldg(a.cnt + qi);
  float4 p[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) p[k] = __ldg(pos_of(a.full, a.m, a.sdiv, nb[k] < 0 ? 0 : nb[k]));
  float m1 = 0.f, m2 = 0.f;  // largest and second largest of the 8
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const float d = (k < 7 || nb[7] >= 0) ? dist2(me.x, me.y, me.z, p[k]) : 0.f;  // no 8th: ignore
    m2 = fmaxf(m2, fminf(m1, d));
    m1 = fmaxf(m1, d);
  }
  if (c < 7) return __int_as_float(0x7f800000);
  return nb[7] >= 0 ? m2 : m1;
}

// Issue the TMA load of global tile counter tc (stage tc % STAGES), waiting until
// every warp released the stage's previous tile.  Called by thread 0 only.
// Tile k of a run over candidates [c0, c1): [tb, te), CT-aligned inside the run.
__device__ __forceinline__ void run_tile(int64_t c0, int64_t c1, int k, int64_t& tb, int64_t& te) {
  const int64_t base = c0 / CT + k;
  tb = k == 0 ? c0 : base * CT;
  te = min(c1, (base + 1) * CT);
}

// Issue the TMA load of candidates [tb, te) as global tile counter tc (stage tc %
// STAGES), after every warp released the stage's previous tile.  Thread 0 only.
// The range never straddles a slice (m % CT == 0); any multiple of 16 bytes.
template <class SM>
__device__ __forceinline__ void issue_tile(SM& sm, const StepArgs& a, uint32_t tc, int64_t tb, int64_t te) {
  const int s = (int)(tc % STAGES);
  if (tc >= STAGES) {
    mbar_wait(&sm.empty[s], ((tc - STAGES) / STAGES) & 1u);
    fence_proxy_async_smem();
  }
  const uint32_t bytes = (uint32_t)(te - tb) * (uint32_t)sizeof(float4);
  mbar_arrive_expect_tx(&sm.full[s], bytes);
  tma_load_1d(sm.ring[s], pos_of(a.full, a.m, a.sdiv, tb), bytes, &sm.full[s]);
}

// Insert key k into a sorted 7-list in shared memory; returns the new worst d2.
__device__ __noinline__ float insert_l7(key_t* L7, key_t k) {
  key_t L[7];
#pragma unroll
  for (int s = 0; s < 7; ++s) L[s] = L7[s];
  insert7(L, k);
#pragma unroll
  for (int s = 0; s < 7; ++s) L7[s] = L[s];
  return key_d2(L[6]);
}

// Flush a warp's record buffer into the global per-query hit buffers.
// 8 records per lane per round: the atomics' round trips overlap.
__device__ __forceinline__ void flush(const StepArgs& a, const Rec* rec, int n, int lane) {
  for (int i0 = 0; i0 < n; i0 += 32 * 8) {
    Rec r[8];
    int slot[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int i = i0 + k * 32 + lane;
      r[k] = i < n ? rec[i] : Rec{-1, 0, 0ull};
    }
#pragma unroll
    for (int k = 0; k < 8; ++k) slot[k] = r[k].qi >= 0 ? atomicAdd(a.hitcnt + r[k].qi, 1) : a.hits_cap;
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (slot[k] < a.hits_cap) a.hits[(int64_t)r[k].qi * a.hits_cap + slot[k]] = r[k].key;
  }
}

__device__ __forceinline__ void stamp_k(const StepArgs& a, int k) {
  if (a.phase && threadIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    a.phase[blockIdx.x * 8 + k] = t;
  }
}

template <int NTS>
__global__ void __launch_bounds__(NTS, NTS == 128 ? 4 : 1) k_scan(StepArgs a, int64_t ncand, int64_t items) {
  pdl_wait();  // k_bound's limits (think mode: the compacted query list)
  pdl_trigger();
  if (a.qcount) {  // think mode: query slots counted on the device
    a.nq = *a.qcount;
    items = (a.nq + NTS * Q - 1) / (NTS * Q) * ncand;
  } else {
    a.nq = a.nloc;
  }
  constexpr int QBS = NTS * Q;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  ScanSmem<NTS>& sm = *reinterpret_cast<ScanSmem<NTS>*>(smem_raw);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  stamp_k(a, 0);
  // equal shares of the (query block, candidate) space, boundaries on multiples of
  // U (ncand % U == 0), so every tile holds whole vote groups
  const int64_t L0 = items * blockIdx.x / gridDim.x / U * U, L1 = items * (blockIdx.x + 1) / gridDim.x / U * U;
  if (tid == 0) {
#pragma unroll
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], NTS / 32);
    }
    mbar_fence_init();
  }
  __syncthreads();
  stamp_k(a, 4);
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  const float r2_in = __uint_as_float(__float_as_uint(r2) - 1u);  // d2 < r2  <=>  d2 <= r2_in
  Rec* rec = sm.rec[warp];
  int wcount = 0;     // records in this warp's buffer (warp-uniform)
  unsigned slow_groups = 0, groups = 0;
  uint32_t tc = 0;    // tiles issued / consumed by this CTA (ring phase bookkeeping)
  for (int64_t L = L0; L < L1;) {
    // run = one query block x candidates [c0, c1): the CTA's range is an exact
    // 1/grid share of (query blocks x candidates), so every CTA has the same work
    const int64_t qb = L / ncand, c0 = L - qb * ncand;
    const int64_t c1 = min(ncand, c0 + (L1 - L));
    const int nu = (int)((c1 - 1) / CT - c0 / CT + 1);  // tiles in this run
    if (L == L0) stamp_k(a, 5);
    // this run's queries: 4 per thread, in spatial order (qperm)
    float2 pxy[Q];
    float pz[Q], lim[Q];
    int gq[Q], qloc[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const int64_t qi = query_of(a, qb * QBS + warp * 32 * Q + q * 32 + lane);
      qloc[q] = (int)qi;
      gq[q] = (int)(a.lo + qi);
      const float4 me = qi < a.nloc ? __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi))
                                    : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
      pxy[q] = make_float2(me.x, me.y);
      pz[q] = me.z;
      lim[q] = qi < a.nloc ? __ldg(a.qlim + qi) : r2_in;  // inclusive limit from k_bound
    }
    // Unbounded queries (no warm bound: t0 >= r2, e.g. the agent wrapped to the far
    // side of the world) would append every in-radius pair; the first UBW of each
    // warp keep a running top-7 here instead (limit tightening as it fills) and
    // flush it as a partial list at the end of the run.
    if (L == L0) stamp_k(a, 6);
    if (tid == 0)
      for (int t = 0; t < STAGES && t < nu; ++t) {
        int64_t tb, te;
        run_tile(c0, c1, t, tb, te);
        issue_tile(sm, a, tc + t, tb, te);
      }
    if (L == L0) stamp_k(a, 7);
    int ul[Q];
    bool warp_ul;
    {
      int used = 0;
#pragma unroll
      for (int q = 0; q < Q; ++q) {
        const bool ub = qloc[q] < a.nloc && lim[q] >= r2_in;
        const unsigned bal = __ballot_sync(0xffffffffu, ub);
        const int idx = used + __popc(bal & ((1u << lane) - 1u));
        ul[q] = (ub && idx < UBW) ? idx : -1;
        used += __popc(bal);
      }
      warp_ul = used > 0;
      __syncwarp();
      for (int i = lane; i < UBW * 7; i += 32) (&sm.ulist[warp][0][0])[i] = KEY_EMPTY;
      __syncwarp();
    }
    float limc = fmaxf(fmaxf(lim[0], lim[1]), fmaxf(lim[2], lim[3]));
    if (L == L0) stamp_k(a, 1);
    for (int t = 0; t < nu; ++t, ++tc) {
      const int s = (int)(tc % STAGES);
      mbar_wait(&sm.full[s], (tc / STAGES) & 1u);
      const float4* tile = sm.ring[s];
      int64_t tb64, te64;
      run_tile(c0, c1, t, tb64, te64);
      const int jb = (int)tb64, cnt = (int)(te64 - tb64);
      auto group = [&](const int c) {
        float4 cc[U];
#pragma unroll
        for (int u = 0; u < U; ++u) cc[u] = tile[c + u];  // cnt % U == 0
        // d2 = ((dx*dx) + (dy*dy)) + (dz*dz), each op rounded: packed (dx, dy) and
        // squares, scalar dz and sums (see k_fused.cu)
        float d[Q][U];
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            const float2 dxy = __fadd2_rn(pxy[q], make_float2(-cc[u].x, -cc[u].y));
            const float2 sq = __fmul2_rn(dxy, dxy);
            const float dz = __fsub_rn(pz[q], cc[u].z);
            d[q][u] = __fadd_rn(__fadd_rn(sq.x, sq.y), __fmul_rn(dz, dz));
          }
        float mq[Q];
#pragma unroll
        for (int q = 0; q < Q; ++q) {
          mq[q] = d[q][0];
#pragma unroll
          for (int u = 1; u < U; ++u) mq[q] = fminf(mq[q], d[q][u]);
        }
        const float m = fminf(fminf(mq[0], mq[1]), fminf(mq[2], mq[3]));  // NaN (phantoms) ignored
        ++groups;
        if (__any_sync(0xffffffffu, m <= limc)) {  // rare, warp-uniform
          ++slow_groups;
          unsigned bits = 0;
#pragma unroll
          for (int q = 0; q < Q; ++q)
#pragma unroll
            for (int u = 0; u < U; ++u)
              if (d[q][u] <= lim[q] && jb + c + u != gq[q]) bits |= 1u << (q * U + u);
          if (warp_ul) {  // warp-uniform and rare: some query of this warp keeps a list
#pragma unroll
            for (int q = 0; q < Q; ++q)
              if (ul[q] >= 0) {
#pragma unroll
                for (int u = 0; u < U; ++u)
                  if (bits & (1u << (q * U + u)))
                    lim[q] = fminf(lim[q], insert_l7(sm.ulist[warp][ul[q]], make_key(d[q][u], jb + c + u)));
                bits &= ~(((1u << U) - 1u) << (q * U));
              }
          }
          const int nrec = __popc(bits);
          int incl = nrec;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
          }
          const int total = __shfl_sync(0xffffffffu, incl, 31);
          if (wcount + total > WB) {  // warp-uniform; total <= WB always
            __syncwarp();
            flush(a, rec, wcount, lane);
            __syncwarp();
            wcount = 0;
          }
          int off = wcount + incl - nrec;
#pragma unroll
          for (int q = 0; q < Q; ++q)
#pragma unroll
            for (int u = 0; u < U; ++u)
              if (bits & (1u << (q * U + u))) {
                rec[off].qi = qloc[q];
                rec[off].key = make_key(d[q][u], jb + c + u);
                ++off;
              }
          wcount += total;
          limc = fmaxf(fmaxf(lim[0], lim[1]), fmaxf(lim[2], lim[3]));
        }
            };
      if (cnt == CT) {  // full tile: constant trip count (the common case)
#pragma unroll 2
        for (int c = 0; c < CT; c += U) group(c);
      } else {  // ragged tile at a run boundary (cnt % U == 0)
        for (int c = 0; c < cnt; c += U) group(c);
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&sm.empty[s]);
      if (tid == 0 && t + STAGES < nu) {
        int64_t tb, te;
        run_tile(c0, c1, t + STAGES, tb, te);
        issue_tile(sm, a, tc + STAGES, tb, te);
      }
    }
    // partial lists of the unbounded queries -> global (merged by k_select)
    __syncwarp();
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      if (ul[q] >= 0) {
        const int slot = atomicAdd(a.pcnt + qloc[q], 1);
        if (slot < PSLOTS) {
          key_t* dst = a.partial + ((int64_t)qloc[q] * PSLOTS + slot) * 7;
#pragma unroll
          for (int s = 0; s < 7; ++s) dst[s] = sm.ulist[warp][ul[q]][s];
        }
      }
    }
    __syncwarp();
    L += c1 - c0;
  }
  stamp_k(a, 2);
  __syncwarp();
  flush(a, rec, wcount, lane);
  stamp_k(a, 3);
  if (a.stats && lane == 0) {
    atomicAdd(a.stats, (unsigned long long)slow_groups);
    atomicAdd(a.stats + 1, (unsigned long long)groups);
  }
}

// ---------------------------------------------------------------- bound ----
// qlim[i] = min(prev(r2), t0_i): each agent's inclusive search limit for the warm
// scan, computed once per step (k_scan reads it instead of re-gathering the 8
// previous neighbours in every CTA that shares the agent's query block).
__global__ void __launch_bounds__(256) k_bound(StepArgs a) {
  pdl_trigger();  // k_scan may be scheduled now; it waits for this grid before reading the limits
  const int64_t qi = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (qi >= a.nloc) return;
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  const float r2_in = __uint_as_float(__float_as_uint(r2) - 1u);
  const float4 me = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi));
  a.qlim[qi] = fminf(r2_in, warm_t0(a, qi, me));
}

// --------------------------------------------------------------- select ----
constexpr int NSEL = 128;

// Brute-force top-7 of local query qi by the whole warp (lanes stride the
// candidates; per-lane top-7; shuffle butterfly merge).  Result in every lane.
__device__ __noinline__ void warp_full_search(const StepArgs& a, int64_t qi, key_t (&A)[7]) {
  const int lane = threadIdx.x & 31;
  const float4 me = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi));
  const int g = (int)(a.lo + qi);
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
#pragma unroll
  for (int s = 0; s < 7; ++s) A[s] = KEY_EMPTY;
  const int64_t total = (int64_t)a.world * a.m;
  // 8 independent loads in flight per lane (total is a multiple of 256)
  for (int64_t j0 = lane; j0 < total; j0 += 32 * 8) {
    float4 c[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) c[u] = __ldg(pos_of(a.full, a.m, a.sdiv, j0 + 32 * u));
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const float d2 = dist2(me.x, me.y, me.z, c[u]);
      const int j = (int)(j0 + 32 * u);
      if (d2 < r2 && j != g) {
        const key_t k = make_key(d2, j);
        if (k < A[6]) insert7(A, k);
      }
    }
  }
#pragma unroll
  for (int w = 1; w < 32; w <<= 1) {
    key_t B[7];
#pragma unroll
    for (int s = 0; s < 7; ++s) B[s] = __shfl_xor_sync(0xffffffffu, A[s], w);
    merge7(A, B);
  }
}

__global__ void __launch_bounds__(NSEL) k_select(StepArgs a) {
  const int64_t qi = (int64_t)blockIdx.x * NSEL + threadIdx.x;
  // think mode: only warm thinkers were k_scan queries; the others (non-thinkers,
  // and thinkers searched by k_fused this step) take their stored vector
  const bool think = qi < a.nloc && thinks(a.lo + qi, a.step_t, a.think_k);
  const bool routed = think && a.routed && a.routed[qi];
  const bool active = think && !routed;
  const int c = active ? a.hitcnt[qi] : 0;
  const int pc = active ? a.pcnt[qi] : 0;
  const bool over = active && (c > a.hits_cap || pc > PSLOTS);
  key_t A[7];
#pragma unroll
  for (int s = 0; s < 7; ++s) A[s] = KEY_EMPTY;
  key_t eighth = KEY_EMPTY;  // 8th smallest passing key: seeds the next step's t0
  if (active && !over) {
    for (int p = 0; p < pc; ++p) {
      key_t B[7];
#pragma unroll
      for (int s = 0; s < 7; ++s) B[s] = a.partial[(qi * PSLOTS + p) * 7 + s];
      merge7(A, B);
    }
    for (int k = 0; k < c; ++k) insert7(A, a.hits[qi * a.hits_cap + k]);
    for (int k = 0; k < c; ++k) {
      const key_t h = a.hits[qi * a.hits_cap + k];
      if (h > A[6] && h < eighth) eighth = h;
    }
  }
  // overflowed buffers: routed to k_route (one CTA per agent, after this kernel),
  // or else the warp searches those agents again, one at a time
  unsigned om = __ballot_sync(0xffffffffu, over);
  if (a.stats && (threadIdx.x & 31) == 0 && om) atomicAdd(a.stats + 2, (unsigned long long)__popc(om));
  if (a.rlist) {
    if (over) {
      a.rlist[atomicAdd(a.rcount, 1)] = (int)qi;
      a.hitcnt[qi] = 0;
      a.pcnt[qi] = 0;
      a.nbr8[qi] = -1;  // the router writes no 8th nearest: a stale one could repeat a new neighbour
      return;
    }
    om = 0;
  }
  while (om) {
    const int src = __ffs(om) - 1;
    om &= om - 1;
    const int64_t qo = __shfl_sync(0xffffffffu, qi, src);
    key_t B[7];
    warp_full_search(a, qo, B);
    if ((int)(threadIdx.x & 31) == src) {
#pragma unroll
      for (int s = 0; s < 7; ++s) A[s] = B[s];
    }
  }
  if (qi >= a.nloc) return;
  const float4 p4 = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi));
  const float4 f4 = __ldg(fwd_of(a.full, a.m, a.sdiv, a.lo + qi));
  if (!active) {  // think mode, not searched by k_scan this step
    if (routed) a.routed[qi] = 0;
    if (routed && a.think_k <= 1) {  // k_sym step: routed, finished by launch_route after this kernel
      a.nbr8[qi] = -1;
      return;
    }
    const float4 F = a.fstore[qi];
    modify_agent(a, qi, v3(p4), f4, v3(F));
    return;
  }
  a.hitcnt[qi] = 0;  // ready for the next step
  a.pcnt[qi] = 0;
  a.nbr8[qi] = eighth == KEY_EMPTY ? -1 : key_idx(eighth);
  int nb[7], cnt = 0;
#pragma unroll
  for (int s = 0; s < 7; ++s) {
    nb[s] = A[s] == KEY_EMPTY ? -1 : key_idx(A[s]);
    cnt += A[s] == KEY_EMPTY ? 0 : 1;
  }
#pragma unroll
  for (int s = 0; s < 7; ++s) a.nbr[qi * 7 + s] = nb[s];
  a.cnt[qi] = cnt;
  const V3 F = steer_agent(a, v3(p4), v3(f4), nb, cnt);
  if (a.think_k > 1) a.fstore[qi] = make_float4(F.x, F.y, F.z, 0.f);
  modify_agent(a, qi, v3(p4), f4, F);
}

// k_select for warm steps without think frequency (routing on): one agent per
// lane.  Its hit-buffer lines are prefetched into L1 before anything waits on
// a load, the hits are inserted into a sorted top-8 (the 7-list of reading Q4
// and the 8th nearest that seeds the next step's warm bound), then the lane
// steers and modifies the agent.  Same lists and state as k_select; at small
// n this kernel is one warp per SM sub-partition and pure latency, so what
// counts is the length of its dependent chain, not its throughput.
__device__ __forceinline__ void select1_body(const StepArgs& a) {
  const int64_t qi = (int64_t)blockIdx.x * NSEL + threadIdx.x;
  if (qi >= a.nloc) return;
  const key_t* h = a.hits + qi * a.hits_cap;
  prefetch_l1(h);
  prefetch_l1(h + 16);
  const bool routed = a.routed && a.routed[qi];
  const int c = a.hitcnt[qi];  // a routed agent has no hits
  const int pc = a.pcnt[qi];
  if (routed) {  // routed by k_sym_prep: finished by k_route
    a.routed[qi] = 0;
    a.nbr8[qi] = -1;
    return;
  }
  if (c > a.hits_cap || pc > PSLOTS) {  // overflowed buffer: k_route searches the agent whole after this kernel
    if (a.stats) atomicAdd(a.stats + 2, 1ull);
    a.rlist[atomicAdd(a.rcount, 1)] = (int)qi;
    a.hitcnt[qi] = 0;
    a.pcnt[qi] = 0;
    a.nbr8[qi] = -1;
    return;
  }
  key_t L[8];
#pragma unroll
  for (int s = 0; s < 8; ++s) L[s] = KEY_EMPTY;
  int k = 0;
  for (; k + 3 < c; k += 4) {  // 4 loads in flight
    const key_t h0 = h[k], h1 = h[k + 1], h2 = h[k + 2], h3 = h[k + 3];
    insert8(L, h0);
    insert8(L, h1);
    insert8(L, h2);
    insert8(L, h3);
  }
  for (; k < c; ++k) insert8(L, h[k]);
  for (int p = 0; p < pc; ++p) {  // rare: partial lists of unbounded agents (k_scan)
    key_t B[8];
#pragma unroll
    for (int s = 0; s < 7; ++s) B[s] = a.partial[(qi * PSLOTS + p) * 7 + s];
    B[7] = KEY_EMPTY;
    merge8(L, B);
  }
  a.hitcnt[qi] = 0;  // ready for the next step
  a.pcnt[qi] = 0;
  a.nbr8[qi] = L[7] == KEY_EMPTY ? -1 : key_idx(L[7]);
  int nb[7], cnt = 0;
#pragma unroll
  for (int s = 0; s < 7; ++s) {
    nb[s] = L[s] == KEY_EMPTY ? -1 : key_idx(L[s]);
    cnt += L[s] == KEY_EMPTY ? 0 : 1;
  }
#pragma unroll
  for (int s = 0; s < 7; ++s) a.nbr[qi * 7 + s] = nb[s];
  a.cnt[qi] = cnt;
  const float4 p4 = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi));
  const float4 f4 = __ldg(fwd_of(a.full, a.m, a.sdiv, a.lo + qi));
  const V3 F = steer_agent(a, v3(p4), v3(f4), nb, cnt);
  modify_agent(a, qi, v3(p4), f4, F);
}

__global__ void __launch_bounds__(NSEL) k_select1(StepArgs a) {
  pdl_wait();  // the scan's hit buffers
  span_begin(a, SPAN_SLOT0 + 1);
  select1_body(a);
  span_end(a, SPAN_SLOT0 + 1);
}

}  // namespace

template <int NT>
int scan_grid(int sms) {
  static int grid = 0;
  if (!grid) {
    int r = 0;
    cudaFuncSetAttribute(k_scan<NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(ScanSmem<NT>));
    cudaFuncSetAttribute(k_scan<NT>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&r, k_scan<NT>, NT, sizeof(ScanSmem<NT>));
    grid = sms * (r > 0 ? r : 1);
  }
  return grid;
}

// Smallest CTA share of the (query block, candidate) items (measured C1: 128 ->
// 42.2, 32 -> 32.5, 16 -> 30.5 us/step; C2 unchanged).  At small n the scan
// is latency-bound (a CTA's time is mostly its fixed prologue and TMA latency),
// so spreading it over more SMs beats whole-tile shares.
#ifndef BOIDS_SCAN_MIN
#define BOIDS_SCAN_MIN 16
#endif
constexpr int64_t SCAN_MIN = BOIDS_SCAN_MIN;

template <int NT>
cudaError_t scan_with(const StepArgs& a, int sms, int64_t ncand, cudaStream_t s) {
  const int64_t nqb = (a.nloc + NT * Q - 1) / (NT * Q);
  const int64_t items = nqb * ncand;  // (query block, candidate) pairs; think mode: recomputed on device
  const int g = a.qcount ? scan_grid<NT>(sms)
                         : (int)std::min<int64_t>(scan_grid<NT>(sms), (items + SCAN_MIN - 1) / SCAN_MIN);
  return launch_pdl(k_scan<NT>, dim3(g), dim3(NT), sizeof(ScanSmem<NT>), s, a, ncand, items);
}

#ifndef BOIDS_SCAN_BIG
#define BOIDS_SCAN_BIG 512  // 640 (20 warps) caps registers at 96 and spills: measured 15% slower
#endif
cudaError_t scan_big(const StepArgs& a, int sms, int64_t ncand, cudaStream_t s) {
  return scan_with<BOIDS_SCAN_BIG>(a, sms, ncand, s);
}

cudaError_t launch_warm_scan(const StepArgs& a, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  BOIDS_PREFER_SMEM(k_bound);
  k_bound<<<(unsigned)((a.nloc + 255) / 256), 256, 0, s>>>(a);
  if (cudaError_t e = cudaGetLastError()) return e;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t ncand = (int64_t)a.world * a.m;
  // one 512-thread CTA per SM when every SM gets >= 4 tiles of (2048 queries x CT)
  const int64_t tiles512 = (a.nloc + 2047) / 2048 * (ncand / CT);
  if (tiles512 >= 4LL * sms) return scan_big(a, sms, ncand, s);
  return scan_with<128>(a, sms, ncand, s);
}

cudaError_t launch_warm_select(const StepArgs& a, cudaStream_t s, bool pdl) {
  if (a.nloc <= 0) return cudaSuccess;
  if (a.think_k <= 1 && a.rlist) {
    BOIDS_PREFER_SMEM(k_select1);
    return launch_pdl_if(pdl, k_select1, dim3((unsigned)((a.nloc + NSEL - 1) / NSEL)), dim3(NSEL), 0, s, a);
  }
  BOIDS_PREFER_SMEM(k_select);
  k_select<<<(unsigned)((a.nloc + NSEL - 1) / NSEL), NSEL, 0, s>>>(a);
  return cudaGetLastError();
}

}  // namespace boids
