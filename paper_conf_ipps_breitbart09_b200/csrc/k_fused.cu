// k_fused.cu -- the fused Boids step for sm_100a: brute-force 7-NN search +
// split merge + steering + modification in ONE kernel per step.
//
// Thesis lineage (prior art, not the blueprint): version 2's shared-memory
// position cache (Listing 6.2), version 4's recompute-not-cache
// (P:493), version 5's device-resident modification.  What is new:
//
//  * Work unit = (query block of QB = NT * Q agents, candidate chunk).  A thread
//    block cluster of K CTAs (K in {1,2,4,8,16}) shares one query block; CTA r
//    of the cluster scans candidate chunk r of K.  NT (64 or 128 threads) and K
//    are chosen by plan_launch so the grid is close to a whole multiple of the
//    SM count with enough warps per SM.
//  * Candidate positions are streamed global -> shared memory by the TMA bulk
//    copy engine (cp.async.bulk + mbarrier complete_tx) through a STAGES-deep
//    ring of 256-candidate tiles; all 4 warps read each candidate with a
//    broadcast LDS.128.
//  * Each thread owns Q = 4 queries (4 independent distance chains per LDS.128;
//    Q = 2 measured ~0.58 of the lane-op peak).  The distance uses packed
//    FADD2/FMUL2 on (x, y) pairs + scalar dz and sums: 6 issue slots per 8 FP32
//    lane-ops, so the loop is bound by the FP32 pipe rather than by issue
//    (tools/probe_loop.cu: 0.78-0.81 vs 0.72-0.75 scalar).  The sorted top-7
//    lists of 64-bit (d2, index) keys (the reading-Q4 total order) live in
//    shared memory: only the rare insertion path touches them.
//  * Warm threshold: t0 = max d2 to the previous step's 7 neighbours at the
//    current positions is an upper bound on the true 7th key, so only
//    candidates with d2 <= t0 can enter (identical result, far fewer inserts).
//    Per query lim = min(r2, next(t0), worst held); the fast test is a min
//    tree over the Q*U distances against the thread's max lim.
//  * The hot loop is warp-uniform: a vote over U candidates x Q queries takes
//    the (rare) insertion path only when some lane needs it (the SIMD branching
//    issue of sec 6.3.1).
//  * Split merge through distributed shared memory: after a cluster barrier the
//    CTA that owns a query gathers the K partial lists (DSMEM), merges them
//    with a bitonic half-cleaner + warp-shuffle butterfly, and runs the
//    steering + modification epilogue, writing the ping-pong state (Jacobi
//    semantics, P:418 / P:440).
#include <cooperative_groups.h>

#include "agent_update.cuh"
#include "tma.cuh"

namespace cg = cooperative_groups;

namespace boids {
namespace {

constexpr int Q = 4;        // queries per thread (4 independent distance chains)
constexpr int CT = 256;     // candidates per tile (4 KB)
constexpr int STAGES = 2;   // TMA ring depth (a tile takes ~10-25 us to consume; TMA latency ~1 us)

__device__ __forceinline__ void stamp(const StepArgs& a, int k) {
  if (a.phase && threadIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    a.phase[blockIdx.x * 8 + k] = t;
  }
}

__device__ __forceinline__ void cluster_arrive() {
  asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_wait() {
  asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}

template <int NT>
struct __align__(16) Smem {
  static constexpr int QB = NT * Q;
  float4 ring[STAGES][CT];  // candidate tiles (TMA destination)
  key_t lists[7 * QB];      // sorted top-7 per query, k-major [7][QB]; touched only on inserts
  float t0[QB];             // warm thresholds (each cluster rank fills its share)
  uint64_t full[STAGES];
  uint64_t empty[STAGES];
};

// Insert (d2, j) into the shared-memory list of query slot ql; returns the new
// worst d2 (+inf while fewer than 7 are held).  Out of line: it runs rarely and
// one copy keeps the hot loop small in the instruction cache.
__device__ __noinline__ float insert_list(key_t* lists, int qb, int ql, float d2, int j) {
  key_t L[7];
#pragma unroll
  for (int s = 0; s < 7; ++s) L[s] = lists[s * qb + ql];
  insert7(L, make_key(d2, j));
#pragma unroll
  for (int s = 0; s < 7; ++s) lists[s * qb + ql] = L[s];
  return key_d2(L[6]);
}

__device__ __forceinline__ const float4* tile_src(const StepArgs& a, int64_t tile) {
  return pos_of(a.full, a.m, a.sdiv, tile * CT);  // m % CT == 0: a tile never straddles a slice
}

// number of query slots (think mode: a device-side count)
__device__ __forceinline__ int64_t num_queries(const StepArgs& a) {
  return a.qcount ? (int64_t)*a.qcount : a.nloc;
}

// local query index held by block slot qs (>= nq: inactive slot)
__device__ __forceinline__ int64_t query_of(const StepArgs& a, int64_t qs) {
  if (qs >= a.nq) return a.nloc;
  return a.qperm ? (int64_t)__ldg(a.qperm + qs) : qs;
}

// t0 for local query ql (returns +inf when there is no valid warm list).
__device__ __forceinline__ float warm_t0(const StepArgs& a, int64_t ql) {
  if (!a.warm || ql >= a.nloc) return __int_as_float(0x7f800000);
  if (a.cnt[ql] < 7) return __int_as_float(0x7f800000);
  float4 me = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + ql));
  float t = 0.f;
#pragma unroll
  for (int k = 0; k < 7; ++k) {
    int j = a.nbr[ql * 7 + k];
    t = fmaxf(t, dist2(me.x, me.y, me.z, __ldg(pos_of(a.full, a.m, a.sdiv, j))));
  }
  return t;
}

// Final list of local query qi -> neighbour list, count, steering, modification.
__device__ __forceinline__ void finish_query(const StepArgs& a, int64_t qi, const key_t (&A)[7]) {
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
  float4 p4 = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi));
  float4 f4 = __ldg(fwd_of(a.full, a.m, a.sdiv, a.lo + qi));
  V3 F = steer_agent(a, v3(p4), v3(f4), nb, cnt);
  // store_only 1: think mode, k_apply/k_select modifies later; 2: store and modify
  if (a.store_only) a.fstore[qi] = make_float4(F.x, F.y, F.z, 0.f);
  if (a.store_only != 1) modify_agent(a, qi, v3(p4), f4, F);
}

template <int NT, int K, int U>
__global__ void __launch_bounds__(NT) k_fused(StepArgs a, int64_t tiles_total) {
  a.nq = num_queries(a);
  if ((int64_t)(blockIdx.x / K) * (NT * Q) >= a.nq) return;  // whole cluster: no queries left
  constexpr int QB = NT * Q;    // queries per CTA (and per cluster)
  constexpr int QPC = QB / K;   // queries owned (merged + finished) by each cluster rank
  constexpr int NW = NT / 32;
  __shared__ Smem<NT> sm;
  float4(*ring)[CT] = sm.ring;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int r = K > 1 ? (int)cg::this_cluster().block_rank() : 0;
  const int64_t q_base = (int64_t)(blockIdx.x / K) * QB;  // local index of the block's first query
  // cluster rank r scans tiles r, r + K, r + 2K, ...: strided, so the hits of a
  // spatially coherent query block are spread evenly over the cluster's CTAs
  const int nt = (int)((tiles_total - r + K - 1) / K);

  stamp(a, 0);
  if (tid == 0) {
#pragma unroll
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], NT);
    }
    mbar_fence_init();
  }
  // fence.mbarrier_init is a release at cluster scope: in a cluster launch the
  // barriers' initialisation is made visible by a cluster barrier (the acquire),
  // before the first arrive / bulk copy uses them
  if constexpr (K > 1) cg::this_cluster().sync();
  else __syncthreads();
  if (tid == 0) {  // prologue: fill the ring
    for (int t = 0; t < STAGES && t < nt; ++t) {
      mbar_arrive_expect_tx(&sm.full[t], CT * sizeof(float4));
      tma_load_1d(ring[t], tile_src(a, r + (int64_t)t * K), CT * sizeof(float4), &sm.full[t]);
    }
  }
  // warm thresholds of this rank's share of the queries, exchanged through DSMEM
  for (int k = tid; k < QPC; k += NT) sm.t0[r * QPC + k] = warm_t0(a, query_of(a, q_base + r * QPC + k));
  if constexpr (K > 1) cg::this_cluster().sync();
  else __syncthreads();
  stamp(a, 1);

  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  const float r2_in = __uint_as_float(__float_as_uint(r2) - 1u);  // largest float < r2 (r2 > 0)
  float2 pxy[Q];  // (x, y) of each query as an aligned register pair (FADD2 operand)
  float pz[Q], lim[Q];
  int gq[Q];  // global index of each query (n < 2^31)
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int ql = warp * 32 * Q + q * 32 + lane;  // query slot within the block
    const int64_t qi = query_of(a, q_base + ql);
    gq[q] = (int)(a.lo + qi);
    float4 me = qi < a.nloc ? __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi))
                            : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
    pxy[q] = make_float2(me.x, me.y);
    pz[q] = me.z;
  }
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int ql = warp * 32 * Q + q * 32 + lane;
    float t0;
    if constexpr (K > 1) t0 = *cg::this_cluster().map_shared_rank(&sm.t0[ql], ql / QPC);
    else t0 = sm.t0[ql];
    // inclusive limit: accept d2 <= t0 (ties at t0 kept) and d2 < r2, i.e. d2 <= prev(r2)
    lim[q] = fminf(r2_in, t0);
#pragma unroll
    for (int s = 0; s < 7; ++s) sm.lists[s * QB + ql] = KEY_EMPTY;
  }
  __syncwarp();

  // ------------------------------------------------------------ scan ----
  // Limits are INCLUSIVE (d2 <= lim): candidates arrive in spatial, not index,
  // order, so a candidate tying the held 7th d2 may still win on its index; the
  // exact (d2, index) comparison is insert7's.  Fast test per U candidates: min
  // over all Q*U distances (an FMNMX3 tree) against limc = max_q lim[q] --
  // conservative, so it never misses a pair that passes its own query's limit;
  // the exact per-query test, the self exclusion and the insertion run only in
  // the rare warp-uniform slow path.
  float limc = fmaxf(fmaxf(lim[0], lim[1]), fmaxf(lim[2], lim[3]));
  unsigned slow_groups = 0;
  for (int t = 0; t < nt; ++t) {
    const int s = t % STAGES;
    mbar_wait(&sm.full[s], (uint32_t)((t / STAGES) & 1));
    const float4* tile = ring[s];
    const int jb = (int)((r + (int64_t)t * K) * CT);
#pragma unroll 2
    for (int c = 0; c < CT; c += U) {
      float4 cc[U];
#pragma unroll
      for (int u = 0; u < U; ++u) cc[u] = tile[c + u];
      // d2 = ((dx*dx) + (dy*dy)) + (dz*dz), every op rounded (Appendix A): (dx, dy)
      // and their squares as packed FADD2 / FMUL2 on the query's (x, y) pair and
      // the candidate's (x, y) pair (both aligned register pairs), dz scalar, the
      // sums scalar FADD (a packed add would be contracted into FFMA2 by ptxas).
      // Same bits as dist2(); 6 issue slots for 8 FP32 lane-ops.
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
      if (__any_sync(0xffffffffu, m <= limc)) {  // rare, warp-uniform
        ++slow_groups;
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            const int j = jb + c + u;
            if (d[q][u] <= lim[q] && j != gq[q])
              lim[q] = fminf(lim[q], insert_list(sm.lists, QB, warp * 32 * Q + q * 32 + lane, d[q][u], j));
          }
        limc = fmaxf(fmaxf(lim[0], lim[1]), fmaxf(lim[2], lim[3]));
      }
    }
    // every thread releases the stage after its own reads of it (release
    // semantics per thread: the stage's reuse by the bulk copy is ordered after
    // all of them without relying on __syncwarp; this kernel runs on cold steps only)
    mbar_arrive(&sm.empty[s]);
    // refill this stage with tile t + STAGES once every thread has released it
    if (tid == 0 && t + STAGES < nt) {
      mbar_wait(&sm.empty[s], (uint32_t)((t / STAGES) & 1));
      fence_proxy_async_smem();
      mbar_arrive_expect_tx(&sm.full[s], CT * sizeof(float4));
      tma_load_1d(ring[s], tile_src(a, r + (int64_t)(t + STAGES) * K), CT * sizeof(float4), &sm.full[s]);
    }
  }

  stamp(a, 2);
  if (a.stats && lane == 0) {
    atomicAdd(a.stats, (unsigned long long)slow_groups);
    atomicAdd(a.stats + 1, (unsigned long long)nt * (CT / U));
  }

  // ------------------------------------------- split merge + epilogue ----
  key_t* lists = sm.lists;  // [7][QB]
  if constexpr (K == 1) {
    __syncwarp();
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const int ql = warp * 32 * Q + q * 32 + lane;
      key_t A[7];
#pragma unroll
      for (int s = 0; s < 7; ++s) A[s] = lists[s * QB + ql];
      finish_query(a, query_of(a, q_base + ql), A);
    }
  } else {
    cg::cluster_group cl = cg::this_cluster();
    cl.sync();  // all partial lists of the cluster are in shared memory
    stamp(a, 3);
    if constexpr (QPC >= NT) {
      // K <= Q: each thread owns QPC / NT queries and merges all K lists of each.
      constexpr int QPT = QPC / NT;
      key_t A[QPT][7];
#pragma unroll
      for (int w = 0; w < QPT; ++w) {
        const int my_q = r * QPC + w * NT + tid;
#pragma unroll
        for (int src = 0; src < K; ++src) {
          const key_t* l = cl.map_shared_rank(lists, src);
          key_t B[7];
#pragma unroll
          for (int s = 0; s < 7; ++s) B[s] = l[s * QB + my_q];
          if (src == 0) {
#pragma unroll
            for (int s = 0; s < 7; ++s) A[w][s] = B[s];
          } else {
            merge7(A[w], B);
          }
        }
      }
      cluster_arrive();  // done reading peers' shared memory
      stamp(a, 4);
#pragma unroll
      for (int w = 0; w < QPT; ++w) finish_query(a, query_of(a, q_base + r * QPC + w * NT + tid), A[w]);
      stamp(a, 5);
      cluster_wait();
      stamp(a, 6);
    } else {
      // K > Q: LP = K / Q lanes per query; each lane merges Q of the K lists,
      // then a shuffle butterfly over the LP lanes.
      constexpr int LP = K / Q;
      const int my_q = r * QPC + tid / LP;
      const int sub = tid % LP;
      key_t A[7];
#pragma unroll
      for (int i = 0; i < Q; ++i) {
        const key_t* l = cl.map_shared_rank(lists, sub + i * LP);
        key_t B[7];
#pragma unroll
        for (int s = 0; s < 7; ++s) B[s] = l[s * QB + my_q];
        if (i == 0) {
#pragma unroll
          for (int s = 0; s < 7; ++s) A[s] = B[s];
        } else {
          merge7(A, B);
        }
      }
      cluster_arrive();  // done reading peers' shared memory
      stamp(a, 4);
#pragma unroll
      for (int w = 1; w < LP; w <<= 1) {
        key_t B[7];
#pragma unroll
        for (int s = 0; s < 7; ++s) B[s] = __shfl_xor_sync(0xffffffffu, A[s], w);
        merge7(A, B);
      }
      if (sub == 0) finish_query(a, query_of(a, q_base + my_q), A);
      stamp(a, 5);
      cluster_wait();
      stamp(a, 6);
    }
  }
}

// ---------------------------------------------------------------- launch ----
// Kernel table [NT 64/128][K 1,2,4,8,16][U 4/8] with lazily queried occupancy.
typedef void (*FusedFn)(StepArgs, int64_t);
struct KEntry {
  FusedFn fn;
  int nt, k;
  int rmax;  // max resident CTAs per SM without padding
  int static_smem;
  bool ready;
};

template <int NT, int U>
void fill_row(KEntry (&tab)[2][5][2], int ni, int ui) {
  const FusedFn fns[5] = {k_fused<NT, 1, U>, k_fused<NT, 2, U>, k_fused<NT, 4, U>, k_fused<NT, 8, U>,
                          k_fused<NT, 16, U>};
  for (int i = 0; i < 5; ++i) tab[ni][i][ui] = KEntry{fns[i], NT, 1 << i, 0, 0, false};
}

KEntry& entry(int ni, int ki, int ui) {
  static KEntry tab[2][5][2];
  static bool init = false;
  if (!init) {
    fill_row<64, 4>(tab, 0, 0);
    fill_row<64, 8>(tab, 0, 1);
    fill_row<128, 4>(tab, 1, 0);
    fill_row<128, 8>(tab, 1, 1);
    init = true;
  }
  KEntry& e = tab[ni][ki][ui];
  if (!e.ready) {
    // all of the SM's unified memory goes to shared memory (the kernel relies on L1
    // only for a few gathers), so residency is governed by the padding below
    cudaFuncSetAttribute(e.fn, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e.k > 8) cudaFuncSetAttribute(e.fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaFuncAttributes at{};
    cudaFuncGetAttributes(&at, e.fn);
    e.static_smem = (int)at.sharedSizeBytes;
    int r = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&r, e.fn, e.nt, 0);
    e.rmax = r > 0 ? r : 1;
    e.ready = true;
  }
  return e;
}

// Dynamic shared memory padding that caps residency at `cap` CTAs per SM, so a
// single wave of C CTAs spreads ceil(C / SMs) per SM instead of the cluster
// scheduler piling its maximum onto some SMs (measured: 2x scan-time spread).
int pad_for_cap(KEntry& e, int cap) {
  if (cap >= e.rmax) return 0;
  int dev = 0, optin = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  int lo = 0, hi = optin - e.static_smem, r = 0;
  cudaFuncSetAttribute(e.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, hi);
  while (lo < hi) {  // smallest padding with occupancy <= cap
    const int mid = (lo + hi) / 2;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&r, e.fn, e.nt, mid);
    if (r <= cap) hi = mid;
    else lo = mid + 1;
  }
  return lo;
}

// Occupancy-aware launch plan.  For CTA size NT (64 or 128) and cluster size K
// the grid is C = K * ceil(n_local / (NT * Q)) CTAs on S SMs:
//   one wave (ceil(C/S) <= rmax): residency capped at r = ceil(C/S) (padding),
//             balance (C/S) / r;   else r = rmax, balance waves / ceil(waves);
//   x loop efficiency at r * NT / 32 warps per SM (tools/probe_loop.cu, packed)
//   x per-CTA fixed cost (ring fill, merge, epilogue ~ 512 candidates).
// Ties go to the smaller NT, then the smaller K.
double loop_eff(double w) {
  static const double W[] = {4, 8, 12, 16, 24, 32, 64};
  static const double E[] = {0.40, 0.66, 0.74, 0.78, 0.80, 0.81, 0.81};
  if (w <= W[0]) return E[0] * w / W[0];
  for (int i = 1; i < 7; ++i)
    if (w <= W[i]) return E[i - 1] + (E[i] - E[i - 1]) * (w - W[i - 1]) / (W[i] - W[i - 1]);
  return E[6];
}

struct Plan {
  int ni, ki, cap;
};

Plan plan_launch(int64_t total_candidates, int64_t nloc, int sm_count, int forced_k, int ui) {
  const int64_t tiles = total_candidates / CT;
  Plan best{1, 0, 1};
  double best_score = -1.0;
  for (int ni = 0; ni < 2; ++ni) {
    const int nt = ni == 0 ? 64 : 128;
    const int64_t nqb = (nloc + nt * Q - 1) / (nt * Q);
    for (int ki = 0; ki < 5; ++ki) {
      const int K = 1 << ki;
      if (forced_k && K != forced_k) continue;
      if (K > 1 && tiles / K < 1) break;
      KEntry& e = entry(ni, ki, ui);
      const double C = (double)(nqb * K), S = (double)sm_count;
      const int per_sm = (int)std::ceil(C / S);
      double balance;
      int r;
      if (per_sm <= e.rmax) {
        r = per_sm;
        balance = (C / S) / per_sm;
      } else {
        r = e.rmax;
        const double waves = C / (S * r);
        balance = waves / std::ceil(waves);
      }
      const double cand = (double)total_candidates / K;
      const double score = balance * loop_eff(r * nt / 32.0) * cand / (cand + 512.0);
      if (score > best_score * (1.0 + 1e-6)) {
        best_score = score;
        best = Plan{ni, ki, r};
      }
    }
  }
  return best;
}

}  // namespace

int fused_auto_cluster(int64_t total_candidates, int64_t nloc, int sm_count) {
  return 1 << plan_launch(total_candidates, nloc, sm_count, 0, 0).ki;
}

cudaError_t launch_fused(const StepArgs& a, int cluster, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  const int64_t tiles = (int64_t)a.world * a.m / CT;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int ui = a.vote_u == 8 ? 1 : 0;
  const Plan p = plan_launch(tiles * CT, a.nloc, sms, cluster, ui);
  KEntry& e = entry(p.ni, p.ki, ui);
  // Residency caps fight the cluster scheduler (whole clusters per GPC), so the
  // cluster kernel runs uncapped; pad_for_cap is kept for K == 1 grids.
  const int pad = e.k == 1 ? pad_for_cap(e, p.cap) : 0;
  const int64_t nqb = (a.nloc + e.nt * Q - 1) / (e.nt * Q);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(nqb * e.k));
  cfg.blockDim = dim3(e.nt);
  cfg.dynamicSmemBytes = pad;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = e.k;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, e.fn, a, tiles);
}

}  // namespace boids
