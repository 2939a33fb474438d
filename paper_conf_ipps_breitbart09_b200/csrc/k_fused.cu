// k_fused.cu -- the fused Boids step for sm_100a: brute-force 7-NN search +
// split merge + steering + modification in ONE kernel per step.
//
// Thesis lineage (prior art, not the blueprint): version 2's shared-memory
// position cache (Listing 6.2), version 4's recompute-not-cache
// (P:493), version 5's device-resident modification.  What is new:
//
//  * Work unit = (query block of QB = 256 agents, candidate chunk).  A thread
//    block cluster of K CTAs (K in {1,2,4,8,16}) shares one query block; CTA r
//    of the cluster scans candidate chunk r of K.  K is chosen so the grid is
//    close to a whole multiple of the SM count (fused_auto_cluster).
//  * Candidate positions are streamed global -> shared memory by the TMA bulk
//    copy engine (cp.async.bulk + mbarrier complete_tx) through a STAGES-deep
//    ring of 256-candidate tiles; all 4 warps read each candidate with a
//    broadcast LDS.128.
//  * Each thread owns Q = 2 queries and keeps two register-resident sorted
//    top-7 lists of (d2, index) keys (64-bit, reading Q4 total order).
//  * Warm threshold: t0 = max d2 to the previous step's 7 neighbours at the
//    current positions is an upper bound on the true 7th key, so only
//    candidates with d2 <= t0 can enter (identical result, far fewer inserts).
//    The per-pair test is one compare against lim = min(r2, next(t0), worst).
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

namespace cg = cooperative_groups;

namespace boids {
namespace {

constexpr int NT = 128;      // threads per CTA (4 warps), all consumers
constexpr int Q = 2;         // queries per thread
constexpr int QB = NT * Q;   // queries per CTA / cluster
constexpr int CT = 256;      // candidates per tile (4 KB)
constexpr int STAGES = 4;    // TMA ring depth
constexpr int U = 4;         // candidates per vote
static_assert(CT % U == 0, "tile");

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "LAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra LAB_WAIT;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void consumer_bar() { asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory"); }

struct __align__(16) Smem {
  float4 tile[STAGES][CT];  // 16 KB candidate ring; reused for the partial lists
  float t0[QB];             // warm thresholds of this CTA's share of the queries
  uint64_t full[STAGES];
  uint64_t empty[STAGES];
};
static_assert(sizeof(key_t) * 7 * QB <= sizeof(float4) * STAGES * CT, "lists fit in the ring");

__device__ __forceinline__ const float4* tile_src(const StepArgs& a, int64_t tile) {
  return pos_of(a.full, a.m, tile * CT);  // m % CT == 0: a tile never straddles a slice
}

// t0 for local query ql (returns +inf when there is no valid warm list).
__device__ __forceinline__ float warm_t0(const StepArgs& a, int64_t ql) {
  if (!a.warm || ql >= a.nloc) return __int_as_float(0x7f800000);
  if (a.cnt[ql] < 7) return __int_as_float(0x7f800000);
  float4 me = __ldg(pos_of(a.full, a.m, a.lo + ql));
  float t = 0.f;
#pragma unroll
  for (int k = 0; k < 7; ++k) {
    int j = a.nbr[ql * 7 + k];
    t = fmaxf(t, dist2(me.x, me.y, me.z, __ldg(pos_of(a.full, a.m, j))));
  }
  return t;
}

template <int K>
__global__ void __launch_bounds__(NT) k_fused(StepArgs a, int64_t tiles_total) {
  __shared__ Smem sm;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int r = K > 1 ? (int)cg::this_cluster().block_rank() : 0;
  const int64_t qb = blockIdx.x / K;
  const int64_t q_base = qb * QB;  // local index of this cluster's first query
  constexpr int QPC = QB / K;      // queries per cluster rank (merge + epilogue owner)

  const int64_t t_lo = tiles_total * r / K, t_hi = tiles_total * (r + 1) / K;
  const int nt = (int)(t_hi - t_lo);

  if (tid == 0) {
#pragma unroll
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], NT / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  // prologue: fill the ring
  if (tid == 0) {
    for (int t = 0; t < STAGES && t < nt; ++t) {
      mbar_arrive_expect_tx(&sm.full[t], CT * sizeof(float4));
      tma_load_1d(sm.tile[t], tile_src(a, t_lo + t), CT * sizeof(float4), &sm.full[t]);
    }
  }

  // warm thresholds of this rank's share of the queries
  for (int k = tid; k < QPC; k += NT) sm.t0[r * QPC + k] = warm_t0(a, q_base + r * QPC + k);
  if constexpr (K > 1) cg::this_cluster().sync();
  else __syncthreads();

  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  float px[Q], py[Q], pz[Q], lim[Q];
  int64_t gq[Q];
  key_t L[Q][7];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    int ql = warp * 64 + q * 32 + lane;  // query slot within the block
    int64_t qi = q_base + ql;
    gq[q] = a.lo + qi;
    float4 me = qi < a.nloc ? __ldg(pos_of(a.full, a.m, a.lo + qi))
                            : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
    px[q] = me.x;
    py[q] = me.y;
    pz[q] = me.z;
    float t0;
    if constexpr (K > 1) t0 = *cg::this_cluster().map_shared_rank(&sm.t0[ql], ql / QPC);
    else t0 = sm.t0[ql];
    // accept d2 <= t0 (inclusive, so ties at t0 are kept) and d2 < r2
    float nt0 = t0 < __int_as_float(0x7f800000) ? __uint_as_float(__float_as_uint(t0) + 1u) : t0;
    lim[q] = fminf(r2, nt0);
#pragma unroll
    for (int s = 0; s < 7; ++s) L[q][s] = KEY_EMPTY;
  }

  // ------------------------------------------------------------ scan ----
  for (int t = 0; t < nt; ++t) {
    const int s = t % STAGES;
    mbar_wait(&sm.full[s], (uint32_t)((t / STAGES) & 1));
    const float4* tile = sm.tile[s];
    const int64_t jb = (t_lo + t) * CT;
#pragma unroll 2
    for (int c = 0; c < CT; c += U) {
      float4 cc[U];
#pragma unroll
      for (int u = 0; u < U; ++u) cc[u] = tile[c + u];
      float d[Q][U];
      bool hit = false;
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < Q; ++q) {
          d[q][u] = dist2(px[q], py[q], pz[q], cc[u]);
          hit |= d[q][u] < lim[q];
        }
      if (__any_sync(0xffffffffu, hit)) {
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            int64_t j = jb + c + u;
            if (d[q][u] < lim[q] && j != gq[q]) {
              insert7(L[q], make_key(d[q][u], (int)j));
              lim[q] = fminf(lim[q], key_d2(L[q][6]));
            }
          }
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.empty[s]);
    // refill this stage with tile t + STAGES once every warp has released it
    if (tid == 0 && t + STAGES < nt) {
      mbar_wait(&sm.empty[s], (uint32_t)((t / STAGES) & 1));
      mbar_arrive_expect_tx(&sm.full[s], CT * sizeof(float4));
      tma_load_1d(sm.tile[s], tile_src(a, t_lo + t + STAGES), CT * sizeof(float4), &sm.full[s]);
    }
  }

  // ----------------------------------------------------- split merge ----
  if constexpr (K == 1) {
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      int ql = warp * 64 + q * 32 + lane;
      int64_t qi = q_base + ql;
      if (qi >= a.nloc) continue;
      int nb[7], cnt = 0;
#pragma unroll
      for (int s = 0; s < 7; ++s) {
        key_t k = L[q][s];
        nb[s] = k == KEY_EMPTY ? -1 : key_idx(k);
        cnt += k == KEY_EMPTY ? 0 : 1;
      }
#pragma unroll
      for (int s = 0; s < 7; ++s) a.nbr[qi * 7 + s] = nb[s];
      a.cnt[qi] = cnt;
      float4 p4 = __ldg(pos_of(a.full, a.m, a.lo + qi));
      float4 f4 = __ldg(fwd_of(a.full, a.m, a.lo + qi));
      V3 F = steer_agent(a, v3(p4), v3(f4), nb, cnt);
      modify_agent(a, qi, v3(p4), f4, F);
    }
  } else {
    key_t* lists = reinterpret_cast<key_t*>(&sm.tile[0][0]);  // [7][QB], k-major
    consumer_bar();  // every warp is done reading the ring
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      int ql = warp * 64 + q * 32 + lane;
#pragma unroll
      for (int s = 0; s < 7; ++s) lists[s * QB + ql] = L[q][s];
    }
    cg::cluster_group cl = cg::this_cluster();
    cl.sync();  // all partial lists of the cluster are in shared memory
    // LP lanes per query; each lane merges 2 of the K source lists, then a
    // butterfly over the LP lanes.  K == 2 * LP.
    constexpr int LP = K / 2;
    const int my_q = r * QPC + tid / LP;  // query slot within the cluster block
    const int sub = tid % LP;
    key_t A[7], B[7];
    {
      const key_t* la = cl.map_shared_rank(lists, sub);
      const key_t* lb = cl.map_shared_rank(lists, sub + LP);
#pragma unroll
      for (int s = 0; s < 7; ++s) {
        A[s] = la[s * QB + my_q];
        B[s] = lb[s * QB + my_q];
      }
    }
    cl.sync();  // no CTA reads a peer's shared memory after this point
    merge7(A, B);
#pragma unroll
    for (int w = 1; w < LP; w <<= 1) {
#pragma unroll
      for (int s = 0; s < 7; ++s) B[s] = __shfl_xor_sync(0xffffffffu, A[s], w);
      merge7(A, B);
    }
    const int64_t qi = q_base + my_q;
    if (sub == 0 && qi < a.nloc) {
      int nb[7], cnt = 0;
#pragma unroll
      for (int s = 0; s < 7; ++s) {
        nb[s] = A[s] == KEY_EMPTY ? -1 : key_idx(A[s]);
        cnt += A[s] == KEY_EMPTY ? 0 : 1;
      }
#pragma unroll
      for (int s = 0; s < 7; ++s) a.nbr[qi * 7 + s] = nb[s];
      a.cnt[qi] = cnt;
      float4 p4 = __ldg(pos_of(a.full, a.m, a.lo + qi));
      float4 f4 = __ldg(fwd_of(a.full, a.m, a.lo + qi));
      V3 F = steer_agent(a, v3(p4), v3(f4), nb, cnt);
      modify_agent(a, qi, v3(p4), f4, F);
    }
  }
}

template <int K>
cudaError_t launch_k(const StepArgs& a, int64_t tiles, int64_t nqb, cudaStream_t s) {
  auto kern = k_fused<K>;
  if (K > 8) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(nqb * K));
  cfg.blockDim = dim3(NT);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = K;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, a, tiles);
}

}  // namespace

// Choose the cluster size K: the grid (K * query blocks) should fill the SMs as
// evenly as possible (efficiency (C/S) / ceil(C/S)), with at least 2 candidate
// tiles per CTA; ties go to the smaller K (less merge work).
int fused_auto_cluster(int64_t total_candidates, int64_t nloc, int sm_count) {
  int64_t nqb = (nloc + QB - 1) / QB;
  int64_t tiles = total_candidates / CT;
  int best = 1;
  double best_eff = -1.0;
  for (int K = 1; K <= 16; K *= 2) {
    if (K > 1 && tiles / K < 2) break;
    double C = (double)(nqb * K), S = (double)sm_count;
    double eff = (C / S) / std::ceil(C / S);
    if (C < 4 * S) eff *= C / (4 * S);  // too few warps per SM to hide latency
    if (eff > best_eff + 1e-9) {
      best_eff = eff;
      best = K;
    }
  }
  return best;
}

cudaError_t launch_fused(const StepArgs& a, int cluster, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  int64_t total = (int64_t)a.world * a.m;
  int64_t tiles = total / CT;
  int64_t nqb = (a.nloc + QB - 1) / QB;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  int K = cluster > 0 ? cluster : fused_auto_cluster(total, a.nloc, sms);
  while (K > 1 && tiles / K < 1) K /= 2;
  switch (K) {
    case 1: return launch_k<1>(a, tiles, nqb, s);
    case 2: return launch_k<2>(a, tiles, nqb, s);
    case 4: return launch_k<4>(a, tiles, nqb, s);
    case 8: return launch_k<8>(a, tiles, nqb, s);
    default: return launch_k<16>(a, tiles, nqb, s);
  }
}

}  // namespace boids
