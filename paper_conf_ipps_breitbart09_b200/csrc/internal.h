// internal.h -- private declarations shared by the CUDA translation units of libboids.
#pragma once
#include <cstdio>
#include <utility>
#include <cuda_runtime.h>
#include <stdint.h>

#include "boids.h"

namespace boids {

constexpr int TILE = 256;  // slice granularity (agents); every slice m is a multiple
constexpr int HITS = 48;   // warm path: hit-buffer slots per agent (more -> full re-search)
// sym-shards: hit slots per agent per rank segment; the blocks cross ranks in an
// all-to-all of fixed-size pieces, so the cap sets its payload (a segment holds a
// 1/G share of an agent's ~8-12 hits; more in one segment -> full re-search)
constexpr int SS_HITS = 16;
constexpr int HITS_THINK = 128;  // ... in think mode (bounds from lists up to k steps old are looser)
constexpr int PSLOTS = 16; // warm path: partial top-7 lists per unbounded agent

// Device view of the agent state for one step.  Layout:
//   full: world segments of 2*m float4; segment g = [pos4(m) | fwd4(m)] of agents
//         [g*m, (g+1)*m); pos4 = (x, y, z, 0), fwd4 = (x, y, z, speed); agents
//         >= n are phantoms with NaN positions (never within any radius).
//   out:  this rank's new [pos4(m) | fwd4(m)].
//   up4, side4: this rank's local frames (read and written by the owner only).
//   nbr (m x 7 int32), cnt (m int32): this rank's neighbour lists (last step).
// Segmented addressing: agent j lives in slice g = j / m at full[g*2m + j - g*m]
// (pos4) and full[g*2m + m + j - g*m] (fwd4), i.e. at j + g*m and j + (g+1)*m.
// The division by the runtime slice m is a precomputed magic-number multiply
// (Granlund-Montgomery, valid for 32-bit j; checked against j / m for the slice
// sizes in use), avoiding a 64-bit division subroutine per gather.
struct SliceDiv {
  uint32_t mult;
  int32_t shift;  // l = ceil(log2 m) >= 8 (m is a multiple of 256)
  int32_t one;    // world == 1: every agent is in slice 0
  int32_t world;  // slices (BOIDS_CHECKS builds bound agent indices by world x m)
};

// Device-side bounds checks of the checks build (build.py: BOIDS_CHECKS=1, used
// in place of compute-sanitizer where the pool does not run it): a failed
// check prints its place and traps, so the launch -- and the test -- fails.
#if defined(BOIDS_CHECKS) && defined(__CUDA_ARCH__)
#define BOIDS_CHECK(c)                                                         \
  do {                                                                         \
    if (!(c)) {                                                                \
      printf("BOIDS_CHECK failed %s:%d: %s\n", __FILE__, __LINE__, #c);       \
      __trap();                                                                \
    }                                                                          \
  } while (0)
#else
#define BOIDS_CHECK(c) ((void)0)
#endif
inline SliceDiv make_slice_div(int64_t m, int32_t world) {
  SliceDiv s{};
  s.world = world;
  int l = 0;
  while ((1ull << l) < (unsigned long long)m) ++l;
  s.mult = (uint32_t)((((unsigned long long)1 << 32) * ((1ull << l) - (unsigned long long)m)) / (unsigned long long)m + 1);
  s.shift = l;
  s.one = world == 1;
  return s;
}
__host__ __device__ inline int64_t slice_of(const SliceDiv& s, int64_t j) {
  if (s.one) return 0;
#ifdef __CUDA_ARCH__
  const uint32_t n = (uint32_t)j, t = __umulhi(s.mult, n);
  return (int64_t)((t + ((n - t) >> 1)) >> (s.shift - 1));
#else
  const uint32_t n = (uint32_t)j, t = (uint32_t)(((unsigned long long)s.mult * n) >> 32);
  return (int64_t)((t + ((n - t) >> 1)) >> (s.shift - 1));
#endif
}
__host__ __device__ inline const float4* pos_of(const float4* full, int64_t m, const SliceDiv& s, int64_t j) {
  BOIDS_CHECK(j >= 0 && j < (int64_t)s.world * m);
  return full + j + slice_of(s, j) * m;
}
__host__ __device__ inline const float4* fwd_of(const float4* full, int64_t m, const SliceDiv& s, int64_t j) {
  BOIDS_CHECK(j >= 0 && j < (int64_t)s.world * m);
  return full + j + (slice_of(s, j) + 1) * m;
}

// Uniform grid for binning (k_bin.cu): cells of size h from lo, dim cells per axis.
struct BinGrid {
  float lo[3];
  float h, inv_h;
  int dim[3];
  int cells;
  int morton;  // 1: cell id = Morton code (dim must be a power of two), 0: row-major
  int reach;   // search grid: cells per axis an agent closer than r can be away (h * reach >= r)
  int block;   // > 0: a grid of BLOCKS of block^3 cells of the fine grid (lo, h, fdim): the block of a
               // position is its fine cell coordinate / block (so it agrees with the fine cell exactly);
               // dim[] then counts blocks per axis
  int fdim[3];  // fine cells per axis (block > 0)
};

struct StepArgs {
  const float4* full;
  float4* out;
  float4* up4;
  float4* side4;
  float4* force4;  // nullptr = do not record steering
  int32_t* nbr;
  int32_t* cnt;
  int64_t n;       // total agents
  int64_t m;       // slice size
  SliceDiv sdiv;   // j -> slice of agent j
  int64_t lo;      // first owned agent
  int64_t nloc;    // owned agents (hi - lo)
  int32_t world;
  int32_t warm;    // 1: nbr/cnt hold the previous step's lists for these agents
  // brute-force candidate stream in spatial (Morton) order: x, y, z, original index
  // as int bits in .w; ncand is a multiple of 256 (NaN-padded).  nullptr = use full.
  const float4* cand;
  int64_t ncand;
  const int32_t* qperm;  // local queries in spatial order (local indices); nullptr = identity
  unsigned long long* stats;  // [0] vote groups that took the insertion path, [1] all vote groups
  int32_t vote_u;             // candidates per warp vote in the fused kernel (4 or 8)
  unsigned long long* hits;   // warm path: [nloc][hits_cap] passing (d2, index) keys
  int32_t hits_cap;           // HITS, or HITS_THINK in think mode
  int32_t* hitcnt;            // warm path: [nloc] number of passing keys (zero between steps)
  int32_t* nbr8;              // [nloc] 8th nearest agent of the last step, or -1 (warm-bound seed)
  unsigned long long* partial;  // warm path: [nloc][PSLOTS][7] partial top-7 lists (unbounded agents)
  int32_t* pcnt;              // warm path: [nloc] partial lists written
  float* qlim;                // warm path: [nloc] inclusive search limit min(prev(r2), t0) (k_bound)
  // think frequency: agent j thinks at step step_t iff (j + step_t) % think_k == 0
  int32_t think_k;            // 1 = every agent thinks every step
  int32_t store_only;         // search epilogues: 1 store F in fstore instead of modifying, 2 both
  int64_t step_t;
  float4* fstore;             // [nloc] last steering vector of each agent
  const int32_t* qcount;      // device-side number of query slots (qperm entries), nullptr = nloc
  int64_t nq;                 // kernel-local copy of the number of query slots
  unsigned char* routed;      // [nloc] think mode: 1 = searched by k_fused this step (k_select skips);
                              // k_sym steps: 1 = routed to k_route by k_sym_prep
  int32_t* rlist;             // warm steps: agents finished by k_route (hit-buffer overflow, routed);
  int32_t* rcount;            // their number (zeroed before the step).  nullptr = warp re-search in k_select
  unsigned long long* rpart;  // k_route: per routed agent, the top-8 of each candidate part [m][16][8]
  int32_t* rbcount;           // k_route: parts finished per routed agent (zero between steps) [m]
  unsigned long long* phase;  // diagnostics: per-CTA %globaltimer stamps [grid][8], nullptr = off
  float4* acc4;               // [m] steer_mode 1: smoothed accelerations (nullptr otherwise)
  BinGrid loc;                // locality (Morton) grid of the last query sort ...
  const int32_t* lstart;      // ... its cell starts in qperm (nullptr = none yet)
  float dt;
  boids_params p;
};

// Grid-mode inputs of k_grid (k_grid.cu), produced by the binning passes.
struct GridArgs {
  const float4* spos;     // all agents sorted by search cell: x, y, z, original index (int bits)
  const int* cstart;      // [cells + 1] start of each cell in spos
  const int* qstart;      // [cells + 1] start of each cell in qperm (owned agents)
  const int* qperm;       // owned agents (local indices) sorted by cell
  const int4* items;      // work items (first query slot, count, first cell, x span) (k_bin_scan)
  const int* nitems;      // their number
  int* counter;           // work-queue counter (reset by the binning scan)
  int* flist;             // queries routed to k_grid_far (limit beyond the adjacent cells)
  int* fcount;            // their number (zeroed before k_grid)
  float* flim;            // their search limits (inclusive d2 bound: min of r2, warm bound, cell bound)
  BinGrid grid;           // the fine search grid of the candidates (cstart)
  BinGrid qgrid;          // its blocks: the queries' binning (qstart, items; item.z = block index)
};

// Does global agent g think at step t (think frequency k)?
__host__ __device__ inline bool thinks(int64_t g, int64_t t, int32_t k) { return k <= 1 || (g + t) % k == 0; }

// Every kernel of a step asks for the same L1/shared-memory split (the maximum
// shared-memory carveout the TMA-ring kernels need), so consecutive kernels do
// not make the SMs drain and reconfigure the split between launches.  Once per
// kernel; BOIDS_CARVEOUT=<percent> overrides, -1 leaves the driver default.
int carveout_pct();
#define BOIDS_PREFER_SMEM(kern)                                                                  \
  do {                                                                                           \
    static const bool boids_once_ = [] {                                                         \
      if (carveout_pct() >= 0)                                                                   \
        cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, carveout_pct()); \
      return true;                                                                               \
    }();                                                                                         \
    (void)boids_once_;                                                                           \
  } while (0)

// Programmatic dependent launch along a warm step's kernel chain (k_bound ->
// k_scan / k_sym_prep -> k_sym -> k_select1 -> k_route): each of these kernels
// lets its dependent be scheduled at once (pdl_trigger) and waits for its
// predecessor's completion and memory (pdl_wait) before its first access to
// step data, so launch latency and CTA rasterisation overlap the predecessor's
// tail.  pdl_wait is a no-op for a kernel launched without the attribute.
// BOIDS_PDL=0 turns the attribute off (diagnostics).
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" :::); }
bool pdl_enabled();
bool pdl_env(const char* name);  // diagnostics: getenv(name) != "0"
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args&&... args) {
  return launch_pdl_if(true, kern, grid, block, smem, s, std::forward<Args>(args)...);
}
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl_if(bool use, void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                          Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = use && pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// launchers (return the cudaError_t of the launch)
cudaError_t launch_init(float4* out, float4* up4, float4* side4, int64_t m, int64_t lo,
                        int64_t nloc, const boids_params& p, uint64_t seed, cudaStream_t s);
cudaError_t launch_fill_phantoms(float4* seg_base, int64_t m, int64_t nloc, int64_t segments,
                                 cudaStream_t s);
cudaError_t launch_bin(const float4* full, int64_t m, const SliceDiv& sd, int64_t j0, int64_t count, const BinGrid& g,
                       int2* cellrank, int* cnt, int* start, float4* spos, int* perm, int perm_base,
                       cudaStream_t s, int* launches, int4* items = nullptr, int* nitems = nullptr, int chunk = 1,
                       int* counter = nullptr, int think_k = 1, int64_t think_t = 0,
                       int* rowbuf = nullptr,  // [2 * rows] scratch: large grids scan on many CTAs
                       const unsigned char* own = nullptr);  // spatial shards: bin only agents with own[k]
BinGrid make_locality_grid(int64_t n, const boids_params& p);
BinGrid make_search_grid(const boids_params& p);
BinGrid make_query_grid(const BinGrid& search);  // blocks of the search grid: the grid search's work items
BinGrid make_slab_grid(const BinGrid& search, int z0, int z1);  // layers [z0, z1) of a search grid
cudaError_t launch_fill_nan(float4* p, int64_t count, cudaStream_t s);
cudaError_t launch_apply(const StepArgs& a, cudaStream_t s);
cudaError_t launch_pack_draw(const float4* local, int64_t m, const float4* up4, const float4* side4, int64_t k,
                             float4* draw, cudaStream_t s);
cudaError_t launch_state_in(const float* stage, bool has_side, int64_t k, float4* local, int64_t m, float4* up4,
                            float4* side4, cudaStream_t s);
cudaError_t launch_order_check(const float* pos3, const int32_t* qperm, int64_t k, float r2, int* out,
                               cudaStream_t s);
cudaError_t launch_state_out(const float4* local, int64_t m, const float4* up4, const float4* side4, int64_t k,
                             float* stage, cudaStream_t s);
cudaError_t launch_think_compact(const StepArgs& a, const int32_t* qperm, int32_t* cold, int32_t* ncold,
                                 int32_t* warm, int32_t* nwarm, cudaStream_t s);
cudaError_t launch_search_simple(const StepArgs& a, cudaStream_t s);
cudaError_t launch_update(const StepArgs& a, cudaStream_t s);
cudaError_t launch_fused(const StepArgs& a, int cluster, cudaStream_t s);
cudaError_t launch_warm_scan(const StepArgs& a, cudaStream_t s);
cudaError_t launch_grid(const StepArgs& a, const GridArgs& g, cudaStream_t s);
cudaError_t launch_grid_far(const StepArgs& a, const GridArgs& g, cudaStream_t s);
int grid_chunk(int64_t nq);
// k_small.cu: the whole warm brute-force step in one kernel for single-rank handles with n < small_max()
int small_max();
cudaError_t launch_small(const StepArgs& a, cudaStream_t s);  // queries per grid work item for nq queries
// pdl: launch k_select1 as a programmatic dependent of the scan.  Measured: a
// gain after k_scan (C1 30 -> 25 us/step), a loss after k_sym (C3 97 -> 121).
cudaError_t launch_warm_select(const StepArgs& a, cudaStream_t s, bool pdl = true);
int64_t sym_capacity(int64_t nloc);
// k_sym work-split feedback record: [0] grid, [1] items, then per CTA j
// [2 + 3j] L0, [3 + 3j] L1, [4 + 3j] SM cycles the CTA took.
constexpr int SYM_FB_MAX_CTAS = 1024;
constexpr int SYM_FB_LEN = 2 + 3 * SYM_FB_MAX_CTAS;
// splits: [SYM_FB_MAX_CTAS + 1] int64 scratch: k_sym_prep writes every k_sym CTA's item range there
cudaError_t launch_sym_scan(const StepArgs& a, float4* sp, int* sidx, const long long* fb_prev, long long* fb_cur,
                            long long* splits, cudaStream_t s,
                            int part = 0);  // part 0: k_sym_prep + k_sym, 1: k_sym_prep, 2: k_sym
cudaError_t launch_route(const StepArgs& a, cudaStream_t s);
// sym-shards (k_sym.cu): the unordered-pair triangle split over index-sharded ranks
cudaError_t launch_ss_lim(const StepArgs& a, float* lim_send, const int* gperm, const int* gstart, int64_t nsorted,
                          cudaStream_t s);
cudaError_t launch_ss_cellsort(int* perm, const int* start, int cells, cudaStream_t s);
cudaError_t launch_ss_search(const StepArgs& a, const int* gperm, int64_t nsorted, const float* lim_full, float4* sp,
                             int* sidx, const long long* fb_prev, long long* fb_cur, long long* splits, int rank,
                             int world, cudaStream_t s);
cudaError_t launch_ss_select(const StepArgs& a, const unsigned long long* recv, const int* rcnt, int world,
                             cudaStream_t s);
int fused_auto_cluster(int64_t n_pad_total, int64_t nloc, int sm_count);
// spatial shards (k_spatial.cu)
int spatial_halo_f4();
int spatial_mig_f4();
cudaError_t launch_zhist(const float4* cur, int64_t n, const BinGrid& g, int* hist, cudaStream_t s);
cudaError_t launch_spatial_init(float4* cur, float4* other, int64_t m, int64_t n, unsigned char* own,
                                const BinGrid& g, const int* zb, int world, int rank, int reach, int* kept,
                                int* nkept, cudaStream_t s);
cudaError_t launch_spatial_pack(float4* cur, float4* prev, int64_t m, int64_t n, unsigned char* own, const float4* up4,
                                const float4* side4, const int32_t* nbr, const int32_t* cnt, const int32_t* nbr8,
                                const float4* acc4, const BinGrid& g, const int* zb, int world, int rank, int reach,
                                float4* halo_out, int64_t cap_h, float4* mig_out, int64_t cap_m, int* counts,
                                int* overflow, const float4* halo_in, int64_t nh_prev, int* kept, int* nkept,
                                int64_t nkept_cap, cudaStream_t s);
cudaError_t launch_spatial_unpack(const float4* halo_in, int64_t nh, const float4* mig_in, int64_t nm, float4* cur,
                                  int64_t m, unsigned char* own, float4* up4, float4* side4, int32_t* nbr,
                                  int32_t* cnt, int32_t* nbr8, float4* acc4, cudaStream_t s);

}  // namespace boids
