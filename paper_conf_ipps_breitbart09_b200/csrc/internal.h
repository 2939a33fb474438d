// internal.h -- private declarations shared by the CUDA translation units of libboids.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "boids.h"

namespace boids {

constexpr int TILE = 256;  // slice granularity (agents); every slice m is a multiple

// Device view of the agent state for one step.  Layout:
//   full: world segments of 2*m float4; segment g = [pos4(m) | fwd4(m)] of agents
//         [g*m, (g+1)*m); pos4 = (x, y, z, 0), fwd4 = (x, y, z, speed); agents
//         >= n are phantoms with NaN positions (never within any radius).
//   out:  this rank's new [pos4(m) | fwd4(m)].
//   up4, side4: this rank's local frames (read and written by the owner only).
//   nbr (m x 7 int32), cnt (m int32): this rank's neighbour lists (last step).
// Uniform grid for binning (k_bin.cu): cells of size h from lo, dim cells per axis.
struct BinGrid {
  float lo[3];
  float h, inv_h;
  int dim[3];
  int cells;
  int morton;  // 1: cell id = Morton code (dim must be a power of two), 0: row-major
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
  unsigned long long* phase;  // diagnostics: per-CTA %globaltimer stamps [grid][8], nullptr = off
  float dt;
  boids_params p;
};

__host__ __device__ inline const float4* pos_of(const float4* full, int64_t m, int64_t j) {
  return full + (j / m) * 2 * m + (j % m);
}
__host__ __device__ inline const float4* fwd_of(const float4* full, int64_t m, int64_t j) {
  return full + (j / m) * 2 * m + m + (j % m);
}

// launchers (return the cudaError_t of the launch)
cudaError_t launch_init(float4* out, float4* up4, float4* side4, int64_t m, int64_t lo,
                        int64_t nloc, const boids_params& p, uint64_t seed, cudaStream_t s);
cudaError_t launch_fill_phantoms(float4* seg_base, int64_t m, int64_t nloc, int64_t segments,
                                 cudaStream_t s);
cudaError_t launch_bin(const float4* full, int64_t m, int64_t j0, int64_t count, const BinGrid& g,
                       int2* cellrank, int* cnt, int* start, float4* spos, int* perm, int perm_base,
                       cudaStream_t s, int* launches);
BinGrid make_locality_grid(int64_t n, const boids_params& p);
cudaError_t launch_fill_nan(float4* p, int64_t count, cudaStream_t s);
cudaError_t launch_search_simple(const StepArgs& a, cudaStream_t s);
cudaError_t launch_update(const StepArgs& a, cudaStream_t s);
cudaError_t launch_fused(const StepArgs& a, int cluster, cudaStream_t s);
int fused_auto_cluster(int64_t n_pad_total, int64_t nloc, int sm_count);

}  // namespace boids
