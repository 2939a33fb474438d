// k_bin.cu -- device counting sort of agents by spatial cell.
//
// The thesis names spatial data structures as future work for the neighbour
// search and proposes building them on the host; here they are built on
// the device every step in three O(n) passes:
//   bin_count   cell of every agent (clamped into the grid), atomic count per
//               cell; the atomic's return value is the agent's rank in its cell
//   bin_scan    exclusive scan of the counts (one CTA; also re-zeroes them)
//   bin_scatter agent -> sorted slot start[cell] + rank: sorted positions with
//               the ORIGINAL index in .w, and/or the permutation itself
// The order inside a cell depends on atomic order; nothing downstream depends
// on it because every result is ordered by the (d2, index) key.
//
// Two grids use it: the Morton-ordered locality grid of the brute-force step
// (sorted query blocks and candidate stream -> spatially coherent warps, far
// fewer insertion-path entries; every pair is still evaluated) and the
// search grid of BOIDS_GRID (cells >= r, see k_grid.cu).
#include "internal.h"

namespace boids {

__device__ __forceinline__ uint32_t spread3(uint32_t x) {  // 10 bits -> every 3rd bit
  x &= 0x3ff;
  x = (x | (x << 16)) & 0x030000FF;
  x = (x | (x << 8)) & 0x0300F00F;
  x = (x | (x << 4)) & 0x030C30C3;
  x = (x | (x << 2)) & 0x09249249;
  return x;
}

__device__ __forceinline__ int cell_coord(float v, const BinGrid& g, int d) {
  // floor((v - lo) * inv_h), clamped into [0, dim-1]; NaN handled by the caller
  float t = (v - g.lo[d]) * g.inv_h;
  int c = (int)floorf(t);
  return c < 0 ? 0 : (c >= g.dim[d] ? g.dim[d] - 1 : c);
}

__device__ __forceinline__ int cell_of(float4 p, const BinGrid& g) {
  int ix = cell_coord(p.x, g, 0), iy = cell_coord(p.y, g, 1), iz = cell_coord(p.z, g, 2);
  if (g.morton) return (int)(spread3(ix) | (spread3(iy) << 1) | (spread3(iz) << 2));
  return (iz * g.dim[1] + iy) * g.dim[0] + ix;
}

// Agents j in [j0, j0 + count) of the segmented buffer `full`.
// keep_nan: bin agents with a NaN position into cell 0 (query binning: every
// owned agent must get a query slot); otherwise NaN slots -- the phantoms that
// pad every slice -- are skipped (candidate binning).
__global__ void k_bin_count(const float4* __restrict__ full, int64_t m, SliceDiv sd, int64_t j0, int64_t count,
                            BinGrid g, int2* __restrict__ cellrank, int* __restrict__ cnt, int keep_nan,
                            int think_k, int64_t think_t) {
  int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= count) return;
  if (!thinks(j0 + k, think_t, think_k)) {  // think mode: only this step's thinkers are queries
    cellrank[k] = make_int2(-1, 0);
    return;
  }
  float4 p = __ldg(pos_of(full, m, sd, j0 + k));
  const bool nan = p.x != p.x || p.y != p.y || p.z != p.z;
  if (nan && !keep_nan) {
    cellrank[k] = make_int2(-1, 0);
    return;
  }
  int c = nan ? 0 : cell_of(p, g);
  int r = atomicAdd(&cnt[c], 1);
  cellrank[k] = make_int2(c, r);
}

constexpr int SCAN_T = 1024;

// Block-wide exclusive scan of the padded shared array v[0..C) (index i at
// i + i/32: each thread's contiguous run is bank-conflict free); returns total.
__device__ __forceinline__ int block_scan_runs(int* sh, int C, int* warp_sums) {
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int per = (C + SCAN_T - 1) / SCAN_T;  // contiguous run per thread
  const int b = tid * per;
  int local = 0;
  for (int i = 0; i < per; ++i)
    if (b + i < C) local += sh[(b + i) + ((b + i) >> 5)];
  int v = local;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += y;
  }
  if (lane == 31) warp_sums[w] = v;
  __syncthreads();
  if (w == 0) {
    int s = warp_sums[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    warp_sums[lane] = s;  // inclusive prefix over warps
  }
  __syncthreads();
  int excl = v - local + (w > 0 ? warp_sums[w - 1] : 0);
  for (int i = 0; i < per; ++i) {
    if (b + i < C) {
      const int k = (b + i) + ((b + i) >> 5);
      const int c = sh[k];
      sh[k] = excl;
      excl += c;
    }
  }
  const int total = warp_sums[SCAN_T / 32 - 1];
  __syncthreads();
  return total;
}

// Exclusive scan of cnt[0..C) into start[0..C], start[C] = total; zeroes cnt.
// One CTA; counts are staged through shared memory with coalesced accesses.
// With item_start: also the work items of the grid search -- ceil(count / chunk)
// per cell -- scanned into item_start[0..C] (item_start[C] = number of items),
// and the grid kernel's work counter is reset.
__global__ void __launch_bounds__(SCAN_T) k_bin_scan(int* __restrict__ cnt, int* __restrict__ start, int C,
                                                    int* __restrict__ item_start, int chunk,
                                                    int* __restrict__ counter) {
  extern __shared__ int sh[];  // C + C / 32 words
  __shared__ int warp_sums[SCAN_T / 32];
  const int tid = threadIdx.x;
  for (int i = tid; i < C; i += SCAN_T) {
    sh[i + (i >> 5)] = cnt[i];
    cnt[i] = 0;
  }
  __syncthreads();
  const int total = block_scan_runs(sh, C, warp_sums);
  for (int i = tid; i < C; i += SCAN_T) start[i] = sh[i + (i >> 5)];
  if (tid == 0) start[C] = total;
  if (!item_start) return;
  __syncthreads();
  for (int i = tid; i < C; i += SCAN_T) {  // chunks per cell from the starts
    const int s0 = sh[i + (i >> 5)];
    const int s1 = i + 1 < C ? sh[(i + 1) + ((i + 1) >> 5)] : total;
    cnt[i] = (s1 - s0 + chunk - 1) / chunk;  // cnt is scratch here (re-zeroed below)
  }
  __syncthreads();
  for (int i = tid; i < C; i += SCAN_T) sh[i + (i >> 5)] = cnt[i];
  __syncthreads();
  const int items = block_scan_runs(sh, C, warp_sums);
  for (int i = tid; i < C; i += SCAN_T) {
    item_start[i] = sh[i + (i >> 5)];
    cnt[i] = 0;
  }
  if (tid == 0) {
    item_start[C] = items;
    *counter = 0;
  }
}

__global__ void k_bin_scatter(const float4* __restrict__ full, int64_t m, SliceDiv sd, int64_t j0, int64_t count,
                              const int2* __restrict__ cellrank, const int* __restrict__ start,
                              float4* __restrict__ spos, int* __restrict__ perm, int perm_base) {
  int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= count) return;
  int2 cr = cellrank[k];
  if (cr.x < 0) return;
  int dst = start[cr.x] + cr.y;
  int64_t j = j0 + k;
  if (spos) {
    float4 p = __ldg(pos_of(full, m, sd, j));
    spos[dst] = make_float4(p.x, p.y, p.z, __int_as_float((int)j));
  }
  if (perm) perm[dst] = (int)(j - perm_base);
}

cudaError_t launch_bin(const float4* full, int64_t m, const SliceDiv& sd, int64_t j0, int64_t count, const BinGrid& g,
                       int2* cellrank, int* cnt, int* start, float4* spos, int* perm, int perm_base,
                       cudaStream_t s, int* launches, int* item_start, int chunk, int* counter, int think_k,
                       int64_t think_t) {
  const unsigned blocks = (unsigned)((count + 255) / 256);
  if (count <= 0) {  // still publish an empty binning (starts, items, counter)
    const size_t shm0 = (size_t)(g.cells + g.cells / 32 + 1) * sizeof(int);
    if (shm0 > 48 * 1024) cudaFuncSetAttribute(k_bin_scan, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)shm0);
    k_bin_scan<<<1, SCAN_T, shm0, s>>>(cnt, start, g.cells, item_start, chunk, counter);
    return cudaGetLastError();
  }
  k_bin_count<<<blocks, 256, 0, s>>>(full, m, sd, j0, count, g, cellrank, cnt, spos == nullptr,
                                     spos == nullptr ? think_k : 1, think_t);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  const size_t shm = (size_t)(g.cells + g.cells / 32 + 1) * sizeof(int);
  if (shm > 48 * 1024) {
    e = cudaFuncSetAttribute(k_bin_scan, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)shm);
    if (e != cudaSuccess) return e;
  }
  k_bin_scan<<<1, SCAN_T, shm, s>>>(cnt, start, g.cells, item_start, chunk, counter);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  k_bin_scatter<<<blocks, 256, 0, s>>>(full, m, sd, j0, count, cellrank, start, spos, perm, perm_base);
  if (launches) *launches += 3;
  return cudaGetLastError();
}

// Search grid of BOIDS_GRID: cells of size h = r (1 + 2^-10) (a margin far above
// the fp32 rounding of the cell coordinate and of d2 < r2), row-major over the
// world box [-B, B]^3, B = max(world, init radius) * 1.02; agents outside are
// clamped into boundary cells, which keeps every pair closer than r in the same
// or adjacent cells (clamping is monotone and 1-Lipschitz on cell coordinates).
// The 27-cell stencil of a cell is then 9 contiguous x-runs of the sorted array.
BinGrid make_search_grid(const boids_params& p) {
  BinGrid g{};
  const float B = fmaxf(p.world_radius, p.init_radius) * 1.02f;
  g.h = p.search_radius * (1.0f + 1.0f / 1024.0f);
  int dim = (int)ceilf(2.f * B / g.h);
  if (dim < 1) dim = 1;
  if (dim > 1024) {  // huge world vs radius: cap the table (cells grow, still >= r)
    dim = 1024;
    g.h = 2.f * B / dim;
  }
  for (int d = 0; d < 3; ++d) {
    g.lo[d] = -B;
    g.dim[d] = dim;
  }
  g.inv_h = 1.f / g.h;
  g.cells = dim * dim * dim;
  g.morton = 0;
  return g;
}

// Morton locality grid for the brute-force step: 2^L cells per dimension over
// the world box (agents outside are clamped into boundary cells -- locality
// only, never correctness, in brute mode).  L = 5 (32^3 cells of ~3.2 units
// for R = 50) from n = 8192 on: fine enough that a 256-query block is compact
// even when the flock fills only part of the world (C3: ball r = 20).
BinGrid make_locality_grid(int64_t n, const boids_params& p) {
  BinGrid g{};
  const int L = n >= 8192 ? 5 : (n >= 1024 ? 4 : 3);
  const int dim = 1 << L;
  const float B = fmaxf(p.world_radius, p.init_radius) * 1.02f;
  for (int d = 0; d < 3; ++d) {
    g.lo[d] = -B;
    g.dim[d] = dim;
  }
  g.h = 2.f * B / dim;
  g.inv_h = 1.f / g.h;
  g.cells = dim * dim * dim;
  g.morton = 1;
  return g;
}

}  // namespace boids
