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
#include <algorithm>

#include "cells.cuh"

namespace boids {

// Agents j in [j0, j0 + count) of the segmented buffer `full`.
// keep_nan: bin agents with a NaN position into cell 0 (query binning: every
// owned agent must get a query slot); otherwise NaN slots -- the phantoms that
// pad every slice -- are skipped (candidate binning).
__global__ void k_bin_count(const float4* __restrict__ full, int64_t m, SliceDiv sd, int64_t j0, int64_t count,
                            BinGrid g, int2* __restrict__ cellrank, int* __restrict__ cnt, int keep_nan,
                            int think_k, int64_t think_t, const unsigned char* __restrict__ own) {
  int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= count) return;
  // think mode: only this step's thinkers are queries; spatial shards: only the owned agents
  if (!thinks(j0 + k, think_t, think_k) || (own && !own[k])) {
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

// Work items of the grid search from the (query) cell starts in sh (padded
// layout): runs of consecutive non-empty cells along x in one row holding at most
// `chunk` agents together; a cell with more than `chunk` agents is split into
// chunk-sized items of its own; a run spans at most MAX_SPAN cells.  Item = (first query slot, count, first cell,
// last x - first x).  One thread per row; pass 0 counts, pass 1 writes.
constexpr int MAX_SPAN = 8;  // cells per item: wider runs scan more candidates per query
#ifndef BOIDS_THINK_SPAN
#define BOIDS_THINK_SPAN 64
#endif
constexpr int THINK_SPAN = BOIDS_THINK_SPAN;  // ... in think mode: whole rows (C5 think 10: span 1 / 2 / 4 / 8 / 34 -> 5.77 / 3.99 / 3.18 / 2.90 / 2.71 ms; per-item cost dominates)
template <class StartOf>
__device__ __forceinline__ int row_items_g(StartOf start_of, int C, int total, int row, int D, int chunk, int4* out,
                                           int span = MAX_SPAN) {
  int n = 0, acc = 0, xs = -1, q0 = 0;
  auto cnt_of = [&](int c, int& s0) {
    s0 = start_of(c);
    const int s1 = c + 1 < C ? start_of(c + 1) : total;
    return s1 - s0;
  };
  auto close = [&](int xe) {
    if (xs >= 0) {
      if (out) out[n] = make_int4(q0, acc, row * D + xs, xe - xs);
      ++n;
    }
    xs = -1;
    acc = 0;
  };
  for (int x = 0; x < D; ++x) {
    int s0;
    const int k = cnt_of(row * D + x, s0);
    if (k == 0) {
      close(x - 1);
    } else if (k > chunk) {
      close(x - 1);
      for (int i = 0; i < k; i += chunk) {
        if (out) out[n] = make_int4(s0 + i, min(chunk, k - i), row * D + x, 0);
        ++n;
      }
    } else {
      if (acc + k > chunk || (xs >= 0 && x - xs >= span)) close(x - 1);
      if (xs < 0) {
        xs = x;
        q0 = s0;
      }
      acc += k;
    }
  }
  close(D - 1);
  return n;
}
__device__ __forceinline__ int row_items(const int* sh, int C, int total, int row, int D, int chunk, int4* out,
                                         int span) {
  return row_items_g([&](int c) { return sh[c + (c >> 5)]; }, C, total, row, D, chunk, out, span);
}

// Exclusive scan of cnt[0..C) into start[0..C], start[C] = total; zeroes cnt.
// One CTA; counts are staged through shared memory with coalesced accesses.
// With items: also the work items of the grid search (row_items) into
// items[0..*nitems), and the grid kernel's work counter is reset.
__global__ void __launch_bounds__(SCAN_T) k_bin_scan(int* __restrict__ cnt, int* __restrict__ start, int C,
                                                    int4* __restrict__ items, int* __restrict__ nitems, int chunk,
                                                    int* __restrict__ counter, int D, int span) {
  extern __shared__ int sh[];  // C + C / 32 words, then (items) rows + rows / 32 + 1 words
  __shared__ int warp_sums[SCAN_T / 32];
  const int tid = threadIdx.x;
  // one CTA reads all C counts: 8 loads in flight per thread, or the loop waits
  // one L2 round trip per element (C5: 39k cells, 42 -> a few us)
  for (int i0 = tid; i0 < C; i0 += SCAN_T * 8) {
    int v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) v[k] = i0 + k * SCAN_T < C ? cnt[i0 + k * SCAN_T] : 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int i = i0 + k * SCAN_T;
      if (i < C) {
        sh[i + (i >> 5)] = v[k];
        cnt[i] = 0;
      }
    }
  }
  __syncthreads();
  const int total = block_scan_runs(sh, C, warp_sums);
  for (int i = tid; i < C; i += SCAN_T) start[i] = sh[i + (i >> 5)];
  if (tid == 0) start[C] = total;
  if (!items) return;
  const int rows = C / D;
  int* rc = sh + C + (C >> 5) + 1;
  for (int r = tid; r < rows; r += SCAN_T) rc[r + (r >> 5)] = row_items(sh, C, total, r, D, chunk, nullptr, span);
  __syncthreads();
  const int n = block_scan_runs(rc, rows, warp_sums);
  for (int r = tid; r < rows; r += SCAN_T) row_items(sh, C, total, r, D, chunk, items + rc[r + (r >> 5)], span);
  if (tid == 0) {
    *nitems = n;
    *counter = 0;
  }
}

// ---- the same scan + work items over many CTAs, for large grids (C5: 39k
// cells; one CTA took 42 us): one warp per grid row of D cells.
//   rows1: row sums and the row's item count (rows are independent: an item
//          never crosses a row);
//   rows2: one CTA scans the row sums and item counts (rows << cells);
//   rows3: cell starts = row base + in-row prefix, the row's items, cnt zeroed.
constexpr int RW_WARPS = 8;
constexpr int RW_MAXD = 256;  // cells per row handled this way (else the one-CTA scan)
__device__ __forceinline__ int row_counts_to_smem(const int* cnt, int row, int D, int* rs, int lane) {
  int sum = 0;
  for (int x0 = 0; x0 < D; x0 += 32) {  // exclusive in-row prefix into rs[0..D], rs[D] = row total
    const int x = x0 + lane;
    const int k = x < D ? cnt[row * D + x] : 0;
    int v = k;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, v, o);
      if (lane >= o) v += y;
    }
    if (x < D) rs[x] = sum + v - k;
    sum += __shfl_sync(0xffffffffu, v, 31);
  }
  if (lane == 0) rs[D] = sum;
  __syncwarp();
  return sum;
}

__global__ void __launch_bounds__(RW_WARPS * 32) k_bin_rows1(const int* __restrict__ cnt, int rows, int D,
                                                             int chunk, int* __restrict__ rowsum,
                                                             int* __restrict__ rowitems, int span) {
  __shared__ int rs[RW_WARPS][RW_MAXD + 1];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int row = blockIdx.x * RW_WARPS + warp;
  if (row >= rows) return;
  const int sum = row_counts_to_smem(cnt, row, D, rs[warp], lane);
  if (lane == 0) {
    rowsum[row] = sum;
    // row_items over a (C = D, total = sum) view of this row's starts
    const int* r = rs[warp];
    if (rowitems) rowitems[row] = row_items_g([&](int c) { return r[c]; }, D, sum, 0, D, chunk, nullptr, span);
  }
}

__global__ void __launch_bounds__(SCAN_T) k_bin_rows2(int* __restrict__ rowsum, int* __restrict__ rowitems, int rows,
                                                     int* __restrict__ start, int C, int* __restrict__ nitems,
                                                     int* __restrict__ counter) {
  extern __shared__ int sh[];  // 2 x (rows + rows / 32 + 1)
  __shared__ int warp_sums[SCAN_T / 32];
  int* a = sh;
  int* b = sh + rows + (rows >> 5) + 1;
  for (int r = threadIdx.x; r < rows; r += SCAN_T) {
    a[r + (r >> 5)] = rowsum[r];
    if (rowitems) b[r + (r >> 5)] = rowitems[r];
  }
  __syncthreads();
  const int total = block_scan_runs(a, rows, warp_sums);
  const int n = rowitems ? block_scan_runs(b, rows, warp_sums) : 0;
  for (int r = threadIdx.x; r < rows; r += SCAN_T) {
    rowsum[r] = a[r + (r >> 5)];  // now the row's base
    if (rowitems) rowitems[r] = b[r + (r >> 5)];
  }
  if (threadIdx.x == 0) {
    start[C] = total;
    if (nitems) *nitems = n;
    if (counter) *counter = 0;
  }
}

__global__ void __launch_bounds__(RW_WARPS * 32) k_bin_rows3(int* __restrict__ cnt, int rows, int D, int chunk,
                                                             const int* __restrict__ rowbase,
                                                             const int* __restrict__ itembase,
                                                             int* __restrict__ start, int4* __restrict__ items,
                                                             int span) {
  __shared__ int rs[RW_WARPS][RW_MAXD + 1];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int row = blockIdx.x * RW_WARPS + warp;
  if (row >= rows) return;
  const int sum = row_counts_to_smem(cnt, row, D, rs[warp], lane);
  const int base = rowbase[row];
  for (int x = lane; x < D; x += 32) {
    start[row * D + x] = base + rs[warp][x];
    cnt[row * D + x] = 0;
  }
  if (items && lane == 0) {
    // the row's starts in absolute terms, then the same greedy items as the one-CTA scan
    int* r = rs[warp];
    for (int x = 0; x <= D; ++x) r[x] += base;
    int4* out = items + itembase[row];
    const int n = row_items_g([&](int c) { return r[c]; }, D, base + sum, 0, D, chunk, out, span);
    for (int k = 0; k < n; ++k) out[k].z += row * D;  // cell index: row-local -> global
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
                       cudaStream_t s, int* launches, int4* items, int* nitems, int chunk, int* counter,
                       int think_k, int64_t think_t, int* rowbuf, const unsigned char* own) {
  const unsigned blocks = (unsigned)((count + 255) / 256);
  const int rows = g.cells / g.dim[0];
  // think mode: items hold only this step's thinkers (1/k of the agents); longer
  // runs stream more candidates per query but amortise each item's fixed cost
  const int span = g.block > 0 ? (think_k > 1 ? 4 : 2) : (think_k > 1 ? THINK_SPAN : MAX_SPAN);
  const size_t shm = (size_t)(g.cells + g.cells / 32 + 1 + (items ? rows + rows / 32 + 1 : 0)) * sizeof(int);
  const int D = g.dim[0];
  // large grids scan on many CTAs (one warp per row); small ones in one CTA's shared memory
  const bool many = rowbuf && g.cells > 16384 && D <= RW_MAXD && g.cells % D == 0;
  if (!many && shm > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(k_bin_scan, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)shm);
    if (e != cudaSuccess) return e;
  }
  if (count <= 0 && !many) {  // still publish an empty binning (starts, items, counter)
    k_bin_scan<<<1, SCAN_T, shm, s>>>(cnt, start, g.cells, items, nitems, chunk, counter, g.dim[0], span);
    return cudaGetLastError();
  }
  BOIDS_PREFER_SMEM(k_bin_count);
  BOIDS_PREFER_SMEM(k_bin_scatter);
  BOIDS_PREFER_SMEM(k_bin_scan);
  if (count > 0)
    k_bin_count<<<blocks, 256, 0, s>>>(full, m, sd, j0, count, g, cellrank, cnt, spos == nullptr && !own,
                                       spos == nullptr ? think_k : 1, think_t, own);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  if (many) {  // large grid: many CTAs
    const unsigned rb = (unsigned)((rows + RW_WARPS - 1) / RW_WARPS);
    int* rowsum = rowbuf;
    int* rowit = items ? rowbuf + rows : nullptr;
    k_bin_rows1<<<rb, RW_WARPS * 32, 0, s>>>(cnt, rows, D, chunk, rowsum, rowit, span);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    const size_t shm2 = (size_t)2 * (rows + rows / 32 + 1) * sizeof(int);
    if (shm2 > 48 * 1024 &&
        (e = cudaFuncSetAttribute(k_bin_rows2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)shm2)) != cudaSuccess)
      return e;
    k_bin_rows2<<<1, SCAN_T, shm2, s>>>(rowsum, rowit, rows, start, g.cells, nitems, counter);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    k_bin_rows3<<<rb, RW_WARPS * 32, 0, s>>>(cnt, rows, D, chunk, rowsum, rowit, start, items, span);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    if (launches) *launches += 2;
  } else {
    k_bin_scan<<<1, SCAN_T, shm, s>>>(cnt, start, g.cells, items, nitems, chunk, counter, g.dim[0], span);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  if (count > 0) k_bin_scatter<<<blocks, 256, 0, s>>>(full, m, sd, j0, count, cellrank, start, spos, perm, perm_base);
  if (launches) *launches += 3;
  return cudaGetLastError();
}

// Search grid of BOIDS_GRID: row-major over the world box [-B, B]^3, B = max(world,
// init radius) * 1.02; agents outside are clamped into boundary cells (clamping
// is monotone and 1-Lipschitz on cell coordinates, so it never separates a pair
// by more cells than the distance allows).  Cells are much SMALLER than r: h =
// r (1 + 2^-10) / 6, so an agent closer than r lies within `reach` = 6 cells per
// axis (the 2^-10 margin is far above the fp32 rounding of the cell coordinate
// and of d2), and the warm bound of k_grid prunes the stencil to the cells its
// queries can reach (at C5's density 1 per axis: a warm limit of ~0.9 against
// cells of 1.5).  The table is capped at MAXD cells per axis: larger worlds get
// coarser cells and a smaller reach (>= 1).
constexpr int MAXD = 128;
constexpr int SEARCH_REACH = 6;
BinGrid make_search_grid(const boids_params& p) {
  BinGrid g{};
  const float B = fmaxf(p.world_radius, p.init_radius) * 1.02f;
  const float hr = p.search_radius * (1.0f + 1.0f / 1024.0f);  // >= r with margin
  int reach = SEARCH_REACH;
  float h = hr / (float)reach;
  int dim = (int)ceilf(2.f * B / h);
  while (dim > MAXD && reach > 1) {  // coarser cells, down to cells >= r (reach 1)
    --reach;
    h = hr / (float)reach;
    dim = (int)ceilf(2.f * B / h);
  }
  if (dim > MAXD) {  // cells larger than r (reach 1 still covers r)
    dim = MAXD;
    h = fmaxf(hr, 2.f * B / dim * (1.0f + 1.0f / 1024.0f));
  }
  if (dim < 1) dim = 1;
  for (int d = 0; d < 3; ++d) {
    g.lo[d] = -B;
    g.dim[d] = dim;
  }
  g.h = h;
  g.inv_h = 1.f / g.h;
  g.cells = dim * dim * dim;
  g.morton = 0;
  g.reach = reach;
  for (int d = 0; d < 3; ++d) g.fdim[d] = dim;
  return g;
}

// The grid search's query blocks: QBLOCK^3 cells of the search grid.  A work
// item of k_grid is (a run along x of) one block's queries, so its stencil is a
// compact box -- (QBLOCK + 2R)^3 cells around QBLOCK^3 -- instead of the long thin
// one of a run of cells along x (C5: ~1500 instead of ~4200 candidates per
// query); the queries are binned by block (cell_of on a block grid divides the
// fine cell coordinates, so a query's block always contains its fine cell).
constexpr int QBLOCK = 4;
BinGrid make_query_grid(const BinGrid& sg) {
  BinGrid g = sg;
  g.block = QBLOCK;
  for (int d = 0; d < 3; ++d) {
    g.fdim[d] = sg.dim[d];
    g.dim[d] = (sg.dim[d] + QBLOCK - 1) / QBLOCK;
  }
  g.cells = g.dim[0] * g.dim[1] * g.dim[2];
  return g;
}

// A spatial shard's own part of the search grid: the cell layers z in [z0, z1)
// (its slab plus its halo layers) with the x and y extent of the whole grid.
// The cells are those of the full grid, so nothing but the table shrinks.
BinGrid make_slab_grid(const BinGrid& sg, int z0, int z1) {
  BinGrid g = sg;
  g.lo[2] = sg.lo[2] + (float)z0 * sg.h;
  g.dim[2] = std::max(1, z1 - z0);
  g.fdim[2] = g.dim[2];
  g.cells = g.dim[0] * g.dim[1] * g.dim[2];
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
