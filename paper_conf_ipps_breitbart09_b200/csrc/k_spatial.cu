// k_spatial.cu -- spatial decomposition of the grid-binned step over ranks
// ("spatial data structures" and multiple devices are the
// thesis's future work).
//
// Rank g of G OWNS the agents whose search-grid cell layer z lies in its slab
// [zb[g], zb[g+1]) (cell coordinates of the fine search grid; the boundaries
// balance the initial agent counts).  Agent indices stay global: a spatial
// handle addresses all n agents (one segment, like a single-GPU handle) but
// holds valid positions only for its own agents and for its HALO -- the agents
// within `reach` cell layers of its slab (reach cells >= r: every agent closer
// than r to an owned agent) -- and NaN everywhere else, which the candidate
// binning skips.  So the grid search of the owned queries sees exactly the
// candidates a single GPU would (identical lists, steering and state), while a
// rank exchanges only its boundary layers instead of all-gathering n agents.
//
// After each step (positions moved): every owned agent whose new cell layer
// belongs to another slab MIGRATES there with its whole state (position,
// forward + speed, up, side, neighbour lists -- the next step's warm bound --,
// OpenSteer's smoothed acceleration); every agent, migrating or not, is sent as
// HALO (position, forward) to each other rank whose halo layers contain it, and
// kept as halo by this rank when its own halo layers do.  Non-owned entries
// that are not kept are cleared to NaN first, so received records land in a
// clean buffer.  Records are packed per destination into fixed-capacity
// outboxes (device counters; an overflow is reported, never silent); the caller
// moves them (NCCL all-to-all, or device copies when emulating) and unpacks.
#include <algorithm>

#include "cells.cuh"

namespace boids {

// Halo record: 2 float4 = (x, y, z, index bits), (fx, fy, fz, speed).
// Migrant record: 8 float4 = pos | fwd | up | side | nbr0..3 | nbr4..6, cnt | nbr8, -, -, - | acc.
constexpr int HALO_F4 = 2;
constexpr int MIG_F4 = 8;

namespace {

__device__ __forceinline__ int slab_of(int cz, const int* zb, int world) {
  int s = 0;
  while (s + 1 < world && cz >= zb[s + 1]) ++s;
  return s;
}

__device__ __forceinline__ bool in_halo(int cz, const int* zb, int r, int reach) {
  return (cz >= zb[r] - reach && cz < zb[r]) || (cz >= zb[r + 1] && cz < zb[r + 1] + reach);
}

__device__ __forceinline__ int zlayer(float z, const BinGrid& g) {
  if (!(z == z)) return -1;
  return cell_coord(z, g, 2);
}

// Initial ownership and halo from the positions every rank holds (after init or
// an upload of all n agents): own[j] = 1 for owned agents, positions of agents
// neither owned nor halo cleared to NaN.
__global__ void k_spatial_init(float4* __restrict__ cur, int64_t m, int64_t n, unsigned char* __restrict__ own,
                               BinGrid g, const int* __restrict__ zb, int world, int rank, int reach,
                               int* __restrict__ kept, int* __restrict__ nkept) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  const int cz = zlayer(cur[j].z, g);
  const bool mine = cz >= 0 && slab_of(cz, zb, world) == rank;
  own[j] = mine ? 1 : 0;
  if (mine) return;
  if (cz >= 0 && in_halo(cz, zb, rank, reach)) {
    kept[atomicAdd(nkept, 1)] = (int)j;  // a halo entry: cleared by the next pack
  } else {
    const float nan = __int_as_float(0x7fc00000);
    cur[j] = make_float4(nan, nan, nan, 0.f);
  }
}

// The two ping-pong state buffers.  Invariant at the start of a step: the
// buffer the step writes (the non-current one) holds NaN for every agent this
// rank does not own, so after the step and the flip the new current buffer
// holds exactly the owned agents -- and the buffer just read holds the owned
// agents' old entries plus last step's halo.  The pack clears that halo there
// (its entries are listed: the records the last unpack applied -- the inbox
// still holds them -- and the entries kept locally), and clears a migrant's
// old entry there too, so the invariant holds for the next step without
// touching the other n entries.
__global__ void k_spatial_clear(float4* __restrict__ cur, const float4* __restrict__ halo_in, int64_t nh,
                                const int* __restrict__ kept, const int* __restrict__ nkept) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const float nan = __int_as_float(0x7fc00000);
  if (k < nh) cur[__float_as_int(halo_in[k * HALO_F4].w)] = make_float4(nan, nan, nan, 0.f);
  if (k < *nkept) cur[kept[k]] = make_float4(nan, nan, nan, 0.f);
}

// One slot per set lane of `want` in destination counter *ctr: one atomic per
// warp (ballot + popc) instead of one per record -- thousands of records per
// destination would otherwise serialise on the counter.  All lanes call it.
__device__ __forceinline__ int warp_slot(bool want, int* ctr) {
  const unsigned b = __ballot_sync(0xffffffffu, want);
  if (!b) return -1;
  const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
  int base = 0;
  if (lane == leader) base = atomicAdd(ctr, __popc(b));
  base = __shfl_sync(0xffffffffu, base, leader);
  return want ? base + __popc(b & ((1u << lane) - 1u)) : -1;
}

__global__ void __launch_bounds__(256) k_spatial_pack(float4* __restrict__ cur, float4* __restrict__ prev, int64_t m,
                               int64_t n, unsigned char* __restrict__ own,
                               const float4* __restrict__ up4, const float4* __restrict__ side4,
                               const int32_t* __restrict__ nbr, const int32_t* __restrict__ cnt,
                               const int32_t* __restrict__ nbr8, const float4* __restrict__ acc4, BinGrid g,
                               const int* __restrict__ zb, int world, int rank, int reach,
                               float4* __restrict__ halo_out, int64_t cap_h, float4* __restrict__ mig_out,
                               int64_t cap_m, int* __restrict__ counts, int* __restrict__ overflow,
                               int* __restrict__ kept, int* __restrict__ nkept) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const float nan = __int_as_float(0x7fc00000);
  const bool valid = j < n;
  const bool mine = valid && own[j];  // (stale halo entries were cleared by k_spatial_clear)
  float4 p = make_float4(0.f, 0.f, 0.f, 0.f), f = p;
  int cz = -1, dest = rank;
  if (mine) {
    p = cur[j];
    f = cur[m + j];
    cz = zlayer(p.z, g);
    dest = cz >= 0 ? slab_of(cz, zb, world) : rank;
  }
  for (int d = 0; d < world; ++d) {  // halo copies for every other rank whose layers hold it
    const bool want = mine && d != rank && d != dest && cz >= 0 && in_halo(cz, zb, d, reach);
    const int slot = warp_slot(want, &counts[d]);
    if (!want) continue;
    if (slot >= cap_h) {
      atomicAdd(overflow, 1);
      continue;
    }
    float4* r = halo_out + ((int64_t)d * cap_h + slot) * HALO_F4;
    r[0] = make_float4(p.x, p.y, p.z, __int_as_float((int)j));
    r[1] = f;
  }
  for (int d = 0; d < world; ++d) {  // migrants: the whole state to the new owner
    const bool want = mine && dest == d && d != rank;
    const int slot = warp_slot(want, &counts[world + d]);
    if (!want) continue;
    if (slot >= cap_m) {
      atomicAdd(overflow, 1);
      continue;
    }
    float4* r = mig_out + ((int64_t)d * cap_m + slot) * MIG_F4;
    r[0] = make_float4(p.x, p.y, p.z, __int_as_float((int)j));
    r[1] = f;
    r[2] = up4[j];
    r[3] = side4[j];
    r[4] = make_float4(__int_as_float(nbr[j * 7 + 0]), __int_as_float(nbr[j * 7 + 1]), __int_as_float(nbr[j * 7 + 2]),
                       __int_as_float(nbr[j * 7 + 3]));
    r[5] = make_float4(__int_as_float(nbr[j * 7 + 4]), __int_as_float(nbr[j * 7 + 5]), __int_as_float(nbr[j * 7 + 6]),
                       __int_as_float(cnt[j]));
    r[6] = make_float4(__int_as_float(nbr8[j]), 0.f, 0.f, 0.f);
    r[7] = acc4 ? acc4[j] : make_float4(0.f, 0.f, 0.f, 0.f);
    own[j] = 0;
    prev[j] = make_float4(nan, nan, nan, 0.f);  // its old entry in the other buffer
    // it left for `dest`; this rank keeps it only as halo (listed for the next clear)
    if (!in_halo(cz, zb, rank, reach)) cur[j] = make_float4(nan, nan, nan, 0.f);
    else kept[atomicAdd(nkept, 1)] = (int)j;
  }
}

__global__ void k_spatial_unpack_mig(const float4* __restrict__ rec, int64_t count, float4* __restrict__ cur,
                                     int64_t m, unsigned char* __restrict__ own, float4* __restrict__ up4,
                                     float4* __restrict__ side4, int32_t* __restrict__ nbr, int32_t* __restrict__ cnt,
                                     int32_t* __restrict__ nbr8, float4* __restrict__ acc4) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= count) return;
  const float4* r = rec + k * MIG_F4;
  const float4 p = r[0];
  const int64_t j = __float_as_int(p.w);
  cur[j] = make_float4(p.x, p.y, p.z, 0.f);
  cur[m + j] = r[1];
  up4[j] = r[2];
  side4[j] = r[3];
  const float4 a = r[4], b = r[5], c = r[6];
  nbr[j * 7 + 0] = __float_as_int(a.x);
  nbr[j * 7 + 1] = __float_as_int(a.y);
  nbr[j * 7 + 2] = __float_as_int(a.z);
  nbr[j * 7 + 3] = __float_as_int(a.w);
  nbr[j * 7 + 4] = __float_as_int(b.x);
  nbr[j * 7 + 5] = __float_as_int(b.y);
  nbr[j * 7 + 6] = __float_as_int(b.z);
  cnt[j] = __float_as_int(b.w);
  nbr8[j] = __float_as_int(c.x);
  if (acc4) acc4[j] = r[7];
  own[j] = 1;
}

__global__ void k_spatial_unpack_halo(const float4* __restrict__ rec, int64_t count, float4* __restrict__ cur,
                                      int64_t m) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= count) return;
  const float4 p = rec[k * HALO_F4];
  const int64_t j = __float_as_int(p.w);
  cur[j] = make_float4(p.x, p.y, p.z, 0.f);
  cur[m + j] = rec[k * HALO_F4 + 1];
}

// Histogram of the agents over the grid's z layers (slab boundaries at creation).
__global__ void k_zhist(const float4* __restrict__ cur, int64_t n, BinGrid g, int* __restrict__ hist) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  const int cz = zlayer(cur[j].z, g);
  if (cz >= 0) atomicAdd(&hist[cz], 1);
}

}  // namespace

int spatial_halo_f4() { return HALO_F4; }
int spatial_mig_f4() { return MIG_F4; }

cudaError_t launch_zhist(const float4* cur, int64_t n, const BinGrid& g, int* hist, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  k_zhist<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(cur, n, g, hist);
  return cudaGetLastError();
}

cudaError_t launch_spatial_init(float4* cur, float4* other, int64_t m, int64_t n, unsigned char* own,
                                const BinGrid& g, const int* zb, int world, int rank, int reach, int* kept,
                                int* nkept, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  if (cudaError_t e = cudaMemsetAsync(nkept, 0, sizeof(int), s)) return e;
  k_spatial_init<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(cur, m, n, own, g, zb, world, rank, reach, kept, nkept);
  if (cudaError_t e = cudaGetLastError()) return e;
  // the other buffer (written by the next step): the owned agents only
  if (cudaError_t e = cudaMemcpyAsync(other, cur, (size_t)2 * m * sizeof(float4), cudaMemcpyDeviceToDevice, s))
    return e;
  k_spatial_clear<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(other, nullptr, 0, kept, nkept);
  return cudaGetLastError();
}

cudaError_t launch_spatial_pack(float4* cur, float4* prev, int64_t m, int64_t n, unsigned char* own, const float4* up4,
                                const float4* side4, const int32_t* nbr, const int32_t* cnt, const int32_t* nbr8,
                                const float4* acc4, const BinGrid& g, const int* zb, int world, int rank, int reach,
                                float4* halo_out, int64_t cap_h, float4* mig_out, int64_t cap_m, int* counts,
                                int* overflow, const float4* halo_in, int64_t nh_prev, int* kept, int* nkept,
                                int64_t nkept_cap, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  const int64_t nc = std::max<int64_t>(nh_prev, nkept_cap);
  if (nc > 0) k_spatial_clear<<<(unsigned)((nc + 255) / 256), 256, 0, s>>>(prev, halo_in, nh_prev, kept, nkept);
  if (cudaError_t e = cudaGetLastError()) return e;
  if (cudaError_t e = cudaMemsetAsync(nkept, 0, sizeof(int), s)) return e;
  k_spatial_pack<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(cur, prev, m, n, own, up4, side4, nbr, cnt, nbr8, acc4, g, zb,
                                                             world, rank, reach, halo_out, cap_h, mig_out, cap_m,
                                                             counts, overflow, kept, nkept);
  return cudaGetLastError();
}

cudaError_t launch_spatial_unpack(const float4* halo_in, int64_t nh, const float4* mig_in, int64_t nm, float4* cur,
                                  int64_t m, unsigned char* own, float4* up4, float4* side4, int32_t* nbr,
                                  int32_t* cnt, int32_t* nbr8, float4* acc4, cudaStream_t s) {
  if (nm > 0) {
    k_spatial_unpack_mig<<<(unsigned)((nm + 255) / 256), 256, 0, s>>>(mig_in, nm, cur, m, own, up4, side4, nbr, cnt,
                                                                      nbr8, acc4);
    if (cudaError_t e = cudaGetLastError()) return e;
  }
  if (nh > 0) {
    k_spatial_unpack_halo<<<(unsigned)((nh + 255) / 256), 256, 0, s>>>(halo_in, nh, cur, m);
    if (cudaError_t e = cudaGetLastError()) return e;
  }
  return cudaSuccess;
}

}  // namespace boids
