// k_grid.cu -- the grid-binned Boids step (search_mode = BOIDS_GRID), one fused
// kernel after the binning passes of k_bin.cu.
//
// The thesis names spatial data structures as the way to speed up the neighbour
// search (future work); north_star asks for a uniform-grid variant that
// returns the IDENTICAL neighbour sets.  Cells have size h >= r / reach
// (make_search_grid, reach = 3 by default), so every agent closer than r lies
// within `reach` cells per axis; within those the search is exactly the
// brute-force definition (d2 < fl(r*r), top-7 by the (d2, index) key, Listing
// 5.2 / 6.3 with readings Q2-Q4), so the result is bit-identical to BOIDS_BRUTE.
//
// Stencil pruning by the warm bound: only agents with d2 <= lim_i can enter query
// i's list (lim_i = min(prev(r2), t0_i), the bound of k_warm.cu), and such an
// agent is at most floor(sqrt(lim_i) / h) + 1 cells away per axis.  Each item
// takes R = that reach for the largest limit among its queries (capped at
// `reach`; a cold step or a wrapped agent gives the full reach), so a warm step
// typically scans 3 x 3 x 3 cells of r/3 -- 1/27 of the volume of the
// unpruned 27-cell stencil of cells >= r.
//
// Work item = a run of consecutive cells along x in one row holding <= 512
// owned agents (a larger cell is split into chunks of its own; k_bin_scan).  A
// persistent grid of CTAs pulls items from an atomic queue (cells hold very
// different numbers of agents -- the flock is a ball inside a box).  Row-major
// cell order makes each of the (2R+1)^2 stencil rows one contiguous range of the
// sorted candidate array (x from the run's first cell - R to its last + R); the
// ranges stream through a TMA ring (cp.async.bulk of any 16-byte multiple, so
// partial tiles need no padding).  A query's whole stencil is scanned by one CTA,
// so its top-7 list (shared memory, limit tightened by the warm bound and by the
// list's own 7th key) is final at the end of the item, and the CTA finishes the
// agents (steering + modification) itself: search, steering and modification
// in one kernel, no merge.
#include <algorithm>
#include <cstdlib>

#include "step_common.cuh"
#include "tma.cuh"

namespace boids {
namespace {

constexpr int NTG = 128;        // threads per CTA
constexpr int Q = 4;            // queries per thread
constexpr int QBG = NTG * Q;    // queries per item (512)
constexpr int CT = 256;         // candidates per tile (<= 4 KB bulk copy)
constexpr int STAGES = 3;
constexpr int U = 4;
constexpr int FAR_MAX = 16;  // queries per item routed to k_grid_far
constexpr int MAXROWS = 256;  // stencil rows of an item: (QBLOCK + 2 reach)^2 <= (4 + 12)^2
// Query slot of (warp, q, lane).  Blocked (full items): a warp's 4 x 32 queries
// are consecutive and warps past the item's queries only keep the ring protocol
// (measured on full C5 items: round-robin 4.13 vs blocked 3.25 ms/step -- the
// padded slots cost more than the idle warps).  Round-robin over the warps
// (small items, <= RR_MAX queries: a spatial shard's or a sparse region's): q
// group q of warp w holds slots q*NTG + 32w + lane, so every warp works.
constexpr int RR_MAX = 2 * NTG;
__device__ __forceinline__ int qslot(int warp, int q, int lane, bool rr) {
  return rr ? q * NTG + warp * 32 + lane : warp * 32 * Q + q * 32 + lane;
}

struct __align__(16) GridSmem {
  float4 ring[STAGES][CT];
  key_t lists[7 * QBG];  // [7][QBG]
  uint64_t full[STAGES];
  uint64_t empty[STAGES];
  int2 range[MAXROWS];   // stencil row ranges [lo, hi) in the sorted candidate array (empty ones too)
  int nrange, item, cell, span, qs0, qn;
  unsigned long long cand;  // candidates of the item's stencil (grid_pairs accounting)
  int maxlim;            // largest query limit of the item (float bits; limits are >= 0)
  int maxnear;           // ... over the queries that need only the adjacent cells
  int nfar;              // queries that need more (routed to k_grid_far when few)
};

// A bound for a query whose warm bound reaches past the adjacent cells (a cold
// step, an agent that wrapped to the diametric opposite point, or whose
// neighbours did): the 7th smallest d2 to the other agents of the 3 x 3 x 3
// cells around its own, which the binning of THIS step put together (current
// positions).  Real, distinct agents, so an upper bound on the 7th key like t0;
// +inf with fewer than 7.  It usually brings the query back within the adjacent
// cells, so it is searched in its item instead of by k_grid_far.
__device__ float cell_bound(const GridArgs& g, float4 me, int gi) {
  auto coord = [&](float v, int d) {
    const int c = (int)floorf((v - g.grid.lo[d]) * g.grid.inv_h);
    return c < 0 ? 0 : (c >= g.grid.dim[d] ? g.grid.dim[d] - 1 : c);
  };
  float b[7];
#pragma unroll
  for (int k = 0; k < 7; ++k) b[k] = __int_as_float(0x7f800000);
  if (!(me.x == me.x && me.y == me.y && me.z == me.z)) return b[6];
  const int Dx = g.grid.dim[0], Dy = g.grid.dim[1], Dz = g.grid.dim[2];
  const int cx = coord(me.x, 0), cy = coord(me.y, 1), cz = coord(me.z, 2);
  const int x0 = max(cx - 1, 0), x1 = min(cx + 1, Dx - 1);
  for (int z = max(cz - 1, 0); z <= min(cz + 1, Dz - 1); ++z)
    for (int y = max(cy - 1, 0); y <= min(cy + 1, Dy - 1); ++y) {
      const int row = (z * Dy + y) * Dx;
      const int lo = __ldg(g.cstart + row + x0), hi = __ldg(g.cstart + row + x1 + 1);
      constexpr int G = 8;  // loads in flight
      for (int k0 = lo; k0 < hi; k0 += G) {
        float4 c[G];
#pragma unroll
        for (int k = 0; k < G; ++k)
          c[k] = k0 + k < hi ? __ldg(g.spos + k0 + k) : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
#pragma unroll
        for (int k = 0; k < G; ++k) {
          if (__float_as_int(c[k].w) == gi) continue;
          float d = dist2(me.x, me.y, me.z, c[k]);
          if (!(d == d)) continue;
#pragma unroll
          for (int t = 0; t < 7; ++t) {  // keep the 7 smallest, ascending
            const float l = fminf(b[t], d);
            d = fmaxf(b[t], d);
            b[t] = l;
          }
        }
      }
    }
  return b[6];
}

// Tiles concatenate consecutive stencil rows: a tile takes up to CT candidates
// from ranges r, r+1, ... (one bulk copy per piece, into consecutive ring
// slots, all completing on the stage's full barrier), so the short rows of a
// compact stencil (~40 candidates each at C5) still fill whole tiles.
// walk(): the tile at (r, off) -> its candidate count; (r, off) advanced past it.
__device__ __forceinline__ int walk(const GridSmem& sm, int& r, int& off) {
  int cnt = 0;
  while (r < sm.nrange && cnt < CT) {
    const int len = sm.range[r].y - sm.range[r].x;
    const int take = min(len - off, CT - cnt);
    cnt += take;
    off += take;
    if (off >= len) {
      ++r;
      off = 0;
    }
  }
  return cnt;
}

__device__ __forceinline__ void issue(GridSmem& sm, const GridArgs& g, uint32_t tc, int& r, int& off) {
  const int s = (int)(tc % STAGES);
  if (tc >= STAGES) {
    mbar_wait(&sm.empty[s], ((tc - STAGES) / STAGES) & 1u);
    fence_proxy_async_smem();
  }
  int r2 = r, off2 = off;
  const int cnt = walk(sm, r2, off2);
  mbar_arrive_expect_tx(&sm.full[s], cnt * (uint32_t)sizeof(float4));
  int done = 0;
  while (done < cnt) {
    const int len = sm.range[r].y - sm.range[r].x;
    const int take = min(len - off, cnt - done);
    if (take > 0)
      tma_load_1d(sm.ring[s] + done, g.spos + sm.range[r].x + off, take * (uint32_t)sizeof(float4), &sm.full[s]);
    done += take;
    off += take;
    if (off >= len) {
      ++r;
      off = 0;
    }
  }
  r = r2;
  off = off2;
}

// One tile of candidates against this thread's first QV queries (the rest of
// the warp's groups hold no queries): distances, vote, rare exact insertion.
template <int QV>
__device__ __forceinline__ void grid_tile(const float4* tile, int cnt, const float2 (&pxy)[Q], const float (&pz)[Q],
                                          float (&lim)[Q], float& limc, const int (&gq)[Q], key_t* lists, int warp,
                                          int lane, bool rr, unsigned& groups, unsigned& slow_groups) {
  for (int c = 0; c < cnt; c += U) {
    float4 cc[U];
    if (c + U <= cnt) {
#pragma unroll
      for (int u = 0; u < U; ++u) cc[u] = tile[c + u];
    } else {  // ragged tail of a range
#pragma unroll
      for (int u = 0; u < U; ++u)
        cc[u] = c + u < cnt ? tile[c + u] : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, __int_as_float(-1));
    }
    // d2 = ((dx*dx) + (dy*dy)) + (dz*dz), every op rounded (Appendix A), packed
    // FADD2/FMUL2 on the (x, y) pairs, scalar dz and sums (see k_sym.cu)
    float d[QV][U];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int q = 0; q < QV; ++q) {
        const float2 dxy = __fadd2_rn(pxy[q], make_float2(-cc[u].x, -cc[u].y));
        const float2 sq = __fmul2_rn(dxy, dxy);
        const float dz = __fsub_rn(pz[q], cc[u].z);
        d[q][u] = __fadd_rn(__fadd_rn(sq.x, sq.y), __fmul_rn(dz, dz));
      }
    float m = d[0][0];
#pragma unroll
    for (int q = 0; q < QV; ++q)
#pragma unroll
      for (int u = 0; u < U; ++u) m = fminf(m, d[q][u]);
    ++groups;
    if (__any_sync(0xffffffffu, m <= limc)) {
      ++slow_groups;
      // Every lane collects its passing (query, candidate) pairs as bits, then
      // the warp inserts them lane-parallel: each round every lane with bits
      // left inserts its lowest one, so the warp runs max-per-lane rounds of the
      // insertion instead of one per distinct (q, u) any lane holds.  A round
      // re-reads its candidate from the tile and recomputes the d2 with the same
      // operations (the same float) -- cheaper than selecting one of the 16
      // distances held in registers.  The order of insertions never matters
      // (exact (d2, index) key; a pair above the tightened limit cannot be among
      // the final 7).
      unsigned bits = 0;
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int j = __float_as_int(cc[u].w);  // original index
#pragma unroll
        for (int q = 0; q < QV; ++q)
          if (d[q][u] <= lim[q] && j != gq[q]) bits |= 1u << (q * U + u);
      }
      while (__any_sync(0xffffffffu, bits != 0)) {
        if (bits) {
          const int b = __ffs(bits) - 1;
          bits &= bits - 1;
          const int qq = b / U;
          float2 qxy = pxy[0];
          float qz = pz[0], lq = lim[0];
#pragma unroll
          for (int q = 1; q < QV; ++q)
            if (qq == q) {
              qxy = pxy[q];
              qz = pz[q];
              lq = lim[q];
            }
          const float4 cu = tile[c + (b % U)];
          const float2 dxy = __fadd2_rn(qxy, make_float2(-cu.x, -cu.y));
          const float2 sq = __fmul2_rn(dxy, dxy);
          const float dz = __fsub_rn(qz, cu.z);
          const float dd = __fadd_rn(__fadd_rn(sq.x, sq.y), __fmul_rn(dz, dz));
          if (dd <= lq) {  // the limit may have tightened since the bit was set
            const float nl = insert_smem7(&lists[qslot(warp, qq, lane, rr)], QBG, make_key(dd, __float_as_int(cu.w)));
#pragma unroll
            for (int q = 0; q < QV; ++q)
              if (q == qq) lim[q] = fminf(lim[q], nl);
          }
        }
      }
      limc = lim[0];
#pragma unroll
      for (int q = 1; q < QV; ++q) limc = fmaxf(limc, lim[q]);
    }
  }
}

__global__ void __launch_bounds__(NTG, 5) k_grid(StepArgs a, GridArgs g) {  // 5 CTAs / SM: 3.38 -> 3.27 ms at C5 (4: 127 regs; 6: spills more, 3.33)
  __shared__ GridSmem sm;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
#pragma unroll
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], NTG);
    }
    mbar_fence_init();
  }
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  const float r2_in = __uint_as_float(__float_as_uint(r2) - 1u);  // d2 < r2  <=>  d2 <= r2_in
  const int D = g.grid.dim[0];
  const int n_items = *g.nitems;
  uint32_t tc = 0;  // tiles issued / consumed by this CTA
  unsigned slow_groups = 0, groups = 0;
  for (;;) {
    __syncthreads();  // previous item fully finished (lists, ranges)
    if (tid == 0) {
      const int it = atomicAdd(g.counter, 1);
      sm.item = it;
      if (it < n_items) {
        const int4 w = g.items[it];
        sm.qs0 = w.x;
        sm.qn = w.y;
        sm.cell = w.z;
        sm.span = w.w;
      }
      sm.maxlim = 0;
      sm.maxnear = 0;
      sm.nfar = 0;
    }
    __syncthreads();
    if (sm.item >= n_items) break;
    const int qs0 = sm.qs0, qn = sm.qn;
    const bool rr = qn <= RR_MAX;  // small item: query slots round-robin over the warps

    // queries: 4 per thread, with their limits (the warm bound)
    float2 pxy[Q];
    float pz[Q], lim[Q];
    int gq[Q];
    int64_t qloc[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const int slot = qslot(warp, q, lane, rr);
      const int64_t qi = slot < qn ? (int64_t)__ldg(g.qperm + qs0 + slot) : a.nloc;
      qloc[q] = qi;
      gq[q] = (int)(a.lo + qi);
      const float4 me = qi < a.nloc ? __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi))
                                    : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
      pxy[q] = make_float2(me.x, me.y);
      pz[q] = me.z;
      lim[q] = fminf(r2_in, a.warm ? warm_bound(a, qi, me) : __int_as_float(0x7f800000));
      if (qi < a.nloc && sqrtf(lim[q]) * g.grid.inv_h * (1.0f + 1.0f / 1024.0f) >= 1.0f)
        lim[q] = fminf(lim[q], cell_bound(g, me, gq[q]));
#pragma unroll
      for (int s = 0; s < 7; ++s) sm.lists[s * QBG + slot] = KEY_EMPTY;
    }
    {
      // A query whose limit reaches past the adjacent cells (a wrapped agent, a
      // neighbour that left) would widen the whole item's stencil: up to FAR_MAX
      // of them per item are routed to k_grid_far (one CTA each, own stencil)
      // and skipped here.  More than that (a cold step) -> the item takes the
      // full reach itself.
      float ml = 0.f, mn = 0.f;  // max limit over all / over the near queries
      bool far[Q];
      int nf = 0;
#pragma unroll
      for (int q = 0; q < Q; ++q) {
        const bool valid = qloc[q] < a.nloc;
        far[q] = valid && g.flist && sqrtf(lim[q]) * g.grid.inv_h * (1.0f + 1.0f / 1024.0f) >= 1.0f;
        if (valid) ml = fmaxf(ml, lim[q]);
        if (valid && !far[q]) mn = fmaxf(mn, lim[q]);
        nf += far[q] ? 1 : 0;
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        ml = fmaxf(ml, __shfl_xor_sync(0xffffffffu, ml, o));
        mn = fmaxf(mn, __shfl_xor_sync(0xffffffffu, mn, o));
        nf += __shfl_xor_sync(0xffffffffu, nf, o);
      }
      if (lane == 0) {
        atomicMax(&sm.maxlim, __float_as_int(ml));
        atomicMax(&sm.maxnear, __float_as_int(mn));
        atomicAdd(&sm.nfar, nf);
      }
      __syncthreads();
      if (sm.nfar > 0 && sm.nfar <= FAR_MAX) {
#pragma unroll
        for (int q = 0; q < Q; ++q)
          if (far[q]) {
            const int fs = atomicAdd(g.fcount, 1);
            g.flist[fs] = (int)qloc[q];
            g.flim[fs] = lim[q];  // its bound (warm bound, cell bound): k_grid_far's reach
            if (a.stats) atomicAdd(a.stats + 2, 1ull);  // boids_info.fallbacks: queries searched by k_grid_far
            qloc[q] = a.nloc;  // not finished here
            pxy[q] = make_float2(__int_as_float(0x7fc00000), 0.f);
            lim[q] = -1.f;
          }
        if (tid == 0) sm.maxlim = sm.maxnear;
      }
    }
    __syncthreads();
    {
      // Stencil of this item: its block run (QBLOCK^3 cells each, `span` + 1
      // blocks along x) grown by R cells per side, where agents within
      // sqrt(maxlim) are at most floor(sqrt(maxlim) / h) + 1 cells away per axis
      // (margin 2^-10 >> fp32 rounding).  One range of the cell-sorted candidate
      // array per row (y, z) of the box, computed by one thread each.
      const float ml = __int_as_float(sm.maxlim);
      const int Rg = g.grid.reach;
      const float cells = sqrtf(ml) * g.grid.inv_h * (1.0f + 1.0f / 1024.0f);
      const int R = cells >= (float)Rg ? Rg : min(Rg, 1 + (int)cells);
      const int NBx = g.qgrid.dim[0], NBy = g.qgrid.dim[1], B = g.qgrid.block;
      const int Dy = g.grid.dim[1], Dz = g.grid.dim[2];
      const int blk = sm.cell;
      const int bx = blk % NBx, by = (blk / NBx) % NBy, bz = blk / (NBx * NBy);
      const int x0 = max(bx * B - R, 0), x1 = min((bx + sm.span + 1) * B - 1 + R, D - 1);
      const int y0 = max(by * B - R, 0), y1 = min(by * B + B - 1 + R, Dy - 1);
      const int z0 = max(bz * B - R, 0), z1 = min(bz * B + B - 1 + R, Dz - 1);
      const int ny = y1 - y0 + 1, nrows = ny * (z1 - z0 + 1);
      if (tid == 0) sm.cand = 0;
      __syncthreads();
      unsigned long long cand = 0;
      for (int t = tid; t < nrows; t += NTG) {
        const int row = ((z0 + t / ny) * Dy + (y0 + t % ny)) * D;
        const int lo_r = __ldg(g.cstart + row + x0), hi_r = __ldg(g.cstart + row + x1 + 1);
        sm.range[t] = make_int2(lo_r, hi_r);
        cand += (unsigned long long)(hi_r - lo_r);
      }
      if (a.stats) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) cand += __shfl_xor_sync(0xffffffffu, cand, o);
        if (lane == 0) atomicAdd(&sm.cand, cand);
      }
      if (tid == 0) sm.nrange = nrows;
      __syncthreads();
      if (tid == 0) {
        if (a.stats) atomicAdd(a.stats + 3, sm.cand * (unsigned long long)sm.qn);
        // producer: first tiles of the item
        int r = 0, off = 0;
        for (int t = 0; t < STAGES; ++t) {
          while (r < nrows && sm.range[r].y == sm.range[r].x) ++r;
          if (r >= nrows) break;
          issue(sm, g, tc + t, r, off);
        }
      }
    }
    __syncthreads();
    const int nr = sm.nrange;
    // query groups of 32 slots this warp holds queries in (blocked slots)
    const int qv = rr ? max(0, min(Q, (qn - warp * 32 + NTG - 1) / NTG)) : max(0, min(Q, (qn - warp * 32 * Q + 31) / 32));
    float limc = 0.f;
#pragma unroll
    for (int q = 0; q < Q; ++q)
      if (q < qv) limc = fmaxf(limc, lim[q]);
    __syncwarp();

    // consumers: walk the same tile sequence as the producer
    int pr = 0, poff = 0;  // producer iterator (thread 0): STAGES tiles ahead
    if (tid == 0)
      for (int t = 0; t < STAGES; ++t) {  // mirror of the producer's first issues
        while (pr < nr && sm.range[pr].y == sm.range[pr].x) ++pr;
        if (pr >= nr) break;
        walk(sm, pr, poff);
      }
    int r = 0, off = 0;
    for (;;) {
      // skip empty rows (a tile never starts on one unless nothing is left)
      while (r < nr && sm.range[r].y == sm.range[r].x) ++r;
      if (r >= nr) break;
      const int s = (int)(tc % STAGES);
      mbar_wait(&sm.full[s], (tc / STAGES) & 1u);
      const float4* tile = sm.ring[s];
      const int cnt = walk(sm, r, off);
      // warps without queries in this item only keep the ring protocol; a warp
      // with 1-2 query groups holding queries computes two (the item's last warp
      // is usually partial: padded groups cost work and loosen the vote)
      // Three specialisations: four (3 or 4 groups hold queries), two and one (the
      // small round-robin items of spatial shards hold 1-2 groups per warp).  The
      // kernel's stall_no_inst (instruction fetch) grows with every copy: C5 k_grid
      // 1.82 ms with 4 copies, 1.72 with {4, 2}, 1.74 with {4, 2, 1}; a spatial
      // rank at 8 ranks 0.69 ms with {4, 2} (one-group warps padded to two), 0.57 here
      if (qv >= 3) grid_tile<4>(tile, cnt, pxy, pz, lim, limc, gq, sm.lists, warp, lane, rr, groups, slow_groups);
      else if (qv == 2) grid_tile<2>(tile, cnt, pxy, pz, lim, limc, gq, sm.lists, warp, lane, rr, groups, slow_groups);
      else if (qv == 1) grid_tile<1>(tile, cnt, pxy, pz, lim, limc, gq, sm.lists, warp, lane, rr, groups, slow_groups);
      // every thread releases the stage after its own reads (per-thread release
      // orders them before the stage's refill by the bulk copy; compute-sanitizer
      // racecheck does not count a __syncwarp before one lane's arrive as ordering)
      mbar_arrive(&sm.empty[s]);
      ++tc;
      if (tid == 0) {
        while (pr < nr && sm.range[pr].y == sm.range[pr].x) ++pr;
        if (pr < nr) issue(sm, g, tc + STAGES - 1, pr, poff);
      }
    }
    // lists are final: finish this thread's agents
    __syncwarp();
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const int slot = qslot(warp, q, lane, rr);
      if (slot < qn && qloc[q] < a.nloc) {
        key_t A[7];
#pragma unroll
        for (int s = 0; s < 7; ++s) A[s] = sm.lists[s * QBG + slot];
        finish_agent(a, qloc[q], A);
      }
    }
  }
  if (a.stats && lane == 0) {
    atomicAdd(a.stats, (unsigned long long)slow_groups);
    atomicAdd(a.stats + 1, (unsigned long long)groups);
  }
}

// Queries routed by k_grid (limit beyond the adjacent cells): one CTA per agent
// scans its own stencil -- the reach of its own limit -- with the exact
// brute-force test, per-thread top-7 lists merged by a shuffle butterfly and a
// shared-memory pass, then finishes the agent.
constexpr int FT = 128;
__global__ void __launch_bounds__(FT) k_grid_far(StepArgs a, GridArgs g) {
  __shared__ key_t wl[FT / 32][7];
  __shared__ int2 rng[(2 * 6 + 1) * (2 * 6 + 1)];  // (2 reach + 1)^2 rows, reach <= 6
  __shared__ int nrng;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nf = *g.fcount;
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  const float r2_in = __uint_as_float(__float_as_uint(r2) - 1u);
  const int D = g.grid.dim[0];
  for (int f = blockIdx.x; f < nf; f += gridDim.x) {
    const int qi = g.flist[f];
    const float4 me = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi));
    const int gi = (int)(a.lo + qi);
    const float lim = fminf(r2_in, g.flim[f]);  // computed once by k_grid when it routed the query
    if (tid == 0) {
      const int Rg = g.grid.reach;
      const float cells = sqrtf(lim) * g.grid.inv_h * (1.0f + 1.0f / 1024.0f);
      const int R = cells >= (float)Rg ? Rg : min(Rg, 1 + (int)cells);
      const float4 c4 = me;
      auto coord = [&](float v, int d) {
        const int c = (int)floorf((v - g.grid.lo[d]) * g.grid.inv_h);
        return c < 0 ? 0 : (c >= g.grid.dim[d] ? g.grid.dim[d] - 1 : c);
      };
      const int cx = coord(c4.x, 0), cy = coord(c4.y, 1), cz = coord(c4.z, 2);
      const int Dy = g.grid.dim[1], Dz = g.grid.dim[2];
      const int x0 = max(cx - R, 0), x1 = min(cx + R, D - 1);
      int nr = 0;
      for (int z = max(cz - R, 0); z <= min(cz + R, Dz - 1); ++z)
        for (int y = max(cy - R, 0); y <= min(cy + R, Dy - 1); ++y) {
          const int row = (z * Dy + y) * D;
          const int lo_r = g.cstart[row + x0], hi_r = g.cstart[row + x1 + 1];
          if (hi_r > lo_r) rng[nr++] = make_int2(lo_r, hi_r);
        }
      nrng = nr;
    }
    __syncthreads();
    key_t A[7];
#pragma unroll
    for (int s = 0; s < 7; ++s) A[s] = KEY_EMPTY;
    for (int r = 0; r < nrng; ++r)
      for (int k = rng[r].x + tid; k < rng[r].y; k += FT) {
        const float4 c = __ldg(g.spos + k);
        const float d2 = dist2(me.x, me.y, me.z, c);
        const int j = __float_as_int(c.w);
        if (d2 <= lim && j != gi) {
          const key_t key = make_key(d2, j);
          if (key < A[6]) insert7(A, key);
        }
      }
#pragma unroll
    for (int w = 1; w < 32; w <<= 1) {
      key_t B[7];
#pragma unroll
      for (int s = 0; s < 7; ++s) B[s] = __shfl_xor_sync(0xffffffffu, A[s], w);
      merge7(A, B);
    }
    if (lane == 0)
#pragma unroll
      for (int s = 0; s < 7; ++s) wl[warp][s] = A[s];
    __syncthreads();
    if (tid == 0) {
      for (int w = 1; w < FT / 32; ++w) {
        key_t B[7];
#pragma unroll
        for (int s = 0; s < 7; ++s) B[s] = wl[w][s];
        merge7(A, B);
      }
      finish_agent(a, qi, A);
    }
    __syncthreads();
  }
}

}  // namespace

cudaError_t launch_grid_far(const StepArgs& a, const GridArgs& g, cudaStream_t s) {
  if (!g.flist) return cudaSuccess;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  BOIDS_PREFER_SMEM(k_grid_far);
  k_grid_far<<<(unsigned)(4 * sms), FT, 0, s>>>(a, g);
  return cudaGetLastError();
}

cudaError_t launch_grid(const StepArgs& a, const GridArgs& g, cudaStream_t s) {
  static int grid = 0;
  if (!grid) {
    int dev = 0, sms = 148, r = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(k_grid, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&r, k_grid, NTG, 0);
    grid = sms * (r > 0 ? r : 1);
  }
  k_grid<<<grid, NTG, 0, s>>>(a, g);
  return cudaGetLastError();
}

// Queries per work item: QBG (512) for large query sets; fewer when the queries
// would make fewer than ~3 items per persistent CTA (a spatial shard's ~n/G
// owned agents), so every SM still gets several items (a block's queries are
// then split over items that share its stencil: the same pairs, more items).
int grid_chunk(int64_t nq) {
  int dev = 0, sms = 148, r = 5;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t ctas = (int64_t)sms * r;
  static const int force = [] {
    const char* e = getenv("BOIDS_GRID_CHUNK");  // diagnostics: queries per item
    return e ? atoi(e) : 0;
  }();
  if (force >= 32 && force <= QBG) return force;
  int64_t c = (nq / (3 * ctas) + 31) / 32 * 32;
  return (int)std::max<int64_t>(128, std::min<int64_t>(QBG, c));
}

}  // namespace boids
