// k_sym.cu -- the warm-step all-pairs hit scan evaluating every UNORDERED pair once
// (single-GPU handles; DESIGN.md sec 5 "k_sym").
//
// The distance is symmetric bit for bit: fl(a - b) = -fl(b - a) under round to
// nearest even, so d2(i, j) = ((dx*dx) + (dy*dy)) + (dz*dz) is the same float
// whichever agent is the query (the oracle pins this invariant).  A pair (i, j)
// evaluated once can therefore be tested against BOTH agents' warm limits: it
// is appended to i's hit buffer if d2 <= lim_i and to j's if d2 <= lim_j.  The
// hit set of every agent is exactly the one k_scan builds ({j != i : d2(i, j) <=
// lim_i}), so k_select (unchanged) returns the identical lists; the search
// evaluates n(n-1)/2 distances instead of n(n-1) and is still brute force in the
// thesis's sense (every pair is tested, Listing 5.2).
//
// Layout.  k_sym_prep writes the agents in spatial (Morton) order: sp[p] = (x, y,
// z, lim) of agent sidx[p], with lim = min(prev(r2), t0) the inclusive warm limit
// (the thread's own limit for its queries and the candidate's limit for the
// reverse test both come from the same array; phantoms p >= n have NaN positions
// and lim = -1).  Query block b holds sorted positions [b*QB, (b+1)*QB); its item
// space is the candidates [b*QB, npad):
//   * diagonal tiles [b*QB, (b+1)*QB): the block's 16 groups of 128 against
//     each other as a triangle -- groups (kc, w) with kc > w tested from both
//     sides, (w, w) from the query side only (self excluded by sorted position);
//   * off-diagonal tiles [(b+1)*QB, npad): both sides are tested.
// Stream-K: the triangular item space sum_b (npad - b*QB) is cut into equal
// contiguous ranges per CTA, as in k_scan.  Candidates and their original
// indices stream through a TMA ring (cp.async.bulk + mbarrier).
#include "cells.cuh"
#include "step_common.cuh"
#include "tma.cuh"

#include <cstdlib>

namespace boids {
namespace {

constexpr int Q = 4;        // queries per thread
constexpr int CT = 128;     // candidates per tile
#ifndef BOIDS_SYM_STAGES
#define BOIDS_SYM_STAGES 24
#endif
// TMA ring depth.  Deep on purpose: with queries AND candidates in spatial order,
// the slow path (passing pairs) of a tile concentrates in the 1-2 warps whose
// queries lie next to it -- on the diagonal, tile k is hot for warp k -- and a
// shallow ring couples every warp to the slowest one tile by tile (measured:
// 27% of stall samples spinning on the full barrier with 4 stages).  With a deep
// ring a warp can run STAGES-1 tiles ahead, so each warp's hot tiles only cost
// that warp.
constexpr int STAGES = BOIDS_SYM_STAGES;
// 256-thread CTAs run two per SM: the ring shrinks so two fit in shared memory
template <int NT>
__host__ __device__ constexpr int sym_stages() { return NT == 256 ? 12 : STAGES; }
constexpr int U = 4;        // candidates per record-emission subgroup (the slow path)
constexpr int UG = 8;       // candidates per warp vote (the fast path); item ranges are multiples of UG
constexpr int WB = Q * U * 32;  // records per warp buffer: one subgroup's maximum per side

struct __align__(8) Rec {
  int qi;  // local agent whose buffer receives the key
  int pad;
  key_t key;
};

// Ring stages hold a tile as structure of arrays (x[CT], y[CT], z[CT], lim[CT],
// index[CT]): a 16-byte shared load then gives four candidates' x (or y, z) --
// two packed pairs for FADD2 with the query's coordinate as a broadcast operand.
template <int NT>
struct __align__(16) SymSmem {
  float rx[sym_stages<NT>()][CT];
  float ry[sym_stages<NT>()][CT];
  float rz[sym_stages<NT>()][CT];
  float rw[sym_stages<NT>()][CT];
  int ridx[sym_stages<NT>()][CT];
  Rec rec[NT / 32][WB];
  int qg[NT / 32][Q * 32];    // each warp's current query group: agent indices ...
  float ql[NT / 32][Q * 32];  // ... and limits (read on the slow path only)
  uint64_t full[sym_stages<NT>()];
  int rel[sym_stages<NT>()];  // query groups done with the tile in the stage (the last one refills it)
  int next_unit;              // work queue of (tile, query group) units
};

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

// A 16-byte shared-memory load the compiler cannot merge with an earlier load of
// the same address: the slow path recomputes the fast path's distances from its
// own loads, so nothing of the fast path stays live (in registers) across the vote.
__device__ __forceinline__ float4 lds_fresh(const float* p) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "r"((unsigned)__cvta_generic_to_shared(p)));
  return v;
}

// Items before query block b: S(b) = sum_{b' < b} (npad - b'*QB).
__device__ __forceinline__ int64_t sym_prefix(int64_t b, int64_t npad, int64_t qb) {
  return b * npad - qb * (b * (b - 1) / 2);
}

// Append the passing keys of one vote group (bits over q*U+u) to the warp buffer.
// `side` 0: query side (buffer of the query, key index = candidate), 1: candidate side.
template <int SIDE>
__device__ __forceinline__ void emit(const StepArgs& a, Rec* rec, int& wcount, int lane, unsigned bits,
                                     const float (&d)[Q][U], const int (&gq)[Q], const int* cidx) {
  // exclusive prefix of the per-lane record counts (0..16) from 5 independent
  // ballots on their bits: no dependent shuffle chain on this path
  const int nrec = __popc(bits);
  const unsigned lt = (1u << lane) - 1u;
  int excl = 0, total = 0;
#pragma unroll
  for (int k = 0; k < 5; ++k) {
    const unsigned bk = __ballot_sync(0xffffffffu, (nrec >> k) & 1);
    excl += __popc(bk & lt) << k;
    total += __popc(bk) << k;
  }
  if (total == 0) return;
  if (wcount + total > WB) {  // warp-uniform; total <= WB always
    __syncwarp();
    flush(a, rec, wcount, lane);
    __syncwarp();
    wcount = 0;
  }
  int off = wcount + excl;
#pragma unroll
  for (int q = 0; q < Q; ++q)
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (bits & (1u << (q * U + u))) {
        if (SIDE == 0) {
          rec[off].qi = gq[q];
          rec[off].key = make_key(d[q][u], cidx[u]);
        } else {
          rec[off].qi = cidx[u];
          rec[off].key = make_key(d[q][u], gq[q]);
        }
        ++off;
      }
  wcount += total;
}

// Stream-K split with weights: a diagonal item (query side only, but where most
// passing pairs -- the slow path -- are, since a query block is spatially
// compact) costs wd4/4 of an off-diagonal one.  Row b has weighted length
// 4*(npad - b*QB) + (wd4 - 4)*QB; CTA i gets the items of the weighted range
// [i*W/grid, (i+1)*W/grid), rounded to multiples of U.
__device__ __forceinline__ int64_t sym_split(int64_t i, int64_t grid, int64_t npad, int64_t qb, int wd4) {
  const int64_t nb = npad / qb;
  auto sw = [&](int64_t b) { return 4 * sym_prefix(b, npad, qb) + (int64_t)(wd4 - 4) * qb * b; };
  const int64_t W = sw(nb);
  if (i >= grid) return sym_prefix(nb, npad, qb);
  const int64_t x = (int64_t)((__int128)W * i / grid);
  int64_t lo = 0, hi = nb - 1;  // largest b with sw(b) <= x
  while (lo < hi) {
    const int64_t mid = (lo + hi + 1) / 2;
    if (sw(mid) <= x) lo = mid; else hi = mid - 1;
  }
  const int64_t o = x - sw(lo), dw = (int64_t)wd4 * qb;
  const int64_t off = o < dw ? o / wd4 : qb + (o - dw) / 4;
  return (sym_prefix(lo, npad, qb) + off) / UG * UG;
}

// Feedback split (BOIDS_OPT_BALANCE).  The cost of an item is not uniform: the
// slow path (passing pairs) concentrates where queries and candidates are near
// each other in space -- on and next to the diagonal of a spatially sorted flock
// -- and its weight depends on the flock's density.  The previous launch measured
// every CTA's SM time for its range [L0_j, L1_j); read as a piecewise-constant
// cost density over the item space, it gives a cumulative cost C(x), and CTA i
// takes [C^-1(i T / G), C^-1((i + 1) T / G)), T = C(total), rounded to U.  The
// flock moves little per step, so the density carries over.  Only the partition
// changes, never a result.  Without a usable record (first launch, another
// launch shape) the static weighted split (sym_split) is used.
//
// k_sym_prep's block 0 computes all G + 1 boundaries into `splits` (one
// thread per boundary, binary search over a shared-memory prefix of the costs),
// off k_sym's critical path: k_sym's CTAs then read their two boundaries.
// [lo, hi): the item sub-range this launch covers (the whole triangle on a single
// GPU; a rank's share of it with sym-shards, k_ss_*); the record's "total" is
// the whole triangle's length, its CTA ranges are absolute item positions, and it
// is used only if its first and last CTA ranges start at lo and end at hi.
__device__ void compute_splits(const long long* __restrict__ fb, int G, int64_t lo, int64_t hi, int64_t npad,
                               int64_t qb, int wd4, long long* __restrict__ splits) {
  __shared__ double pre[SYM_FB_MAX_CTAS];
  __shared__ double wsum[32];
  __shared__ int ok;
  const int64_t total = hi - lo;
  const bool whole = lo == 0 && hi == sym_prefix(npad / qb, npad, qb);
  const int tid = threadIdx.x, nt = blockDim.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0)
    ok = fb != nullptr && G <= SYM_FB_MAX_CTAS && fb[0] == G && fb[1] == sym_prefix(npad / qb, npad, qb) &&
         fb[2] == lo && fb[3 * G] == hi;
  __syncthreads();
  if (ok) {  // inclusive prefix of the measured CTA costs (block scan over per-thread chunks)
    const int per = (G + nt - 1) / nt, j0 = min(G, tid * per), j1 = min(G, j0 + per);
    double own = 0.0;
    for (int j = j0; j < j1; ++j) own += (double)fb[4 + 3 * j];
    double incl = own;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const double v = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += v;
    }
    if (lane == 31) wsum[warp] = incl;
    __syncthreads();
    double woff = 0.0;
    for (int w = 0; w < warp; ++w) woff += wsum[w];
    double run = woff + incl - own;
    for (int j = j0; j < j1; ++j) {
      run += (double)fb[4 + 3 * j];
      pre[j] = run;
    }
    __syncthreads();
    if (tid == 0 && !(pre[G - 1] > 0.0)) ok = 0;
    __syncthreads();
  }
  const double T = ok ? pre[G - 1] : 0.0;
  for (int k = tid; k <= G; k += nt) {
    int64_t x;
    if (k == 0) {
      x = lo;
    } else if (k == G) {
      x = hi;
    } else if (ok) {
      const double c = T * (double)k / (double)G;
      int jl = 0, jh = G - 1;  // first j with pre[j] > c
      while (jl < jh) {
        const int mid = (jl + jh) >> 1;
        if (pre[mid] > c) jh = mid; else jl = mid + 1;
      }
      const double t = (double)fb[4 + 3 * jl], cum = pre[jl] - t;
      const int64_t a0 = fb[2 + 3 * jl], a1 = fb[3 + 3 * jl];
      x = t > 0.0 ? a0 + (int64_t)((c - cum) / t * (double)(a1 - a0)) : a0;
      x = x / UG * UG;
      x = x < lo ? lo : (x > hi ? hi : x);
    } else if (whole) {
      x = sym_split(k, G, npad, qb, wd4);
    } else {  // a sub-range without a record: equal item shares
      x = lo + (int64_t)((__int128)total * k / G) / UG * UG;
    }
    splits[k] = x;
  }
}

// Tile k of a CTA whose item range is [L0, L1): items [max(L0, A + k*CT), min(L1,
// A + (k+1)*CT)) with A = L0 rounded down to CT.  Rows (npad - b*QB items) and
// their starts S(b) are multiples of CT, so a tile never straddles two rows.
struct TileDesc {
  int64_t b;   // query block (row)
  int64_t jb;  // first candidate (sorted position)
  int cnt;     // candidates (multiple of U)
};
__device__ __forceinline__ TileDesc tile_desc(int k, int64_t L0, int64_t L1, int64_t npad, int64_t qb) {
  const int64_t A = L0 / CT * CT;
  const int64_t Ls = max(L0, A + (int64_t)k * CT), Le = min(L1, A + (int64_t)(k + 1) * CT);
  // row: largest b with S(b) <= Ls; S is increasing and concave -> solve in fp32
  // (a few ulps off at most: the integer fix-ups below make it exact), then fix up
  const float nb2 = (float)npad / (float)qb + 0.5f;
  int64_t b = (int64_t)(nb2 - sqrtf(fmaxf(0.f, nb2 * nb2 - 2.f * (float)Ls / (float)qb)));
  b = b < 0 ? 0 : b;
  while (b > 0 && sym_prefix(b, npad, qb) > Ls) --b;
  while (sym_prefix(b + 1, npad, qb) <= Ls) ++b;
  return TileDesc{b, b * qb + (Ls - sym_prefix(b, npad, qb)), (int)(Le - Ls)};
}

template <int NTS>
__global__ void __launch_bounds__(NTS, NTS == 128 ? 4 : (NTS == 256 ? 2 : 1))
    k_sym(StepArgs a, const float* __restrict__ spf, int64_t cap, const int* __restrict__ sidx, int64_t npad,
          const long long* __restrict__ splits, long long* __restrict__ fb_cur) {
  constexpr int QBS = NTS * Q, NW = NTS / 32, SST = sym_stages<NTS>();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  SymSmem<NTS>& sm = *reinterpret_cast<SymSmem<NTS>*>(smem_raw);
  __shared__ int64_t s_range[2];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  pdl_wait();  // k_sym_prep's sp / limits (and the previous launch's feedback record)
  __shared__ long long s_cstart;
  __shared__ unsigned long long s_tw[NTS / 32], s_ts[NTS / 32];  // diagnostics (a.phase): per-warp wait / emit cycles
  if (tid == 0) s_cstart = clock64();
  if (tid < NTS / 32) s_tw[tid] = s_ts[tid] = 0;
  const int64_t total = sym_prefix(npad / QBS, npad, QBS);
  if (tid < 2) s_range[tid] = splits[blockIdx.x + tid];  // k_sym_prep's boundaries (compute_splits)
  __syncthreads();
  const int64_t L0 = s_range[0], L1 = s_range[1];
  const int ntiles = L1 > L0 ? (int)((L1 + CT - 1) / CT - L0 / CT) : 0;
  // Work units.  Unit u = (tile k = u / NW, query group w = u % NW): the 128
  // candidates of tile k against the 4 x 32 queries [w*128, (w+1)*128) of tile
  // k's query block.  Warps take units from a shared counter, in order, instead
  // of each warp owning one query group: the slow path of a tile (passing pairs,
  // record emission) concentrates in the query group next to it in space -- on
  // the diagonal, tile k is hot for group k only -- and with fixed groups that
  // one warp set the CTA's end while the others waited at the final barrier
  // (C3: stall_barrier 20 % of samples).  Taken dynamically, hot units spread
  // over whichever warps are free.
  //
  // Ring protocol: stage s = k % SST holds tile k.  full[s] completes when the
  // tile's bytes land (TMA complete_tx).  Each finished unit of tile k
  // increments rel[s]; the unit that completes the tile's NW query groups
  // refills the stage with tile k + SST.  A warp takes a new unit only after
  // finishing its current one, so at most NW units are open: a unit of tile
  // k + SST can only be taken once tile k's units are all taken, and its wait
  // on full[s] (parity of k + SST) cannot be satisfied by tile k's phase.
  auto issue = [&](int k) {
    const TileDesc d = tile_desc(k, L0, L1, npad, QBS);
    const int s = k % SST;
    const uint32_t n = (uint32_t)d.cnt;
    mbar_arrive_expect_tx(&sm.full[s], n * 20u);
    tma_load_1d(sm.rx[s], spf + d.jb, n * 4u, &sm.full[s]);
    tma_load_1d(sm.ry[s], spf + cap + d.jb, n * 4u, &sm.full[s]);
    tma_load_1d(sm.rz[s], spf + 2 * cap + d.jb, n * 4u, &sm.full[s]);
    tma_load_1d(sm.rw[s], spf + 3 * cap + d.jb, n * 4u, &sm.full[s]);
    tma_load_1d(sm.ridx[s], sidx + d.jb, n * 4u, &sm.full[s]);
  };
  if (tid == 0) {
    if (a.phase) {  // diagnostics: [0] start, [1] end (%globaltimer), [2] L0, [3] L1, [4] slow groups
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      a.phase[blockIdx.x * 8 + 0] = t;
      a.phase[blockIdx.x * 8 + 2] = (unsigned long long)L0;
      a.phase[blockIdx.x * 8 + 3] = (unsigned long long)L1;
      a.phase[blockIdx.x * 8 + 4] = 0;
      a.phase[blockIdx.x * 8 + 5] = 0;
      a.phase[blockIdx.x * 8 + 6] = 0;
    }
#pragma unroll
    for (int s = 0; s < SST; ++s) {
      mbar_init(&sm.full[s], 1);
      sm.rel[s] = 0;
    }
    sm.next_unit = 0;
    mbar_fence_init();
  }
  if (warp == 0) {  // the first SST tiles, one lane each
    __syncwarp();
    for (int k = lane; k < SST && k < ntiles; k += 32) issue(k);
  }
  __syncthreads();
  Rec* rec = sm.rec[warp];
  int wcount = 0;
  unsigned slow_groups = 0;
  int cur_b = -1;
  int cur_w = -1;
  float px[Q], py[Q], pz[Q], limq = 0.f;
  int qbase = 0;  // sorted position of the thread's query 0 (query q: qbase + 32 q)
  int* wqg = sm.qg[warp];
  float* wql = sm.ql[warp];
  const float INF = __int_as_float(0x7f800000);
  const int nunits = ntiles * NW;
  for (;;) {
    int u = 0;
    if (lane == 0) u = atomicAdd(&sm.next_unit, 1);
    u = __shfl_sync(0xffffffffu, u, 0);
    if (u >= nunits) break;
    const int k = u / NW, wq = u - k * NW;
    // the range is re-read from shared memory per unit: keeping L0 / L1 (int64)
    // live in registers across the pair loop cost the fast path spills
    const TileDesc td = tile_desc(k, *(volatile int64_t*)&s_range[0], *(volatile int64_t*)&s_range[1], npad, QBS);
    if ((int)td.b != cur_b || wq != cur_w) {  // query group wq of row b: 4 x 32 spatially compact queries
      cur_b = (int)td.b;
      cur_w = wq;
      qbase = cur_b * QBS + wq * 32 * Q + lane;
      float lq[Q];
      __syncwarp();  // the previous group's slow path is done with wqg / wql
#pragma unroll
      for (int q = 0; q < Q; ++q) {
        const int p = qbase + q * 32;
        wqg[q * 32 + lane] = __ldg(sidx + p);
        px[q] = __ldg(spf + p);
        py[q] = __ldg(spf + cap + p);
        pz[q] = __ldg(spf + 2 * cap + p);
        lq[q] = __ldg(spf + 3 * cap + p);
        wql[q * 32 + lane] = lq[q];
      }
      limq = fmaxf(fmaxf(lq[0], lq[1]), fmaxf(lq[2], lq[3]));
    }
    const int s = k % SST;
    long long tw0 = 0;
    if (a.phase) tw0 = clock64();
    mbar_wait(&sm.full[s], (uint32_t)(k / SST) & 1u);
    if (a.phase && lane == 0) s_tw[warp] += clock64() - tw0;
    {
      const float* tx = sm.rx[s];
      const float* ty = sm.ry[s];
      const float* tz = sm.rz[s];
      const float* tw = sm.rw[s];
      const int* tidx = sm.ridx[s];
      const int jb = (int)td.jb;
      const int cnt = td.cnt;  // a multiple of UG
      const bool diag = td.jb < (cur_b + 1) * QBS;  // candidates of the query block itself
      // d2 of query q to candidates (c + 2p, c + 2p + 1), reading Q3: the x, y, z
      // differences of the two pairs in one FADD2 each (query coordinate broadcast),
      // their squares in one FMUL2 each, the sums ((dx dx) + (dy dy)) + (dz dz) scalar
      // -- never a packed add of packed products, which ptxas would contract into FFMA2.
      auto dist_pair = [&](int q, float4 X, float4 Y, float4 Z, int hi, float& d0, float& d1) {
        const float2 cx = hi ? make_float2(X.z, X.w) : make_float2(X.x, X.y);
        const float2 cy = hi ? make_float2(Y.z, Y.w) : make_float2(Y.x, Y.y);
        const float2 cz = hi ? make_float2(Z.z, Z.w) : make_float2(Z.x, Z.y);
        const float2 dx = __fadd2_rn(make_float2(px[q], px[q]), make_float2(-cx.x, -cx.y));
        const float2 dy = __fadd2_rn(make_float2(py[q], py[q]), make_float2(-cy.x, -cy.y));
        const float2 dz = __fadd2_rn(make_float2(pz[q], pz[q]), make_float2(-cz.x, -cz.y));
        const float2 x2 = __fmul2_rn(dx, dx), y2 = __fmul2_rn(dy, dy), z2 = __fmul2_rn(dz, dz);
        d0 = __fadd_rn(__fadd_rn(x2.x, y2.x), z2.x);
        d1 = __fadd_rn(__fadd_rn(x2.y, y2.y), z2.y);
      };
      // Slow path of one subgroup of U = 4 candidates (c .. c+3): recompute its
      // 16 distances (the same arithmetic, so the same floats as the fast path),
      // test them against the exact limits, append the passing keys.
      auto slow4 = [&](const int c, auto diag_c) {
        constexpr bool DIAG = decltype(diag_c)::value;
        const float4 X = lds_fresh(tx + c);
        const float4 Y = lds_fresh(ty + c);
        const float4 Z = lds_fresh(tz + c);
        const float4 W = lds_fresh(tw + c);
        const float cw[U] = {W.x, W.y, W.z, W.w};
        float d[Q][U];
#pragma unroll
        for (int q = 0; q < Q; ++q) {
          dist_pair(q, X, Y, Z, 0, d[q][0], d[q][1]);
          dist_pair(q, X, Y, Z, 1, d[q][2], d[q][3]);
        }
        int cidx[U], gq[Q];
        float lim[Q];
#pragma unroll
        for (int u = 0; u < U; ++u) cidx[u] = tidx[c + u];
#pragma unroll
        for (int q = 0; q < Q; ++q) {
          gq[q] = wqg[q * 32 + lane];
          lim[q] = wql[q * 32 + lane];
        }
        unsigned qb = 0, cb = 0;
#pragma unroll
        for (int q = 0; q < Q; ++q)
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (d[q][u] <= lim[q] && (!DIAG || jb + c + u != qbase + q * 32)) qb |= 1u << (q * U + u);
            if (!DIAG && d[q][u] <= cw[u]) cb |= 1u << (q * U + u);
          }
        long long ts0 = 0;
        if (a.phase) ts0 = clock64();
        emit<0>(a, rec, wcount, lane, qb, d, gq, cidx);
        if (!DIAG) emit<1>(a, rec, wcount, lane, cb, d, gq, cidx);
        if (a.phase && lane == 0) s_ts[warp] += clock64() - ts0;
      };
      // Fast path of one vote group of UG = 8 candidates: only the minimum of the
      // 32 distances per lane, against the largest limit that could accept a pair
      // (the thread's queries', and on off-diagonal tiles the candidates' too);
      // one warp vote -- nearly always false -- decides whether the slow path runs.
      auto group = [&](const int c, auto diag_c) {
        constexpr bool DIAG = decltype(diag_c)::value;
        const float4 X0 = *reinterpret_cast<const float4*>(tx + c);
        const float4 X1 = *reinterpret_cast<const float4*>(tx + c + 4);
        const float4 Y0 = *reinterpret_cast<const float4*>(ty + c);
        const float4 Y1 = *reinterpret_cast<const float4*>(ty + c + 4);
        const float4 Z0 = *reinterpret_cast<const float4*>(tz + c);
        const float4 Z1 = *reinterpret_cast<const float4*>(tz + c + 4);
        float mq[Q];
#pragma unroll
        for (int q = 0; q < Q; ++q) {
          float e0, e1, e2, e3, e4, e5, e6, e7;
          dist_pair(q, X0, Y0, Z0, 0, e0, e1);
          dist_pair(q, X0, Y0, Z0, 1, e2, e3);
          dist_pair(q, X1, Y1, Z1, 0, e4, e5);
          dist_pair(q, X1, Y1, Z1, 1, e6, e7);
          mq[q] = fminf(fminf(fminf(e0, e1), fminf(e2, e3)), fminf(fminf(e4, e5), fminf(e6, e7)));
        }
        const float m = fminf(fminf(mq[0], mq[1]), fminf(mq[2], mq[3]));  // NaN (phantoms) ignored
        float thr = limq;
        if (!DIAG) {
          const float4 W0 = *reinterpret_cast<const float4*>(tw + c);
          const float4 W1 = *reinterpret_cast<const float4*>(tw + c + 4);
          thr = fmaxf(fmaxf(fmaxf(thr, fmaxf(W0.x, W0.y)), fmaxf(W0.z, W0.w)),
                      fmaxf(fmaxf(W1.x, W1.y), fmaxf(W1.z, W1.w)));
        }
        if (__any_sync(0xffffffffu, m <= thr)) {  // rare, warp-uniform
          ++slow_groups;
#pragma unroll 1
          for (int c4 = c; c4 < c + UG; c4 += U) slow4(c4, diag_c);
        }
      };
      if (!diag && cnt == CT) {  // full off-diagonal tile: constant trip count (the common case)
#pragma unroll 1
        for (int c = 0; c < CT; c += UG) group(c, std::false_type{});
      } else {
        // Diagonal tile (candidates of the query block itself): the block's pairs are
        // symmetric too.  Candidate group kc (block positions [kc*128, kc*128 + 128), the
        // positions of query group kc) against query group wq: kc > wq -- both sides,
        // like an off-diagonal tile; kc == wq -- the group with itself, query side only
        // (self excluded); kc < wq -- skipped: unit (kc, wq) evaluates those pairs.  Every
        // unordered pair of the block is evaluated once (UG divides 128).  kc grows with
        // c, so the three cases are three contiguous candidate ranges of the tile.
        int ce = 0, co = 0;  // [ce_start, ce) query-side-only range, [co, cnt) both sides
        int cs = 0;
        if (diag) {
          const int rel0 = jb - cur_b * QBS;
          cs = min(max(wq * 32 * Q - rel0, 0), cnt);
          ce = co = min(max((wq + 1) * 32 * Q - rel0, 0), cnt);
        }
        for (int c = cs; c < ce; c += UG) group(c, std::true_type{});
        for (int c = co; c < cnt; c += UG) group(c, std::false_type{});
      }
    }
    __syncwarp();
    if (lane == 0) {  // this query group is done with stage s; the tile's last one refills it
      __threadfence_block();
      const int old = atomicAdd(&sm.rel[s], 1);
      if (old == NW - 1) {
        sm.rel[s] = 0;
        __threadfence_block();
        if (k + SST < ntiles) {
          fence_proxy_async_smem();
          issue(k + SST);
        }
      }
    }
  }
  __syncwarp();
  flush(a, rec, wcount, lane);
  if (fb_cur) {  // this CTA's range and SM time: the next launch's split (compute_splits)
    __syncthreads();
    if (tid == 0) {
      fb_cur[2 + 3 * blockIdx.x] = L0;
      fb_cur[3 + 3 * blockIdx.x] = L1;
      fb_cur[4 + 3 * blockIdx.x] = clock64() - s_cstart;
      if (blockIdx.x == 0) {
        fb_cur[0] = gridDim.x;
        fb_cur[1] = total;  // the whole triangle's length (the record's CTA 0 range starts the covered sub-range)
      }
    }
  }
  if (a.stats && lane == 0) {
    atomicAdd(a.stats, (unsigned long long)slow_groups);
    // vote groups: every candidate item of the range meets every query group, UG candidates per vote
    if (warp == 0) atomicAdd(a.stats + 1, (unsigned long long)((L1 - L0) / UG * NW));
  }
  if (a.phase) {
    if (lane == 0) {
      atomicAdd(a.phase + blockIdx.x * 8 + 4, (unsigned long long)slow_groups);
      atomicMax(a.phase + blockIdx.x * 8 + 5, s_tw[warp]);  // [5] max wait cycles of a warp
      atomicMax(a.phase + blockIdx.x * 8 + 6, s_ts[warp]);  // [6] max emit cycles of a warp
      if (warp == 0) a.phase[blockIdx.x * 8 + 7] = s_tw[0];  // [7] warp 0 wait
    }
    __syncthreads();
    if (tid == 0) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      a.phase[blockIdx.x * 8 + 1] = t;
    }
  }
}

// t0 of local agent qi (see k_warm.cu warm_t0): 7th smallest current d2 to the
// previous 7 neighbours and the previous 8th nearest; +inf without 7.
__device__ __forceinline__ float sym_t0(const StepArgs& a, int64_t qi, float4 me, int& c) {
  int nb[8];
#pragma unroll
  for (int k = 0; k < 7; ++k) nb[k] = __ldg(a.nbr + qi * 7 + k);
  nb[7] = __ldg(a.nbr8 + qi);
  c = __ldg(a.cnt + qi);
  float4 p[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) p[k] = __ldg(pos_of(a.full, a.m, a.sdiv, nb[k] < 0 ? 0 : nb[k]));
  float m1 = 0.f, m2 = 0.f;
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const float d = (k < 7 || nb[7] >= 0) ? dist2(me.x, me.y, me.z, p[k]) : 0.f;
    m2 = fmaxf(m2, fminf(m1, d));
    m1 = fmaxf(m1, d);
  }
  if (c < 7) return __int_as_float(0x7f800000);
  return nb[7] >= 0 ? m2 : m1;
}

// A second bound for an agent whose previous neighbours no longer bound it (t0
// > r2: it wrapped to the diametric opposite point, or its neighbours
// did): the 7th smallest current d2 to the agents around its cell in the
// last spatial sort (WIN of them; qperm is in Morton order of the locality grid; lstart the
// cells' starts), self excluded.  They are real, distinct agents, so it is an
// upper bound on the 7th key like t0; +inf with fewer than 7 of them.  The
// sort is up to BOIDS_OPT_RESORT steps old: only the bound's tightness depends
// on that, never the result.
constexpr int WIN = 256;  // C4: 64 -> 11 routed agents per step, 256 -> 3 (route 32 -> 22 us, prep +17 us; net -0.5..1 %)
// The window over an explicit order: perm[0..n) agent indices (offset by base
// into the position buffer) in Morton order of grid g, start[c] = the first
// position of cell c; self = the querying agent's own index in perm's terms.
// The bound is computed by the whole warp for each lane that needs it
// (`need`; every lane of the warp calls this): the WIN window agents are split
// over the 32 lanes (WIN / 32 gathers each, all in flight at once), each lane
// keeps its 7 smallest d2, and the 7th smallest of the warp comes from seven
// warp-minimum extractions -- one gather round trip per needing agent instead
// of WIN / 16 dependent rounds in one thread (round 2's serial version set
// k_sym_prep's time: C4 46 us for a handful of agents).  Agents this handle
// does not hold (NaN) are skipped, never counted.
__device__ float window_bound_warp(const StepArgs& a, const int* __restrict__ perm, const int* __restrict__ start,
                                   const BinGrid& g, int n, int64_t base, int64_t self, float4 me, bool need) {
  const int lane = threadIdx.x & 31;
  const float INF = __int_as_float(0x7f800000);
  float out = INF;
  unsigned todo = __ballot_sync(0xffffffffu, need);
  while (todo) {
    const int src = __ffs(todo) - 1;
    todo &= todo - 1;
    const float mx = __shfl_sync(0xffffffffu, me.x, src), my = __shfl_sync(0xffffffffu, me.y, src),
                mz = __shfl_sync(0xffffffffu, me.z, src);
    const long long sf = __shfl_sync(0xffffffffu, (long long)self, src);
    if (!start || !perm || n < 8 || !(mx == mx && my == my && mz == mz)) continue;  // warp-uniform: +inf
    const float4 m4 = make_float4(mx, my, mz, 0.f);
    const int p0 = __ldg(start + cell_of(m4, g));
    int lo = p0 - WIN / 2;
    lo = lo > n - WIN ? n - WIN : lo;
    lo = lo < 0 ? 0 : lo;
    const int hi = lo + WIN < n ? lo + WIN : n;
    constexpr int PER = WIN / 32;
    int j[PER];
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int pos = lo + k * 32 + lane;
      j[k] = pos < hi ? __ldg(perm + pos) : -1;
    }
    float4 q[PER];
#pragma unroll
    for (int k = 0; k < PER; ++k) q[k] = __ldg(pos_of(a.full, a.m, a.sdiv, base + (j[k] < 0 ? 0 : j[k])));
    float b[7];
#pragma unroll
    for (int t = 0; t < 7; ++t) b[t] = INF;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      if (j[k] < 0 || j[k] == sf) continue;
      float d = dist2(mx, my, mz, q[k]);
      if (!(d == d)) continue;  // an agent this handle does not hold
#pragma unroll
      for (int t = 0; t < 7; ++t) {  // keep the 7 smallest, ascending
        const float l = fminf(b[t], d);
        d = fmaxf(b[t], d);
        b[t] = l;
      }
    }
    // 7 extractions of the warp minimum (d2 >= 0: its bits order like the value;
    // ties broken by lane, so exactly one lane pops per round)
    float kth = INF;
#pragma unroll 1
    for (int t = 0; t < 7; ++t) {
      const unsigned hb = __float_as_uint(b[0]);
      const unsigned mb = __reduce_min_sync(0xffffffffu, hb);
      kth = __uint_as_float(mb);
      const unsigned who = __reduce_min_sync(0xffffffffu, hb == mb ? (unsigned)lane : 32u);
      if (lane == (int)who) {
#pragma unroll
        for (int s2 = 0; s2 < 6; ++s2) b[s2] = b[s2 + 1];
        b[6] = INF;
      }
    }
    if (lane == src) out = kth;
  }
  return out;
}

// Structure of arrays over the sorted positions p: spf[p], spf[cap + p], spf[2 cap + p] = x, y, z and
// spf[3 cap + p] = min(prev(r2), t0) of agent sidx[p] = qperm[p]; phantoms beyond nloc.
// An agent whose previous 7 neighbours are all out of range now (t0 >= r2 with a
// full previous list: it wrapped to the far side of the world) would append
// every in-radius pair -- hundreds -- to its hit buffer.  It is ROUTED instead:
// limit -1 (no hits on either side in k_sym) and searched whole by k_route.
__device__ __forceinline__ void sym_prep_body(const StepArgs& a, float* __restrict__ spf, int64_t cap,
                                              int* __restrict__ sidx, int64_t npad) {
  const int64_t p = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (p >= npad) return;  // (npad is a multiple of 256: whole warps)
  const bool real = p < a.nloc;  // else a phantom slot: NaN position, limit -1
  const int qi = real ? (a.qperm ? __ldg(a.qperm + p) : (int)p) : 0;
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  const float r2_in = __uint_as_float(__float_as_uint(r2) - 1u);  // d2 < r2  <=>  d2 <= r2_in
  const float nan = __int_as_float(0x7fc00000);
  const float4 me = real ? __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi)) : make_float4(nan, nan, nan, 0.f);
  int c = 0;
  const float t0 = real ? sym_t0(a, qi, me, c) : 0.f;
  float lim = fminf(r2_in, t0);
  // every lane of the warp takes part in the warp's window bounds
  const float wb = window_bound_warp(a, a.qperm, a.lstart, a.loc, (int)a.nloc, a.lo, qi, me, real && t0 > r2_in);
  if (real && t0 > r2_in) lim = fminf(lim, wb);
  if (real && c == 7 && lim > r2_in && a.rlist) {
    a.rlist[atomicAdd(a.rcount, 1)] = qi;
    a.routed[qi] = 1;
    if (a.stats) atomicAdd(a.stats + 2, 1ull);
    lim = -1.f;
  }
  spf[p] = me.x;
  spf[cap + p] = me.y;
  spf[2 * cap + p] = me.z;
  spf[3 * cap + p] = real ? lim : -1.f;
  sidx[p] = real ? qi : -1;
}

__global__ void __launch_bounds__(256) k_sym_prep(StepArgs a, float* __restrict__ spf, int64_t cap,
                                                   int* __restrict__ sidx, int64_t npad, int64_t qb, int G, int wd4,
                                                   const long long* __restrict__ fb_prev,
                                                   long long* __restrict__ splits) {
  pdl_trigger();  // k_sym may be scheduled now; it waits for this grid before reading sp
  span_begin(a, SPAN_SLOT0 + 0);
  if (blockIdx.x == gridDim.x - 1)  // the last block (fewest real agents) also cuts k_sym's work
    compute_splits(fb_prev, G, 0, sym_prefix(npad / qb, npad, qb), npad, qb, wd4, splits);
  sym_prep_body(a, spf, cap, sidx, npad);
  span_end(a, SPAN_SLOT0 + 0);
}

// Routed agents (k_sym_prep): one CTA per agent searches all candidates (Listing
// 5.2: every agent, index order irrelevant under the (d2, index) key), keeping the
// 8 smallest keys per thread; a shuffle butterfly and a shared-memory pass merge
// them.  The CTA then finishes the agent -- list, 8th nearest (the next step's
// warm-bound seed), steering, modification -- and k_select skips it.
// The 8 smallest keys over the warp's 32 ascending 8-lists (keys unique across
// lanes), ascending, in every lane: extract the warp minimum of the list heads
// (two 32-bit min reductions: d2 bits, then the index among the lanes holding
// that d2) and pop it from its lane, up to 8 times, stopping at the first empty
// minimum.  k_route's lists are nearly empty (a routed agent has few agents
// within r, and they are spread over 512 threads x P parts), so this takes a
// round or two where a shuffle butterfly of merge8 networks took five full
// levels (C4 sym-shards, 8 ranks: k_route 66 us, most of it merging).
__device__ __forceinline__ void warp_top8(key_t (&A)[8], key_t (&out)[8]) {
#pragma unroll
  for (int t = 0; t < 8; ++t) out[t] = KEY_EMPTY;
#pragma unroll 1
  for (int t = 0; t < 8; ++t) {
    const unsigned hi = (unsigned)(A[0] >> 32), lo = (unsigned)A[0];
    const unsigned mhi = __reduce_min_sync(0xffffffffu, hi);
    const unsigned mlo = __reduce_min_sync(0xffffffffu, hi == mhi ? lo : 0xffffffffu);
    const key_t m = ((key_t)mhi << 32) | mlo;
    if (m == KEY_EMPTY) break;  // warp-uniform
#pragma unroll
    for (int s = 0; s < 8; ++s)
      if (s == t) out[s] = m;
    if (A[0] == m) {  // the one lane holding it pops its head
#pragma unroll
      for (int s = 0; s < 7; ++s) A[s] = A[s + 1];
      A[7] = KEY_EMPTY;
    }
  }
}

constexpr int RT = 512, RU = 16;
constexpr int RP_MAX = 16;  // candidate parts per routed agent (few routed agents -> more CTAs each)
__device__ __forceinline__ void route_body(const StepArgs& a) {
  __shared__ key_t wl[RT / 32][8];
  __shared__ int s_last;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nr = *a.rcount;
  if (nr <= 0) return;
  // P parts per agent so that a handful of routed agents still fills the GPU;
  // the CTA that finishes an agent's last part merges the parts' top-8 lists
  const int P = a.rpart ? max(1, min(RP_MAX, (int)(2 * gridDim.x / nr))) : 1;
  const int64_t total = (int64_t)a.world * a.m;           // candidate slots (slot t = agent t)
  const int64_t chunk = ((total + P - 1) / P + RT - 1) / RT * RT;
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  for (int w = blockIdx.x; w < nr * P; w += gridDim.x) {
    const int r = w / P, part = w - r * P;
    const int qi = a.rlist[r];
    const float4 me = __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + qi));
    const int g = (int)(a.lo + qi);
    key_t A[8];
#pragma unroll
    for (int s = 0; s < 8; ++s) A[s] = KEY_EMPTY;
    // slice by slice within this part (no per-candidate slice division); 16
    // independent loads in flight per thread: the candidates are L2-resident
    // and this loop is latency-bound
    const int64_t c0 = part * chunk, c1 = min(total, c0 + chunk);
    for (int64_t sl = c0 / a.m; sl * a.m < c1; ++sl) {
      const float4* base = a.full + sl * 2 * a.m;
      const int jg0 = (int)(sl * a.m);
      const int jlo = (int)(max(c0, sl * a.m) - sl * a.m), jhi = (int)(min(c1, (sl + 1) * a.m) - sl * a.m);
      for (int j0 = jlo + tid; j0 < jhi; j0 += RT * RU) {
        float4 c[RU];
#pragma unroll
        for (int u = 0; u < RU; ++u) {
          const int j = j0 + RT * u;
          c[u] = j < jhi ? __ldg(base + j) : make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
        }
#pragma unroll
        for (int u = 0; u < RU; ++u) {
          const float d2 = dist2(me.x, me.y, me.z, c[u]);
          if (d2 < r2) {  // rare: in radius
            const int j = jg0 + j0 + RT * u;
            const key_t k = make_key(d2, j);
            if (j != g && k < A[7]) insert8(A, k);
          }
        }
      }
    }
    {
      key_t W[8];
      warp_top8(A, W);
      if (lane == 0)
#pragma unroll
        for (int s = 0; s < 8; ++s) wl[warp][s] = W[s];
    }
    __syncthreads();
    if (warp == 0) {  // the 16 warps' lists, one per lane
#pragma unroll
      for (int s = 0; s < 8; ++s) A[s] = lane < RT / 32 ? wl[lane][s] : KEY_EMPTY;
      key_t W[8];
      warp_top8(A, W);
#pragma unroll
      for (int s = 0; s < 8; ++s) A[s] = W[s];
    }
    if (tid == 0) {
      s_last = 1;
      if (P > 1) {  // publish this part; the last part's CTA merges all of them
#pragma unroll
        for (int s = 0; s < 8; ++s) a.rpart[((int64_t)r * RP_MAX + part) * 8 + s] = A[s];
        __threadfence();
        s_last = atomicAdd(a.rbcount + r, 1) == P - 1;
        if (s_last) {
          __threadfence();
          a.rbcount[r] = 0;  // ready for the next step
        }
      }
    }
    __syncthreads();
    if (P > 1 && s_last && warp == 0) {  // the P parts' lists, one per lane
#pragma unroll
      for (int s = 0; s < 8; ++s) A[s] = lane < P ? __ldcg(a.rpart + ((int64_t)r * RP_MAX + lane) * 8 + s) : KEY_EMPTY;
      key_t W[8];
      warp_top8(A, W);
#pragma unroll
      for (int s = 0; s < 8; ++s) A[s] = W[s];
    }
    if (tid == 0) {
      if (s_last) {
        a.nbr8[qi] = A[7] == KEY_EMPTY ? -1 : key_idx(A[7]);
        int nb[7], cnt = 0;
#pragma unroll
        for (int s = 0; s < 7; ++s) {
          nb[s] = A[s] == KEY_EMPTY ? -1 : key_idx(A[s]);
          cnt += A[s] == KEY_EMPTY ? 0 : 1;
        }
#pragma unroll
        for (int s = 0; s < 7; ++s) a.nbr[qi * 7 + s] = nb[s];
        a.cnt[qi] = cnt;
        const float4 f4 = __ldg(fwd_of(a.full, a.m, a.sdiv, a.lo + qi));
        const V3 F = steer_agent(a, v3(me), v3(f4), nb, cnt);
        if (a.think_k > 1) a.fstore[qi] = make_float4(F.x, F.y, F.z, 0.f);  // think mode: a warm thinker
        modify_agent(a, qi, v3(me), f4, F);
      }
    }
    __syncthreads();
  }
}

__global__ void __launch_bounds__(RT) k_route(StepArgs a) {
  pdl_wait();  // k_select1's routing list
  span_begin(a, SPAN_SLOT0 + 2);
  route_body(a);
  span_end(a, SPAN_SLOT0 + 2);
}

template <int NT>
int sym_grid(int sms) {
  static int grid = 0;
  if (!grid) {
    int r = 0;
    cudaFuncSetAttribute(k_sym<NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(SymSmem<NT>));
    cudaFuncSetAttribute(k_sym<NT>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&r, k_sym<NT>, NT, sizeof(SymSmem<NT>));
    grid = sms * (r > 0 ? r : 1);
  }
  return grid;
}

template <int NT>
cudaError_t sym_with(const StepArgs& a, float4* sp, int* sidx, const long long* fb_prev, long long* fb_cur,
                     long long* splits, int sms, cudaStream_t s, int part) {
  constexpr int64_t QBS = NT * Q;
  const int64_t npad = (a.nloc + QBS - 1) / QBS * QBS;
  const int64_t nb = npad / QBS;
  const int64_t items = nb * npad - QBS * (nb * (nb - 1) / 2);
  const int g = (int)std::min<int64_t>(std::min<int64_t>(sym_grid<NT>(sms), (items + CT - 1) / CT), SYM_FB_MAX_CTAS);
  static const int wd4 = [] {
    const char* e = getenv("BOIDS_SYM_WD4");  // diagnostics: diagonal item weight x4
    return e ? atoi(e) : 6;  // measured best of 4..16 at C3 and C4
  }();
  BOIDS_PREFER_SMEM(k_sym_prep);
  const int64_t cap = sym_capacity(a.nloc);  // sp holds 4 * cap floats: x[cap] | y[cap] | z[cap] | lim[cap]
  float* spf = reinterpret_cast<float*>(sp);
  if (part != 2) {
    k_sym_prep<<<(unsigned)((npad + 255) / 256), 256, 0, s>>>(a, spf, cap, sidx, npad, QBS, g, wd4, fb_prev, splits);
    if (cudaError_t e = cudaGetLastError()) return e;
  }
  if (part == 1) return cudaSuccess;
  return launch_pdl(k_sym<NT>, dim3(g), dim3(NT), sizeof(SymSmem<NT>), s, a, (const float*)spf, cap,
                    (const int*)sidx, npad, (const long long*)splits, fb_cur);
}

// ---------------------------------------------------------------------------
// Sym-shards: the unordered-pair triangle of the whole flock split over the
// ranks of an index-sharded (boids_create_shard) brute-force flock.
//   prep    (k_ss_lim)      each rank: the warm limits of its own agents (as
//                           k_sym_prep: t0, window bound, routing) -> its slice
//   [all-gather of the limits]
//   search  (k_ss_spbuild,  every rank: the same deterministic global Morton
//            k_sym)         order (binning + a per-cell sort by index), the
//                           agents as SoA with their limits, and k_sym over this
//                           rank's share [T g / G, T (g + 1) / G) of the triangle:
//                           hits for ANY agent into full-size buffers
//   [all-to-all: the hits of rank h's agents to rank h]
//   finish  (k_ss_select)   each rank: its agents' hits from all G segments ->
//                           top-7, steering, modification (k_route as usual)
// Every unordered pair is evaluated exactly once over all ranks (the ranks'
// shares tile the triangle of ONE order), so the hit set of every agent is the
// single-GPU one: identical lists.
__global__ void __launch_bounds__(256) k_ss_lim(StepArgs a, float* __restrict__ lim_send, const int* __restrict__ gperm,
                                                const int* __restrict__ gstart, int nsorted) {
  const int64_t i = (int64_t)blockIdx.x * 256 + threadIdx.x;
  const bool real = i < a.nloc;  // (threads up to the block's end take part in the warp's window bounds)
  const float r2 = __fmul_rn(a.p.search_radius, a.p.search_radius);
  const float r2_in = __uint_as_float(__float_as_uint(r2) - 1u);
  const float nan = __int_as_float(0x7fc00000);
  const float4 me = real ? __ldg(pos_of(a.full, a.m, a.sdiv, a.lo + i)) : make_float4(nan, nan, nan, 0.f);
  int c = 0;
  const float t0 = real ? sym_t0(a, i, me, c) : 0.f;
  float lim = fminf(r2_in, t0);
  // the window over the GLOBAL Morton order (every rank's agents): over this
  // rank's own 1/G of them the 7th nearest lies ~G^(1/3) times farther and many
  // more agents stayed unbounded (C4, 8 ranks: ~45 routed per rank vs ~36 in all)
  const float wb = window_bound_warp(a, gperm, gstart, a.loc, nsorted, 0, a.lo + i, me, real && t0 > r2_in);
  if (real && t0 > r2_in) lim = fminf(lim, wb);
  if (real && c == 7 && lim > r2_in && a.rlist) {  // unbounded (a wrap): k_route searches it whole
    a.rlist[atomicAdd(a.rcount, 1)] = (int)i;
    a.routed[i] = 1;
    if (a.stats) atomicAdd(a.stats + 2, 1ull);
    lim = -1.f;
  }
  if (i < a.m) lim_send[i] = real ? lim : -1.f;
}

// The binning's order inside a cell follows its atomics: sort every cell's
// entries by agent index, so every rank holds the same global order.
__global__ void k_ss_cellsort(int* __restrict__ perm, const int* __restrict__ start, int cells) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= cells) return;
  const int lo = start[c], hi = start[c + 1];
  for (int i = lo + 1; i < hi; ++i) {
    const int v = perm[i];
    int k = i - 1;
    while (k >= lo && perm[k] > v) {
      perm[k + 1] = perm[k];
      --k;
    }
    perm[k + 1] = v;
  }
}

// SoA of the globally sorted agents with their gathered limits (phantom slots
// beyond n: NaN, limit -1); the last block also cuts this rank's item share.
__global__ void __launch_bounds__(256) k_ss_spbuild(StepArgs a, const int* __restrict__ gperm, int64_t nsorted,
                                                    const float* __restrict__ lim_full, float* __restrict__ spf,
                                                    int64_t cap, int* __restrict__ sidx, int64_t npad, int64_t qb,
                                                    int G, int64_t lo, int64_t hi, int wd4,
                                                    const long long* __restrict__ fb_prev,
                                                    long long* __restrict__ splits) {
  pdl_trigger();
  if (blockIdx.x == gridDim.x - 1) compute_splits(fb_prev, G, lo, hi, npad, qb, wd4, splits);
  const int64_t p = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (p >= npad) return;
  if (p >= nsorted) {
    const float nan = __int_as_float(0x7fc00000);
    spf[p] = nan;
    spf[cap + p] = nan;
    spf[2 * cap + p] = nan;
    spf[3 * cap + p] = -1.f;
    sidx[p] = -1;
    return;
  }
  const int j = __ldg(gperm + p);
  const float4 q = __ldg(pos_of(a.full, a.m, a.sdiv, j));
  spf[p] = q.x;
  spf[cap + p] = q.y;
  spf[2 * cap + p] = q.z;
  spf[3 * cap + p] = __ldg(lim_full + j);  // agent j's limit, computed by its owner
  sidx[p] = j;
}

// An owned agent's hits from the G ranks' segments -> exact top-7 (+ 8th),
// steering, modification (k_select1's work over G hit buffers).
__global__ void __launch_bounds__(128) k_ss_select(StepArgs a, const key_t* __restrict__ recv,
                                                   const int* __restrict__ rcnt, int world) {
  pdl_wait();
  const int64_t qi = (int64_t)blockIdx.x * 128 + threadIdx.x;
  if (qi >= a.nloc) return;
  if (a.routed[qi]) {  // routed by k_ss_lim: finished by k_route
    a.routed[qi] = 0;
    a.nbr8[qi] = -1;
    return;
  }
  bool over = false;
  for (int sg = 0; sg < world; ++sg) over |= rcnt[(int64_t)sg * a.m + qi] > a.hits_cap;
  if (over) {  // a rank's buffer for this agent overflowed: searched whole by k_route
    if (a.stats) atomicAdd(a.stats + 2, 1ull);
    a.rlist[atomicAdd(a.rcount, 1)] = (int)qi;
    a.nbr8[qi] = -1;
    return;
  }
  key_t L[8];
#pragma unroll
  for (int t = 0; t < 8; ++t) L[t] = KEY_EMPTY;
  for (int sg = 0; sg < world; ++sg) {
    const int c = rcnt[(int64_t)sg * a.m + qi];
    const key_t* h = recv + ((int64_t)sg * a.m + qi) * a.hits_cap;
    for (int k = 0; k < c; ++k) insert8(L, h[k]);
  }
  a.nbr8[qi] = L[7] == KEY_EMPTY ? -1 : key_idx(L[7]);
  key_t A[7];
#pragma unroll
  for (int t = 0; t < 7; ++t) A[t] = L[t];
  finish_agent(a, qi, A);
}

}  // namespace

cudaError_t launch_ss_lim(const StepArgs& a, float* lim_send, const int* gperm, const int* gstart, int64_t nsorted,
                          cudaStream_t s) {
  if (a.m <= 0) return cudaSuccess;
  k_ss_lim<<<(unsigned)((a.m + 255) / 256), 256, 0, s>>>(a, lim_send, gperm, gstart, (int)nsorted);
  return cudaGetLastError();
}

cudaError_t launch_ss_cellsort(int* perm, const int* start, int cells, cudaStream_t s) {
  k_ss_cellsort<<<(unsigned)((cells + 255) / 256), 256, 0, s>>>(perm, start, cells);
  return cudaGetLastError();
}

// This rank's share of the global triangle over the nsorted sorted agents.
cudaError_t launch_ss_search(const StepArgs& a, const int* gperm, int64_t nsorted, const float* lim_full, float4* sp,
                             int* sidx, const long long* fb_prev, long long* fb_cur, long long* splits, int rank,
                             int world, cudaStream_t s) {
  constexpr int NT = 512;
  constexpr int64_t QBS = NT * Q;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t npad = (nsorted + QBS - 1) / QBS * QBS;
  const int64_t nb = npad / QBS;
  const int64_t T = nb * npad - QBS * (nb * (nb - 1) / 2);
  const int64_t lo = (int64_t)((__int128)T * rank / world) / UG * UG;
  const int64_t hi = rank + 1 == world ? T : (int64_t)((__int128)T * (rank + 1) / world) / UG * UG;
  const int g = (int)std::max<int64_t>(1, std::min<int64_t>(std::min<int64_t>(sym_grid<NT>(sms), (hi - lo + CT - 1) / CT),
                                                             SYM_FB_MAX_CTAS));
  const int64_t cap = sym_capacity(nsorted);
  float* spf = reinterpret_cast<float*>(sp);
  k_ss_spbuild<<<(unsigned)((npad + 255) / 256), 256, 0, s>>>(a, gperm, nsorted, lim_full, spf, cap, sidx, npad, QBS,
                                                              g, lo, hi, 6, fb_prev, splits);
  if (cudaError_t e = cudaGetLastError()) return e;
  if (hi <= lo) return cudaSuccess;
  return launch_pdl(k_sym<NT>, dim3(g), dim3(NT), sizeof(SymSmem<NT>), s, a, (const float*)spf, cap,
                    (const int*)sidx, npad, (const long long*)splits, fb_cur);
}

cudaError_t launch_ss_select(const StepArgs& a, const key_t* recv, const int* rcnt, int world, cudaStream_t s) {
  if (a.nloc <= 0) return cudaSuccess;
  BOIDS_PREFER_SMEM(k_ss_select);
  return launch_pdl(k_ss_select, dim3((unsigned)((a.nloc + 127) / 128)), dim3(128), 0, s, a, recv, rcnt, world);
}

int64_t sym_capacity(int64_t nloc) { return (nloc + 2047) / 2048 * 2048; }

// Launches k_sym_prep (spatial order + limits; routing into a.rlist, flagged in
// a.routed) and k_sym.  a.rcount must be zero.  Requires the
// handle's previous lists (warm step), qperm = the spatial order of the owned
// agents, world == 1, and think_every == 1.
// After k_select: agents in a.rlist (routed by k_sym_prep, or hit-buffer overflow)
// are searched whole and finished, one CTA each (grid-stride over the device count).
cudaError_t launch_route(const StepArgs& a, cudaStream_t s) {
  if (a.nloc <= 0 || !a.rlist) return cudaSuccess;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  BOIDS_PREFER_SMEM(k_route);
  return launch_pdl(k_route, dim3((unsigned)std::min<int64_t>(a.nloc, 2LL * sms)), dim3(RT), 0, s, a);
}

cudaError_t launch_sym_scan(const StepArgs& a, float4* sp, int* sidx, const long long* fb_prev, long long* fb_cur,
                            long long* splits, cudaStream_t s, int part) {
  if (a.nloc <= 0) return cudaSuccess;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // one 512-thread CTA per SM when every SM gets >= 2 tiles of (2048 queries x CT)
  const int64_t nb = (a.nloc + 2047) / 2048, np = nb * 2048;
  const int64_t tiles512 = (nb * np - 2048 * (nb * (nb - 1) / 2)) / CT;
  static const int force = [] {
    const char* e = getenv("BOIDS_SYM_NT");  // diagnostics: force a CTA shape (128 or 512)
    return e ? atoi(e) : 0;
  }();
  if (force == 256) return sym_with<256>(a, sp, sidx, fb_prev, fb_cur, splits, sms, s, part);
  if (force == 512 || (force != 128 && tiles512 >= 2LL * sms)) return sym_with<512>(a, sp, sidx, fb_prev, fb_cur, splits, sms, s, part);
  return sym_with<128>(a, sp, sidx, fb_prev, fb_cur, splits, sms, s, part);
}

}  // namespace boids
