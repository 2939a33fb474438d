/*
 * boids.h -- C ABI of libboids.so, the B200 (sm_100a) Boids step.
 *
 * One call of boids_step() advances every agent by one OpenSteer Boids update
 * stage (PAPER.md = the thesis text; "P:<line> sec" cites it):
 *   1. neighbour search: the up-to-7 nearest agents within the search radius,
 *      brute force over all agents (Listing 5.2, sec 5.2.1;
 *      Listing 6.3, sec 6.3.1) or, with search_mode = BOIDS_GRID, over
 *      a uniform grid that returns the identical sets (future work);
 *   2. steering: weighted sum of normalised separation, alignment and
 *      cohesion over those neighbours (Listings 5.1, 5.3-5.5);
 *   3. modification substage: clamp force, integrate velocity and position,
 *      regenerate the local space, wrap around the world sphere (P:345,
 *      P:418 sec 5.3, sec 6.2.3).
 * The update is synchronous: all of S(t+1) is computed from S(t) (the two
 * substages of P:418 / the two kernels of P:440).  Exact arithmetic contract:
 * DESIGN.md Appendix A; parameter readings: DESIGN.md Table C1 / Q1-Q17.
 *
 * Conventions
 *   - Every function returns BOIDS_OK (0) or a negative BOIDS_E* code and
 *     never throws; boids_last_error() gives a thread-local message.
 *   - Host arrays are AoS float32: pos3/fwd3/up3/side3 are n*3 floats
 *     (x,y,z per agent), speed is n floats, caller-owned.  A NULL output
 *     array is skipped.  The device layout is private (SoA float4, DESIGN.md
 *     "Data layout"); the 4x4 draw matrix of P:502 is (side, up, fwd, pos).
 *   - The handle owns all device memory.  Device pointers escape only via
 *     boids_shard_buffers (for the caller's NCCL all-gather).
 *   - Work is enqueued on the stream set with boids_set_stream (default: the
 *     legacy default stream) and is asynchronous; launch errors surface at the
 *     next synchronising call (get_*, set_*, boids_sync).
 */
#ifndef BOIDS_H
#define BOIDS_H

#include <stdint.h>

#if defined(__GNUC__)
#define BOIDS_API __attribute__((visibility("default")))
#else
#define BOIDS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

#define BOIDS_OK 0
#define BOIDS_EINVAL (-1) /* bad argument: n < 1, max_neighbors != 7, radius <= 0, NaN param,
                             dt < 0 or NaN, steps < 0, NULL handle/pointer, wrong call for mode */
#define BOIDS_ECUDA (-2)  /* CUDA runtime error; message holds cudaGetErrorString */
#define BOIDS_ENCCL (-3)  /* reserved for the Python binding (torch.distributed failures) */
#define BOIDS_ENOMEM (-4) /* device or host allocation failed */

#define BOIDS_BRUTE 0 /* O(n^2) scan over all agents, Listing 5.2 */
#define BOIDS_GRID 1  /* uniform-grid binned search, identical neighbour sets */

#define BOIDS_INIT_OPENSTEER 0 /* positions uniform in the ball of radius init_radius */
#define BOIDS_INIT_WORLD 1     /* positions uniform in the ball of radius world_radius */

/* Parameters.  Defaults (boids_default_params) are DESIGN.md Table C1; the
 * thesis prints only k = 7, every other value is a documented reading. */
typedef struct boids_params {
  float search_radius;   /* neighbour search radius r; candidate iff d2 < fl(r*r) (Q2). 9.0 */
  float w_separation;    /* weightA of Listing 5.1. 12 */
  float w_alignment;     /* weightB. 8 */
  float w_cohesion;      /* weightC. 8 */
  float max_force;       /* steering vector length clamp. 27 */
  float max_speed;       /* speed clamp. 9 */
  float mass;            /* a = F / mass (length of the steering vector = acceleration). 1 */
  float world_radius;    /* spherical world radius R. 50 */
  float init_radius;     /* ball radius of BOIDS_INIT_OPENSTEER. 20 */
  float init_speed_frac; /* initial speed = init_speed_frac * max_speed. 0.3 */
  int32_t max_neighbors; /* must be 7 */
  int32_t search_mode;   /* BOIDS_BRUTE or BOIDS_GRID */
  int32_t init_mode;     /* BOIDS_INIT_OPENSTEER or BOIDS_INIT_WORLD */
  int32_t think_every;   /* think frequency k >= 1 (skipThink, sec 5.3): agent i runs the
                            simulation substage at step t iff (i + t) mod k == 0 and otherwise
                            reuses its stored steering vector; every agent is modified.  1 */
  int32_t steer_mode;    /* BOIDS_STEER_THESIS (default): steering of Listings 5.1-5.5 and the
                            modification of reading Q10.  BOIDS_STEER_OPENSTEER: OpenSteer 0.8.2's
                            flocking [ext] over the same <= 7 neighbours (
                            "based on the CPU version of OpenSteer"): per-behaviour
                            inBoidNeighborhood filters (radii 5 / 7.5 / 9, cos -0.707 / 0.7 / -0.15,
                            always within 1.5), averaged behaviours, adjustRawSteeringForce below
                            0.2 max_speed and acceleration smoothing (per-agent state, see
                            boids_get_accel).  DESIGN.md readings Q20-Q24. */
} boids_params;

#define BOIDS_STEER_THESIS 0
#define BOIDS_STEER_OPENSTEER 1

typedef struct boids_ctx boids_ctx; /* opaque handle */

/* Read-only description of a handle (boids_info). */
typedef struct boids_info_t {
  int64_t n;         /* total agents */
  int64_t lo, hi;    /* agents [lo, hi) are owned (updated) by this handle */
  int64_t slice;     /* padded per-rank slice m (multiple of 256); agent j lives in slice j / m */
  int32_t rank, world;
  int32_t kernel;    /* brute-force kernel variant in use (BOIDS_KERNEL_*) */
  int32_t cluster;   /* candidate split (CTAs per cluster) of the fused kernel */
  int64_t launches;  /* number of kernels this handle has launched so far */
  int64_t slow_groups; /* fused kernel, cumulative: vote groups (U candidates x Q queries x 32
                          lanes) that took the insertion path ... */
  int64_t vote_groups; /* ... out of this many (diagnostics; boids_info synchronises) */
  int64_t fallbacks;   /* warm path, cumulative: agents searched whole (k_route) after a hit-buffer
                          overflow or, on k_sym steps, because their previous neighbours all
                          left the radius (a wrap); grid mode: queries whose bound reached past the
                          adjacent cells, searched alone by k_grid_far */
  int64_t grid_pairs;  /* grid mode, cumulative: (query, candidate) pairs evaluated over the
                          27-cell stencils -- the grid search's algorithmic work */
  int64_t step_index;  /* steps taken by this handle (the t of the think schedule) */
  int32_t last_path;   /* search path the last step ran (BOIDS_PATH_*; -1 before the first step) --
                          what bench.py's roofline counts as the algorithmic work */
  int32_t reserved0;
  int64_t steps_sorted; /* cumulative: steps that rebuilt the spatial query order (binning) */
  int64_t graph_launches; /* cumulative: boids_step steps run as a captured CUDA graph (BOIDS_OPT_GRAPH) */
} boids_info_t;

/* boids_info_t.last_path */
#define BOIDS_PATH_FUSED 0   /* cold step: k_fused (cluster kernel, ordered pairs n_local x n) */
#define BOIDS_PATH_SCAN 1    /* warm step: k_bound + k_scan over ordered pairs n_local x n */
#define BOIDS_PATH_SYM 2     /* warm step: k_sym_prep + k_sym over unordered pairs n(n-1)/2 */
#define BOIDS_PATH_GRID 3    /* grid mode: binning + k_grid (+ k_grid_far) */
#define BOIDS_PATH_SIMPLE 4  /* BOIDS_KERNEL_SIMPLE: k_search_simple + k_update */
#define BOIDS_PATH_THINK 5   /* brute force, think mode: thinkers on k_bound + k_scan (cold ones k_fused) */
#define BOIDS_PATH_SMALL 6   /* warm step of a small single-rank flock: k_small (ordered pairs n x n, one kernel) */

#define BOIDS_KERNEL_FUSED 0   /* default: cold steps run the fused cluster kernel (search + merge +
                                  steer + modify); warm steps (previous lists known) run the
                                  all-pairs hit scan + select/update pair */
#define BOIDS_KERNEL_SIMPLE 1  /* two kernels: tiled search -> neighbour lists -> update */
#define BOIDS_KERNEL_CLUSTER 2 /* every step on the fused cluster kernel */

/* Options for boids_set_option. */
#define BOIDS_OPT_RECORD_STEERING 1 /* 1: keep the last step's steering vectors (boids_get_steering) */
#define BOIDS_OPT_KERNEL 2          /* BOIDS_KERNEL_* */
#define BOIDS_OPT_PROFILE 3         /* 1: bracket each kernel launch with CUDA events (boids_get_profile);
                                       2: only the search launches (and the update launches in think
                                       mode): fewer event records inside a timed step; 0: off */
#define BOIDS_OPT_CLUSTER 4         /* 0 = automatic, else force the fused kernel's cluster size (1..16) */
#define BOIDS_OPT_RESORT 6          /* refresh the spatial order of the fused kernel's query blocks every
                                       `value` steps (default 8; results never depend on it) */
#define BOIDS_OPT_VOTE_U 7          /* fused kernel: candidates per warp vote, 4 (default) or 8 */
#define BOIDS_OPT_SYMMETRIC 8       /* warm brute-force steps of a single-GPU handle with n >= 8192:
                                       1 (default) = evaluate every unordered pair once and test it
                                       against both agents' limits (k_sym; d2 is bitwise symmetric),
                                       0 = every ordered pair (k_scan).  Results are identical. */
#define BOIDS_OPT_BALANCE 9         /* k_sym work split: 1 (default) = cut the unordered-pair item space
                                       so that every CTA gets an equal share of the SM time the previous
                                       k_sym launch measured per item range (feedback; the first launch
                                       uses a static weighted split), 0 = static split always.  Only the
                                       partition of the work changes; results are identical. */
#define BOIDS_OPT_GRAPH 10          /* 1: boids_step replays a captured CUDA graph of each warm single-rank
                                       step (think_every 1; profiling events are retargeted per replay);
                                       0 (default): every kernel is launched from the host (measured on
                                       B200: the graph saves host enqueue time but a step of 4-6 dependent
                                       kernels behind a cold L2 runs 5-6 us slower as a graph, C1-C3).
                                       Results are identical either way. */
#define BOIDS_OPT_SMALL 11          /* 1 (default): warm brute-force steps of a single-rank handle with
                                       n < 8192 run as one kernel (k_small: P threads per query scan all
                                       agents, merge their top-8 lists, steer and modify); 0: the
                                       k_bound + k_scan + k_select1 + k_route chain.  Results identical. */
#define BOIDS_OPT_PHASES 5          /* diagnostics: value = max CTAs; the fused kernel records per-CTA
                                       %globaltimer stamps (read with boids_get_phases); 0 = off */

BOIDS_API void boids_default_params(boids_params* out);

/* Allocate and initialise n agents from (params, seed) per DESIGN.md Appendix B.
 * Returns BOIDS_EINVAL for bad params, BOIDS_ENOMEM / BOIDS_ECUDA on failure.
 * The initial state is a pure function of (n, params, seed). */
BOIDS_API int boids_create(int64_t n, const boids_params* p, uint64_t seed, boids_ctx** out);

/* Like boids_create, but this handle owns agents [rank*m, min((rank+1)*m, n)) of an
 * n-agent flock split over `world` ranks (m = boids_info.slice).  The caller
 * exchanges positions between ranks (all-gather of the send slices, see
 * boids_shard_buffers) before every boids_step_shard.  world == 1 is allowed. */
BOIDS_API int boids_create_shard(int64_t n, const boids_params* p, uint64_t seed, int32_t rank,
                       int32_t world, boids_ctx** out);

/* ---- Sym-shards: the unordered-pair triangle of a brute-force flock split over
 * index shards (boids_create_shard handles, search_mode BOIDS_BRUTE, think_every 1;
 * the search is Listing 5.2's brute force, multiple devices are the thesis's future
 * work).
 * A single-GPU handle evaluates every unordered pair once (k_sym: d2 is bitwise
 * symmetric); plain index shards evaluate n/G x n ordered pairs each.  Here the
 * ranks share the n(n-1)/2 pairs of ONE global order instead.  A warm step (the
 * first step of a handle runs boids_step_shard) is, after the usual all-gather of
 * the [pos4 | fwd4] slices:
 *   boids_symshard_prep(h)        this rank's agents' warm limits -> lim_send (m floats)
 *   all-gather lim_send -> lim_full (world * m floats, rank g's slice at g * m)
 *   boids_symshard_search(h)      the same deterministic global Morton order on every
 *                                 rank, this rank's 1/world share of the triangle: hits
 *                                 (u64 keys) for ANY agent j into hits[j * hits_cap ...],
 *                                 counts hitcnt[j] (world * m slots, agent j at slot j)
 *   all-to-all: block d of hits / hitcnt (slots [d*m, (d+1)*m)) to rank d, received
 *                                 from rank s into recv / rcnt block s
 *   boids_symshard_finish(h, dt)  this rank's agents: the hits of all world blocks ->
 *                                 top-7, steering, modification into the send slice.
 * hits_cap (16) bounds one agent's hits per rank segment; an agent with more in any
 * segment is searched whole by its owner in finish (exact either way).
 * Lists and states are those of the single-GPU step.  Asynchronous; EINVAL if the
 * handle is not a warm brute-force shard handle. */
BOIDS_API int boids_symshard_prep(boids_ctx* ctx);
BOIDS_API int boids_symshard_search(boids_ctx* ctx);
BOIDS_API int boids_symshard_finish(boids_ctx* ctx, float dt);
/* Device buffers of the two exchanges (allocated on first use). */
BOIDS_API int boids_symshard_buffers(boids_ctx* ctx, void** lim_send, void** lim_full, void** hits, void** hitcnt,
                                     void** recv, void** rcnt, int32_t* hits_cap);

/* ---- Spatial decomposition (future work of the thesis) ----
 * A spatial shard of a grid-mode flock (search_mode BOIDS_GRID, think_every 1):
 * rank `rank` of `world` OWNS the agents whose search-grid cell layer z lies in
 * its slab [zb[rank], zb[rank+1]) (boundaries balance the initial agent counts,
 * boids_spatial_bounds) and holds, besides them, only its HALO -- the agents
 * within `reach` cell layers of the slab, i.e. within the search radius of any
 * owned agent.  Indices stay global: the handle addresses all n agents (arrays
 * of boids_get_state / get_neighbors have n rows; rows of agents not owned are
 * meaningless, see boids_spatial_owned).  Every rank creates its handle from
 * the same (n, params, seed).  A step is
 *   boids_step_spatial(h, dt)           owned agents: search + steer + modify,
 *                                       then pack the outgoing records;
 *   boids_spatial_outbox(h, ...)        record counts per destination rank;
 *   (caller moves the records: destination d's halo records of every rank into
 *    d's halo inbox, migrant records likewise -- NCCL all-to-all, or copies);
 *   boids_spatial_unpack(h, nh, nm)     apply the received records.
 * Records are float4 arrays: halo = 2 float4 (x, y, z, index bits | forward,
 * speed); migrant = 8 float4 (the whole per-agent state incl. neighbour lists).
 * Outbox of destination d: halo_out + d * cap_halo * 2 float4, mig_out + d *
 * cap_mig * 8 float4.  The results are those of the single-GPU step (identical
 * neighbour lists and states for every agent, each computed by its owner). */
BOIDS_API int boids_create_spatial(int64_t n, const boids_params* p, uint64_t seed, int32_t rank, int32_t world,
                                   boids_ctx** out);
BOIDS_API int boids_step_spatial(boids_ctx* ctx, float dt);
/* Synchronises.  halo_counts / mig_counts: world int32 each (records for each
 * destination; 0 for this rank).  BOIDS_ENOMEM if an outbox overflowed. */
BOIDS_API int boids_spatial_outbox(boids_ctx* ctx, int32_t* halo_counts, int32_t* mig_counts, void** halo_out,
                                   void** mig_out, int64_t* cap_halo, int64_t* cap_mig);
/* Device inboxes (records are placed at their start, contiguous) and capacities in records. */
BOIDS_API int boids_spatial_inbox(boids_ctx* ctx, void** halo_in, void** mig_in, int64_t* cap_halo_in,
                                  int64_t* cap_mig_in);
/* Apply n_halo halo and n_mig migrant records from the inboxes (asynchronous).
 * BOIDS_EINVAL if a count exceeds its inbox capacity. */
BOIDS_API int boids_spatial_unpack(boids_ctx* ctx, int64_t n_halo, int64_t n_mig);
/* own[n]: 1 for the agents this rank owns now.  Synchronises. */
BOIDS_API int boids_spatial_owned(boids_ctx* ctx, uint8_t* own);
/* zb[world + 1]: slab boundaries in search-cell layers; *reach: halo width in layers. */
BOIDS_API int boids_spatial_bounds(boids_ctx* ctx, int32_t* zb, int32_t* reach);

/* Enqueue all later work on `cuda_stream` (a cudaStream_t; NULL = legacy default). */
BOIDS_API int boids_set_stream(boids_ctx* ctx, void* cuda_stream);

BOIDS_API int boids_set_option(boids_ctx* ctx, int32_t option, int64_t value);

/* Advance `steps` synchronous steps of length dt (single-rank handles only).
 * steps = 0 is a no-op; dt = 0 computes steering but leaves positions unchanged.
 * Asynchronous on the handle's stream. */
BOIDS_API int boids_step(boids_ctx* ctx, float dt, int32_t steps);

/* One step of a shard handle: reads the full gathered (pos, fwd) buffer, writes
 * this rank's new slice into the send buffer.  Asynchronous. */
BOIDS_API int boids_step_shard(boids_ctx* ctx, float dt);

/* Device buffers of a shard handle, for the caller's all-gather:
 *   *send: this rank's slice, 2*m float4 = [pos4(m) | fwd4(m)], *slice_bytes bytes;
 *   *full: world * (*slice_bytes) bytes, rank g's slice at byte offset g * (*slice_bytes).
 * all_gather(full <- send) must complete (stream-ordered) before boids_step_shard. */
BOIDS_API int boids_shard_buffers(boids_ctx* ctx, void** send, void** full, int64_t* slice_bytes);

/* Copy the owned agents' state to host AoS arrays (count = hi - lo).  Synchronises. */
BOIDS_API int boids_get_state(boids_ctx* ctx, float* pos3, float* fwd3, float* up3, float* side3,
                    float* speed);

/* Overwrite the owned agents' state from host AoS arrays (count = hi - lo).
 * side is recomputed by the next step.  The last step's neighbour lists are kept
 * as the seed of the next step's search bound (valid for any new positions).
 * pos3, fwd3, up3, speed must be non-NULL; side3 may be NULL (then zero).  Synchronises. */
BOIDS_API int boids_set_state(boids_ctx* ctx, const float* pos3, const float* fwd3, const float* up3,
                    const float* side3, const float* speed);

/* steer_mode BOIDS_STEER_OPENSTEER only: the smoothed accelerations
 * (OpenSteer's _smoothedAcceleration, zero at creation) of the owned agents,
 * host AoS float acc3[(hi - lo) * 3].  get: copies into caller memory and
 * synchronises the handle's stream; set: copies from caller memory (used from
 * the next step on).  BOIDS_EINVAL on a NULL argument or another steer_mode. */
BOIDS_API int boids_get_accel(boids_ctx* ctx, float* acc3);
BOIDS_API int boids_set_accel(boids_ctx* ctx, const float* acc3);

/* Neighbour lists of the last step for the owned agents: idx7 = count*7 int32,
 * ascending by (d2, index), -1 padded; cnt = count int32, or -1 for an agent that
 * has not been searched yet (before its first step / first think).  Synchronises. */
BOIDS_API int boids_get_neighbors(boids_ctx* ctx, int32_t* idx7, int32_t* cnt);

/* Steering vectors F (before the max_force clamp) of the last step, count*3 floats.
 * Requires BOIDS_OPT_RECORD_STEERING = 1 before that step (else BOIDS_EINVAL). */
BOIDS_API int boids_get_steering(boids_ctx* ctx, float* force3);

/* Wait for all enqueued work; returns the first pending CUDA error. */
BOIDS_API int boids_sync(boids_ctx* ctx);

/* Double-buffered asynchronous readback of the draw data (the thesis's double
 * buffering; "only the required information to draw the agents -- a
 * 4x4 matrix containing 16 float values -- is moved from the device").
 * begin: enqueue, on the handle's stream, a kernel packing each owned agent's
 * 4x4 local-space matrix of the CURRENT state (rows side, up, fwd, pos as
 * (x,y,z,0|0|0|1), count*16 floats, row-major) into a device buffer, then a copy
 * to host16 on a separate copy stream; returns at once, so later boids_step
 * calls overlap the copy.  At most one readback in flight per handle (begin
 * waits for the previous one).  host16 should be pinned (page-locked) memory and
 * must stay valid until boids_readback_wait; alternate two host buffers to draw
 * step n while step n+1 runs.  wait: block until the readback landed in host16. */
BOIDS_API int boids_readback_begin(boids_ctx* ctx, float* host16);
BOIDS_API int boids_readback_wait(boids_ctx* ctx);

/* Think-frequency state (complete snapshot together with boids_get_state and
 * boids_get_neighbors): the step index t of the next step and every owned agent's
 * stored steering vector (count*3 floats; zero until the agent first thinks).
 * set: fstore3 NULL keeps the stored vectors.  Both synchronise. */
BOIDS_API int boids_get_think_state(boids_ctx* ctx, int64_t* step_index, float* fstore3);
BOIDS_API int boids_set_think_state(boids_ctx* ctx, int64_t step_index, const float* fstore3);

/* Measurement hook (SURVEY.md 8(d), B5 "update_standalone"): time `reps` launches
 * of the standalone update kernel k_update -- steering from the neighbour lists
 * of the last step (boids_get_neighbors) plus the modification substage, one
 * thread per owned agent (the thesis's separate modification kernel, P:440,
 * P:497-502) -- with CUDA events on the handle's stream, each launch alone.
 * The kernel writes into private scratch buffers (copies of the frame), so the
 * handle's state, lists and step index are unchanged.  *ms_per_launch = mean
 * launch duration.  Synchronises.  EINVAL: NULL argument, reps < 1, bad dt. */
BOIDS_API int boids_bench_update(boids_ctx* ctx, float dt, int32_t reps, double* ms_per_launch);

/* Describe the handle (synchronises: it reads the device-side counters). */
BOIDS_API int boids_info(boids_ctx* ctx, boids_info_t* out);

/* Accumulated kernel time (ms) and launch count per kernel class since the last
 * reset, measured with CUDA events on the handle's stream (BOIDS_OPT_PROFILE).
 * Classes: 0 fused/search, 1 update, 2 binning, 3 grid search, 4 k_route (agents searched
 * whole after a hit-buffer overflow or a wrap), 5 search prologue (k_sym_prep: the warm limits
 * and the agents' spatially ordered copy k_sym reads).  Synchronises. */
#define BOIDS_PROF_CLASSES 6
BOIDS_API int boids_get_profile(boids_ctx* ctx, double* ms, int64_t* launches, int32_t reset);

/* Diagnostics: copy `count` u64 phase stamps (8 per CTA) of the last fused step to host. */
BOIDS_API int boids_get_phases(boids_ctx* ctx, uint64_t* out, int64_t count);

BOIDS_API void boids_destroy(boids_ctx* ctx);

BOIDS_API const char* boids_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* BOIDS_H */
