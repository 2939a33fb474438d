// api.cu -- the C ABI of include/boids.h: handles, buffers, validation, the step
// loop and host<->device state transfer.  No exception crosses the ABI.
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <algorithm>
#include <vector>

#include "internal.h"

using namespace boids;

namespace {

thread_local std::string g_err;

int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}

#define CK(expr)                                                                  \
  do {                                                                            \
    cudaError_t e_ = (expr);                                                      \
    if (e_ != cudaSuccess) {                                                      \
      (void)cudaGetLastError();                                                   \
      return fail(e_ == cudaErrorMemoryAllocation ? BOIDS_ENOMEM : BOIDS_ECUDA,   \
                  std::string(#expr) + ": " + cudaGetErrorString(e_));            \
    }                                                                             \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
    else prev = -1;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

}  // namespace

struct boids_ctx {
  int64_t n = 0, m = 0, lo = 0, hi = 0, nloc = 0;
  int32_t rank = 0, world = 1;
  bool shard = false;
  boids_params p{};
  int dev = 0, sm_count = 148;
  cudaStream_t stream = nullptr;
  // !shard: buf[0], buf[1] = ping-pong full buffers (2m float4 each), current = buf[cur].
  //  shard: buf[0] = full gathered buffer (world*2m), buf[1] = this rank's send slice (2m).
  float4* buf[2] = {nullptr, nullptr};
  int cur = 0;
  float4 *up4 = nullptr, *side4 = nullptr, *force4 = nullptr;
  int32_t *nbr = nullptr, *cnt = nullptr;
  // spatial binning (k_bin.cu): locality grid of the brute-force step
  BinGrid loc_grid{};
  int2* cellrank = nullptr;
  int32_t *bcnt = nullptr, *bstart = nullptr, *qperm = nullptr;
  float4* cand = nullptr;
  int64_t ncand = 0;
  float4* acc4 = nullptr;               // steer_mode 1: smoothed accelerations [m]
  unsigned long long* stats = nullptr;  // fused-kernel insertion-path counters (device)
  unsigned long long* hits = nullptr;   // warm path hit buffers [m][HITS]
  int32_t* hitcnt = nullptr;            // warm path hit counts [m]
  int32_t* nbr8 = nullptr;              // 8th nearest of the last step or -1 [m]
  unsigned long long* partial = nullptr;  // warm path partial lists [m][PSLOTS][7]
  float* qlim = nullptr;                  // warm path search limits [m]
  float4* sym_sp = nullptr;               // k_sym: agents in spatial order (x, y, z, limit) [sym_capacity]
  int32_t* sym_idx = nullptr;             // k_sym: their local indices [sym_capacity]
  long long* sym_fb = nullptr;            // k_sym: per-CTA (range, cycles) of the last two launches [2][SYM_FB_LEN]
  int sym_fb_par = 0;                     // which half the next launch writes
  int32_t* sym_rlist = nullptr;           // k_sym: agents routed to k_route this step [m]
  int32_t* sym_rcount = nullptr;          // ... and their number
  int32_t* growbuf = nullptr;             // grid mode: row scratch of the many-CTA binning scan
  unsigned long long* rpart = nullptr;    // k_route partial lists [m][16][8]
  int32_t* rbcount = nullptr;             // k_route parts done per routed agent [m]
  bool symmetric = true;                  // BOIDS_OPT_SYMMETRIC
  bool use_small = true;                  // BOIDS_OPT_SMALL
  bool balance = true;                    // BOIDS_OPT_BALANCE: k_sym split from the last launch's CTA times
  int32_t* pcnt = nullptr;
  unsigned long long* phase = nullptr;  // diagnostics (BOIDS_OPT_PHASES): per-CTA timestamps
  // grid mode (BOIDS_GRID): search grid and its binning buffers
  BinGrid sgrid{};
  BinGrid qgrid{};  // blocks of sgrid: the queries' binning and the grid search's work items
  // the grids the binning and the search use: sgrid / qgrid, or a spatial shard's slab of them
  BinGrid bgrid{}, bqgrid{};
  int2* gcellrank = nullptr;
  int32_t *gcnt = nullptr, *gstart = nullptr, *gqstart = nullptr, *counter = nullptr;
  int4* gitems = nullptr;      // grid search work items (k_bin_scan)
  int32_t* gnitems = nullptr;  // their number
  float4* spos = nullptr;
  float* stage = nullptr;  // host-transfer staging [13][m] (lazy)
  // double-buffered readback (lazy): packed draw matrices, copy stream, events
  float4* draw = nullptr;  // [m][4] rows
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t packed = nullptr, landed = nullptr;
  bool rb_pending = false;
  // think frequency
  float4* fstore = nullptr;         // [m] last steering vector per agent
  unsigned char* routed = nullptr;  // [m] 1 = searched by k_fused this step (think mode)
  int32_t *tcold = nullptr, *twarm = nullptr, *tcnt = nullptr;  // thinker lists and their counts
  int* ocheck = nullptr;            // [2] boids_set_state's locality check (k_order_check)
  float4* ubench = nullptr;         // boids_bench_update scratch: out [2m] | up [m] | side [m] | acc [m]
  int64_t step_index = 0, steps_taken = 0;
  int32_t last_path = -1;  // BOIDS_PATH_* of the last step
  int64_t steps_sorted = 0;
  int vote_u = 4;          // fused kernel: candidates per warp vote
  int resort_every = 8;    // refresh the spatial query order every this many steps
  int64_t since_sort = -1; // steps since the last refresh (-1: never sorted)
  bool warm = false;
  bool record_steering = false, steering_valid = false;
  int kernel = BOIDS_KERNEL_FUSED;
  int cluster_opt = 0;
  int profile = 0;          // BOIDS_OPT_PROFILE level
  int64_t launches = 0;
  // CUDA graphs of single warm steps (boids_step): one per distinct launch
  // sequence (search path, resort-or-not, k_sym feedback parity, ping-pong
  // parity, dt); replayed with cudaGraphLaunch, the host-side step state advanced
  // by a dry run of one_step
  // spatial shard (boids_create_spatial; k_spatial.cu): this rank owns the agents whose
  // search-cell layer z is in [zb[rank], zb[rank+1]), holds them and its halo layers
  bool spatial = false;
  int sp_reach = 0;                        // halo width in cell layers (cells >= r)
  int* zb = nullptr;                       // device slab boundaries [world + 1]
  std::vector<int> zb_host;
  unsigned char* own = nullptr;            // [n] 1 = owned
  float4 *halo_out = nullptr, *mig_out = nullptr, *halo_in = nullptr, *mig_in = nullptr;
  int64_t cap_h = 0, cap_m = 0, cap_in_h = 0, cap_in_m = 0;
  int* sp_counts = nullptr;                // [2 world]: halo records per destination, then migrants
  int* kept = nullptr;                     // [n] non-owned entries kept as halo locally (cleared next pack)
  int* nkept = nullptr;                    // their number (device)
  int64_t kept_bound = 0;                  // host upper bound of *nkept
  int64_t last_nh = 0;                     // halo records applied by the last unpack (cleared next pack)
  int* sp_overflow = nullptr;
  // sym-shards (an index-sharded brute-force handle stepping its share of the global
  // unordered-pair triangle; k_sym.cu "Sym-shards"): lazily allocated
  float *ss_lim_send = nullptr, *ss_lim_full = nullptr;
  unsigned long long *ss_hits = nullptr, *ss_recv = nullptr;
  int32_t *ss_hitcnt = nullptr, *ss_rcnt = nullptr, *ss_gperm = nullptr, *ss_gbcnt = nullptr, *ss_gbstart = nullptr;
  float4* ss_spos = nullptr;
  int64_t ss_since_sort = -1;
  bool dry = false;
  bool capturing = false;  // one_step runs inside graph_step's stream capture
  bool use_graphs = false;  // BOIDS_OPT_GRAPH
  cudaStream_t cap_stream = nullptr;
  struct GraphEntry {
    uint32_t key;
    float dt;
    cudaGraphExec_t exec;
    cudaGraph_t graph;  // kept: its event-record nodes address the exec's nodes
    struct Prof {
      int cls;
      cudaGraphNode_t a, b;  // event-record nodes bracketing one profiled launch (BOIDS_OPT_PROFILE)
    };
    std::vector<Prof> prof;
  };
  std::vector<GraphEntry> graphs;
  int64_t graph_launches = 0;
  struct Rec {
    int cls;
    cudaEvent_t a, b;
  };
  std::vector<Rec> recs;
  std::vector<cudaEvent_t> pool;
  double prof_ms[BOIDS_PROF_CLASSES] = {};
  int64_t prof_n[BOIDS_PROF_CLASSES] = {};

  float4* local() const { return shard ? buf[1] : buf[cur]; }
};

namespace {

bool finite(float x) { return std::isfinite(x); }

int validate(const boids_params* p) {
  if (!p) return fail(BOIDS_EINVAL, "params is NULL");
  if (p->max_neighbors != 7) return fail(BOIDS_EINVAL, "max_neighbors must be 7 (P:364)");
  if (!finite(p->search_radius) || p->search_radius <= 0.f)
    return fail(BOIDS_EINVAL, "search_radius must be finite and > 0");
  if (!finite(p->w_separation) || !finite(p->w_alignment) || !finite(p->w_cohesion))
    return fail(BOIDS_EINVAL, "weights must be finite");
  if (!finite(p->max_force) || p->max_force < 0.f) return fail(BOIDS_EINVAL, "max_force must be >= 0");
  if (!finite(p->max_speed) || p->max_speed < 0.f) return fail(BOIDS_EINVAL, "max_speed must be >= 0");
  if (!finite(p->mass) || p->mass <= 0.f) return fail(BOIDS_EINVAL, "mass must be > 0");
  if (!finite(p->world_radius) || p->world_radius <= 0.f)
    return fail(BOIDS_EINVAL, "world_radius must be > 0");
  if (!finite(p->init_radius) || p->init_radius <= 0.f)
    return fail(BOIDS_EINVAL, "init_radius must be > 0");
  if (p->think_every < 1) return fail(BOIDS_EINVAL, "think_every must be >= 1");
  if (!finite(p->init_speed_frac) || p->init_speed_frac < 0.f)
    return fail(BOIDS_EINVAL, "init_speed_frac must be >= 0");
  if (p->search_mode != BOIDS_BRUTE && p->search_mode != BOIDS_GRID)
    return fail(BOIDS_EINVAL, "search_mode must be BOIDS_BRUTE or BOIDS_GRID");
  if (p->init_mode != BOIDS_INIT_OPENSTEER && p->init_mode != BOIDS_INIT_WORLD)
    return fail(BOIDS_EINVAL, "init_mode must be BOIDS_INIT_OPENSTEER or BOIDS_INIT_WORLD");
  if (p->steer_mode != BOIDS_STEER_THESIS && p->steer_mode != BOIDS_STEER_OPENSTEER)
    return fail(BOIDS_EINVAL, "steer_mode must be BOIDS_STEER_THESIS or BOIDS_STEER_OPENSTEER");
  return BOIDS_OK;
}

void free_ctx(boids_ctx* c) {
  if (!c) return;
  DeviceGuard g(c->dev);
  for (float4* b : c->buf) cudaFree(b);
  cudaFree(c->up4);
  cudaFree(c->side4);
  cudaFree(c->force4);
  cudaFree(c->acc4);
  cudaFree(c->nbr);
  cudaFree(c->cnt);
  cudaFree(c->cellrank);
  cudaFree(c->bcnt);
  cudaFree(c->bstart);
  cudaFree(c->qperm);
  cudaFree(c->cand);
  cudaFree(c->stats);
  cudaFree(c->hits);
  cudaFree(c->hitcnt);
  cudaFree(c->nbr8);
  cudaFree(c->partial);
  cudaFree(c->pcnt);
  cudaFree(c->qlim);
  cudaFree(c->gcellrank);
  cudaFree(c->gcnt);
  cudaFree(c->gstart);
  cudaFree(c->gqstart);
  cudaFree(c->gitems);
  cudaFree(c->gnitems);
  cudaFree(c->counter);
  cudaFree(c->spos);
  cudaFree(c->stage);
  if (c->rb_pending) cudaEventSynchronize(c->landed);
  cudaFree(c->draw);
  if (c->packed) cudaEventDestroy(c->packed);
  if (c->landed) cudaEventDestroy(c->landed);
  if (c->copy_stream) cudaStreamDestroy(c->copy_stream);
  cudaFree(c->fstore);
  cudaFree(c->routed);
  cudaFree(c->tcold);
  cudaFree(c->twarm);
  cudaFree(c->tcnt);
  cudaFree(c->ocheck);
  cudaFree(c->ss_lim_send);
  cudaFree(c->ss_lim_full);
  cudaFree(c->ss_hits);
  cudaFree(c->ss_recv);
  cudaFree(c->ss_hitcnt);
  cudaFree(c->ss_rcnt);
  cudaFree(c->ss_gperm);
  cudaFree(c->ss_gbcnt);
  cudaFree(c->ss_gbstart);
  cudaFree(c->ss_spos);
  cudaFree(c->zb);
  cudaFree(c->own);
  cudaFree(c->halo_out);
  cudaFree(c->mig_out);
  cudaFree(c->halo_in);
  cudaFree(c->mig_in);
  cudaFree(c->sp_counts);
  cudaFree(c->sp_overflow);
  cudaFree(c->kept);
  cudaFree(c->nkept);
  cudaFree(c->ubench);
  cudaFree(c->phase);
  cudaFree(c->sym_sp);
  cudaFree(c->sym_idx);
  cudaFree(c->sym_fb);
  cudaFree(c->sym_rlist);
  cudaFree(c->growbuf);
  cudaFree(c->rpart);
  cudaFree(c->rbcount);
  cudaFree(c->sym_rcount);
  for (auto& g : c->graphs) {
    cudaGraphExecDestroy(g.exec);
    cudaGraphDestroy(g.graph);
  }
  if (c->cap_stream) cudaStreamDestroy(c->cap_stream);
  for (auto& r : c->recs) {
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  for (auto e : c->pool) cudaEventDestroy(e);
  delete c;
}

cudaEvent_t get_event(boids_ctx* c) {
  if (!c->pool.empty()) {
    cudaEvent_t e = c->pool.back();
    c->pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

// A step's memset on the handle's stream (skipped on a dry run: see replay_step).
cudaError_t mset(boids_ctx* c, void* p, int v, size_t bytes) {
  return c->dry ? cudaSuccess : cudaMemsetAsync(p, v, bytes, c->stream);
}

// Launch wrapper: counts launches and, when profiling, brackets with events.
// On a dry run (replay_step) nothing is enqueued: only the host-side state of
// the step advances, exactly as it did when the step's graph was captured.
template <class F>
int launch(boids_ctx* c, int cls, F&& f, int kernels = 1) {
  if (c->dry) {
    c->launches += kernels;
    return BOIDS_OK;
  }
  cudaEvent_t a = nullptr, b = nullptr;
  // level 2: only the search classes (0, 3), plus the update (1) in think mode
  // (k_apply / k_select carry that step's modification roofline) -- fewer event
  // records in a timed step (each costs GPU time between dependent kernels)
  const bool rec = c->profile == 1 ||
                   (c->profile == 2 && (cls == 0 || cls == 3 || (cls == 1 && c->p.think_every > 1)));
  if (rec) {
    a = get_event(c);
    b = get_event(c);
    // External: inside a stream capture (graph_step) the record becomes an
    // event-record node of the graph instead of a capture-internal marker
    CK(cudaEventRecordWithFlags(a, c->stream, c->capturing ? cudaEventRecordExternal : cudaEventRecordDefault));
  }
  CK(f());
  c->launches += kernels;
  if (rec) {
    CK(cudaEventRecordWithFlags(b, c->stream, c->capturing ? cudaEventRecordExternal : cudaEventRecordDefault));
    c->recs.push_back({cls, a, b});
  }
  return BOIDS_OK;
}

int create_impl(int64_t n, const boids_params* p, uint64_t seed, int32_t rank, int32_t world,
                bool shard, boids_ctx** out) {
  if (!out) return fail(BOIDS_EINVAL, "out is NULL");
  *out = nullptr;
  if (n < 1) return fail(BOIDS_EINVAL, "n must be >= 1");
  if (n > (int64_t)0x7FFFFFFF) return fail(BOIDS_EINVAL, "n must fit in int32 (neighbour indices)");
  if (world < 1 || rank < 0 || rank >= world) return fail(BOIDS_EINVAL, "bad rank/world");
  int rc = validate(p);
  if (rc) return rc;
  boids_ctx* c = new (std::nothrow) boids_ctx();
  if (!c) return fail(BOIDS_ENOMEM, "host allocation failed");
  c->n = n;
  c->rank = rank;
  c->world = world;
  c->shard = shard;
  c->p = *p;
  cudaGetDevice(&c->dev);
  cudaDeviceGetAttribute(&c->sm_count, cudaDevAttrMultiProcessorCount, c->dev);
  int64_t per = (n + world - 1) / world;
  c->m = (per + TILE - 1) / TILE * TILE;
  c->lo = std::min<int64_t>((int64_t)rank * c->m, n);
  c->hi = std::min<int64_t>((int64_t)(rank + 1) * c->m, n);
  c->nloc = c->hi - c->lo;
  int64_t m = c->m;
  auto alloc = [&](void** ptr, size_t bytes) -> int {
    cudaError_t e = cudaMalloc(ptr, bytes);
    if (e != cudaSuccess) {
      (void)cudaGetLastError();
      return fail(BOIDS_ENOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
    }
    return BOIDS_OK;
  };
  size_t seg = (size_t)2 * m * sizeof(float4);
  if ((rc = alloc((void**)&c->buf[0], shard ? seg * world : seg)) ||
      (rc = alloc((void**)&c->buf[1], seg)) ||
      (rc = alloc((void**)&c->up4, m * sizeof(float4))) ||
      (rc = alloc((void**)&c->side4, m * sizeof(float4))) ||
      (rc = alloc((void**)&c->nbr, m * 7 * sizeof(int32_t))) ||
      (rc = alloc((void**)&c->cnt, m * sizeof(int32_t)))) {
    free_ctx(c);
    return rc;
  }
  const int64_t slots = shard ? (int64_t)world * m : m;
  c->loc_grid = make_locality_grid(n, *p);
  c->ncand = (n + TILE - 1) / TILE * TILE;
  if ((rc = alloc((void**)&c->cellrank, slots * sizeof(int2))) ||
      (rc = alloc((void**)&c->bcnt, c->loc_grid.cells * sizeof(int32_t))) ||
      (rc = alloc((void**)&c->bstart, (c->loc_grid.cells + 1) * sizeof(int32_t))) ||
      (rc = alloc((void**)&c->qperm, m * sizeof(int32_t))) ||
      (rc = alloc((void**)&c->cand, c->ncand * sizeof(float4))) ||
      (rc = alloc((void**)&c->stats, 4 * sizeof(unsigned long long))) ||
      (rc = alloc((void**)&c->nbr8, m * sizeof(int32_t))) ||
      (rc = alloc((void**)&c->fstore, m * sizeof(float4))) ||
      (rc = alloc((void**)&c->routed, m)) ||
      (rc = alloc((void**)&c->tcold, m * sizeof(int32_t))) ||
      (rc = alloc((void**)&c->twarm, m * sizeof(int32_t))) ||
      (rc = alloc((void**)&c->tcnt, 2 * sizeof(int32_t))) ||
      (rc = alloc((void**)&c->ocheck, 2 * sizeof(int)))) {
    free_ctx(c);
    return rc;
  }
  if (p->search_mode == BOIDS_GRID) {
    c->sgrid = make_search_grid(*p);
    c->qgrid = make_query_grid(c->sgrid);
    c->bgrid = c->sgrid;
    c->bqgrid = c->qgrid;
    const int C = c->sgrid.cells;
    if ((rc = alloc((void**)&c->gcellrank, slots * sizeof(int2))) ||
        (rc = alloc((void**)&c->gcnt, C * sizeof(int32_t))) ||
        (rc = alloc((void**)&c->gstart, (C + 1) * sizeof(int32_t))) ||
        (rc = alloc((void**)&c->gqstart, (C + 1) * sizeof(int32_t))) ||
        (rc = alloc((void**)&c->gitems, (size_t)(C + m / 128 + 2) * sizeof(int4))) ||
        (rc = alloc((void**)&c->gnitems, sizeof(int32_t))) ||
        (rc = alloc((void**)&c->growbuf, (size_t)2 * (C / c->sgrid.dim[0] + 1) * sizeof(int32_t))) ||
        (rc = alloc((void**)&c->counter, sizeof(int32_t))) ||
        (rc = alloc((void**)&c->sym_rlist, m * sizeof(int32_t))) ||
        (rc = alloc((void**)&c->sym_rcount, sizeof(int32_t))) ||
        (rc = alloc((void**)&c->qlim, m * sizeof(float))) ||
        (rc = alloc((void**)&c->spos, (size_t)n * sizeof(float4)))) {
      free_ctx(c);
      return rc;
    }
  } else if ((rc = alloc((void**)&c->hits, (size_t)m * (p->think_every > 1 ? HITS_THINK : HITS) * sizeof(unsigned long long))) ||
             (rc = alloc((void**)&c->hitcnt, m * sizeof(int32_t))) ||
             (rc = alloc((void**)&c->partial, (size_t)m * PSLOTS * 7 * sizeof(unsigned long long))) ||
             (rc = alloc((void**)&c->pcnt, m * sizeof(int32_t))) ||
             (rc = alloc((void**)&c->qlim, m * sizeof(float))) ||
             (rc = alloc((void**)&c->sym_rlist, m * sizeof(int32_t))) ||
             (rc = alloc((void**)&c->sym_rcount, sizeof(int32_t))) ||
             (rc = alloc((void**)&c->rpart, (size_t)m * 16 * 8 * sizeof(unsigned long long))) ||
             (rc = alloc((void**)&c->rbcount, (size_t)m * sizeof(int32_t))) ||
             (!shard && ((rc = alloc((void**)&c->sym_sp, sym_capacity(c->nloc) * sizeof(float4))) ||
                         (rc = alloc((void**)&c->sym_idx, sym_capacity(c->nloc) * sizeof(int32_t))) ||
                         (rc = alloc((void**)&c->sym_fb, (2 * SYM_FB_LEN + SYM_FB_MAX_CTAS + 1) * sizeof(long long)))))) {
    free_ctx(c);
    return rc;
  }
  if (p->steer_mode == BOIDS_STEER_OPENSTEER && (rc = alloc((void**)&c->acc4, m * sizeof(float4)))) {
    free_ctx(c);
    return rc;
  }
  cudaStream_t s = c->stream;
  cudaError_t e = cudaSuccess;
  if (c->acc4) e = cudaMemsetAsync(c->acc4, 0, m * sizeof(float4), s);
  // phantoms in every segment of every buffer; then the owned agents
  if (e == cudaSuccess) e = cudaMemsetAsync(c->buf[0], 0, shard ? seg * world : seg, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->buf[1], 0, seg, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->cnt, 0xFF, m * sizeof(int32_t), s);  // -1: never searched
  if (e == cudaSuccess && c->sym_fb) e = cudaMemsetAsync(c->sym_fb, 0, 2 * SYM_FB_LEN * sizeof(long long), s);
  if (e == cudaSuccess && c->rbcount) e = cudaMemsetAsync(c->rbcount, 0, (size_t)m * sizeof(int32_t), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->fstore, 0, m * sizeof(float4), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->routed, 0, m, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->nbr, 0xFF, m * 7 * sizeof(int32_t), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->up4, 0, m * sizeof(float4), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->side4, 0, m * sizeof(float4), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->bcnt, 0, c->loc_grid.cells * sizeof(int32_t), s);
  if (e == cudaSuccess) e = launch_fill_nan(c->cand, c->ncand, s);  // entries >= n stay NaN
  if (e == cudaSuccess) e = cudaMemsetAsync(c->stats, 0, 4 * sizeof(unsigned long long), s);
  if (e == cudaSuccess && c->hitcnt) e = cudaMemsetAsync(c->hitcnt, 0, m * sizeof(int32_t), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->nbr8, 0xFF, m * sizeof(int32_t), s);
  if (e == cudaSuccess && c->pcnt) e = cudaMemsetAsync(c->pcnt, 0, m * sizeof(int32_t), s);
  if (e == cudaSuccess && c->gcnt) e = cudaMemsetAsync(c->gcnt, 0, c->sgrid.cells * sizeof(int32_t), s);
  if (e == cudaSuccess)
    e = launch_fill_phantoms(c->buf[0], m, shard ? 0 : c->nloc, shard ? world : 1, s);
  if (e == cudaSuccess) e = launch_fill_phantoms(c->buf[1], m, c->nloc, 1, s);
  if (e == cudaSuccess) e = launch_init(c->local(), c->up4, c->side4, m, c->lo, c->nloc, c->p, seed, s);
  if (e == cudaSuccess && !shard) e = cudaMemcpyAsync(c->buf[1], c->buf[0], seg, cudaMemcpyDeviceToDevice, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) {
    (void)cudaGetLastError();
    free_ctx(c);
    return fail(BOIDS_ECUDA, std::string("create: ") + cudaGetErrorString(e));
  }
  *out = c;
  return BOIDS_OK;
}

StepArgs make_args(boids_ctx* c, float dt) {
  StepArgs a;
  a.full = c->shard ? c->buf[0] : c->buf[c->cur];
  a.out = c->shard ? c->buf[1] : c->buf[c->cur ^ 1];
  a.up4 = c->up4;
  a.side4 = c->side4;
  a.force4 = c->record_steering ? c->force4 : nullptr;
  a.nbr = c->nbr;
  a.cnt = c->cnt;
  a.n = c->n;
  a.m = c->m;
  a.sdiv = make_slice_div(c->m, c->shard ? c->world : 1);
  a.lo = c->lo;
  a.nloc = c->nloc;
  a.world = c->shard ? c->world : 1;
  a.warm = c->warm ? 1 : 0;
  a.dt = dt;
  a.p = c->p;
  a.cand = c->cand;
  a.ncand = c->ncand;
  a.qperm = c->qperm;
  a.stats = c->stats;
  a.phase = c->phase;
  a.vote_u = c->vote_u;
  a.hits = c->hits;
  a.hits_cap = c->p.think_every > 1 ? HITS_THINK : HITS;
  a.hitcnt = c->hitcnt;
  a.nbr8 = c->nbr8;
  a.partial = c->partial;
  a.pcnt = c->pcnt;
  a.qlim = c->qlim;
  a.think_k = c->p.think_every;
  a.store_only = 0;
  a.step_t = c->step_index;
  a.fstore = c->fstore;
  a.qcount = nullptr;
  a.nq = c->nloc;
  a.routed = c->p.think_every > 1 ? c->routed : nullptr;
  a.rlist = c->sym_rlist;  // warm brute-force steps route overflowed agents to k_route
  a.rcount = c->sym_rcount;
  a.rpart = c->rpart;
  a.rbcount = c->rbcount;
  a.loc = c->loc_grid;
  a.acc4 = c->acc4;
  a.lstart = c->bstart;  // brute-force steps sort the queries (qperm) before any search
  return a;
}

int one_step(boids_ctx* c, float dt) {
  StepArgs a = make_args(c, dt);
  int rc;
  const bool grid = c->p.search_mode == BOIDS_GRID;
  const bool think = c->p.think_every > 1;
  if (think && !grid && c->kernel != BOIDS_KERNEL_FUSED)
    return fail(BOIDS_EINVAL, "think frequency runs on the default kernels (BOIDS_KERNEL_FUSED or BOIDS_GRID)");
  // Only the warm path keeps the 8th-nearest seed consistent with the lists it
  // writes; other steps invalidate it (a stale seed could repeat one of the new 7
  // neighbours and break the t0 bound).  Think mode keeps it per agent (k_select
  // writes it for warm thinkers, k_think_compact clears it for cold ones).
  const bool warm_path = !grid && !think && c->kernel == BOIDS_KERNEL_FUSED && c->warm;
  if (!warm_path && !(think && !grid)) CK(mset(c, c->nbr8, 0xFF, c->m * sizeof(int32_t)));
  if (grid) {
    // a2: bin all agents (candidates) and the owned ones (queries) by search cell;
    // think mode: only this step's thinkers are queries
    // candidates: every agent by fine search cell (spos, gstart); queries: the
    // owned agents (this step's thinkers in think mode) by block of cells
    // (qperm, gqstart) and the work items over the blocks
    const int64_t slots = c->shard ? (int64_t)c->world * c->m : c->m;
    // owned queries: a spatial shard owns about n / world of its n slots
    const int chunk = grid_chunk(c->spatial ? c->nloc / c->world : c->nloc / (think ? c->p.think_every : 1));
    if ((rc = launch(c, 2, [&] {
           cudaError_t e = launch_bin(a.full, c->m, a.sdiv, 0, slots, c->bgrid, c->gcellrank, c->gcnt, c->gstart,
                                      c->spos, nullptr, 0, c->stream, nullptr, nullptr, nullptr, chunk, nullptr, 1,
                                      0, c->growbuf);
           if (e == cudaSuccess)
             e = launch_bin(a.full, c->m, a.sdiv, c->lo, c->nloc, c->bqgrid, c->gcellrank, c->gcnt, c->gqstart,
                            nullptr, c->qperm, (int)c->lo, c->stream, nullptr, c->gitems, c->gnitems, chunk,
                            c->counter, c->p.think_every, c->step_index, c->growbuf, c->spatial ? c->own : nullptr);
           return e;
         }, 6)))
      return rc;
    GridArgs g;
    g.spos = c->spos;
    g.cstart = c->gstart;
    g.qstart = c->gqstart;
    g.qperm = c->qperm;
    g.items = c->gitems;
    g.nitems = c->gnitems;
    g.flist = c->sym_rlist;  // (the brute-force routing list; unused in grid mode otherwise)
    g.fcount = c->sym_rcount;
    g.flim = c->qlim;
    g.counter = c->counter;
    g.grid = c->bgrid;
    g.qgrid = c->bqgrid;
    StepArgs ag = a;
    ag.store_only = think ? 1 : 0;
    CK(mset(c, c->sym_rcount, 0, sizeof(int32_t)));
    c->last_path = BOIDS_PATH_GRID;
    if ((rc = launch(c, 3, [&] { return launch_grid(ag, g, c->stream); }))) return rc;
    if ((rc = launch(c, 4, [&] { return launch_grid_far(ag, g, c->stream); }))) return rc;
    if (think && (rc = launch(c, 1, [&] { return launch_apply(a, c->stream); }))) return rc;
  } else if (c->kernel == BOIDS_KERNEL_SIMPLE) {
    c->last_path = BOIDS_PATH_SIMPLE;
    if ((rc = launch(c, 0, [&] { return launch_search_simple(a, c->stream); }))) return rc;
    if ((rc = launch(c, 1, [&] { return launch_update(a, c->stream); }))) return rc;
  } else {
    // small flocks: the whole warm step in one kernel (k_small.cu), no spatial order needed
    const bool small = warm_path && !think && !c->shard && c->use_small && c->nloc < small_max();
    if (small) {
      c->last_path = BOIDS_PATH_SMALL;
      if ((rc = launch(c, 0, [&] { return launch_small(a, c->stream); }))) return rc;
    }
    // a2: spatial (Morton) order of the owned queries, so the 128 queries of a
    // warp are spatially coherent.  It is only a permutation of the work (results
    // never depend on it), so it is refreshed every resort_every steps.
    if (!small && (c->since_sort < 0 || c->since_sort >= c->resort_every)) {
      if ((rc = launch(c, 2, [&] {
             return launch_bin(a.full, c->m, a.sdiv, c->lo, c->nloc, c->loc_grid, c->cellrank, c->bcnt, c->bstart,
                               nullptr, c->qperm, (int)c->lo, c->stream, nullptr);
           }, 3)))
        return rc;
      c->since_sort = 0;
      c->steps_sorted++;
    }
    if (!small) c->since_sort++;
    if (small) {
      // done above
    } else if (think) {
      // this step's thinkers, in spatial order, split into never-searched (cold)
      // and warm-bounded ones
      c->last_path = BOIDS_PATH_THINK;
      CK(mset(c, c->tcnt, 0, 2 * sizeof(int32_t)));
      if ((rc = launch(c, 2, [&] {
             return launch_think_compact(a, c->qperm, c->tcold, c->tcnt, c->twarm, c->tcnt + 1, c->stream);
           })))
        return rc;
      if (c->steps_taken < c->p.think_every) {  // some agents have never thought
        StepArgs ac = a;
        ac.qperm = c->tcold;
        ac.qcount = c->tcnt;
        ac.store_only = 1;
        const int cl = c->cluster_opt;
        if ((rc = launch(c, 0, [&] { return launch_fused(ac, cl, c->stream); }))) return rc;
      }
      StepArgs aw = a;
      aw.qperm = c->twarm;
      aw.qcount = c->tcnt + 1;
      CK(mset(c, c->sym_rcount, 0, sizeof(int32_t)));
      if ((rc = launch(c, 0, [&] { return launch_warm_scan(aw, c->stream); }, 2))) return rc;
      if ((rc = launch(c, 1, [&] { return launch_warm_select(a, c->stream); }))) return rc;
      if ((rc = launch(c, 4, [&] { return launch_route(a, c->stream); }))) return rc;
    } else if (warm_path) {
      // warm step: all-pairs scan appending passing keys, then select + update;
      // a single-GPU handle evaluates each unordered pair once (k_sym) from 8192
      // agents on (below, k_small runs the whole step unless BOIDS_OPT_SMALL is
      // off; then the ordered-pair path, one launch shorter, is the faster one)
      static const int64_t sym_min = [] {
        const char* e = getenv("BOIDS_SYM_MIN");  // diagnostics: smallest n on k_sym
        return e ? atoll(e) : 8192LL;
      }();
      if (c->symmetric && c->sym_sp && c->nloc >= sym_min) {
        c->last_path = BOIDS_PATH_SYM;
        StepArgs as = a;
        as.routed = c->routed;  // agents routed to k_route by k_sym_prep (k_select skips them)
        CK(mset(c, c->sym_rcount, 0, sizeof(int32_t)));
        long long* fb_prev = c->sym_fb + (c->sym_fb_par ^ 1) * SYM_FB_LEN;
        long long* fb_cur = c->sym_fb + c->sym_fb_par * SYM_FB_LEN;
        c->sym_fb_par ^= 1;
        // two launch records: the prologue (class 5) and k_sym itself (class 0, the search roofline)
        for (int part = 1; part <= 2; ++part)
          if ((rc = launch(c, part == 1 ? 5 : 0, [&] {
                 return launch_sym_scan(as, c->sym_sp, c->sym_idx, c->balance ? fb_prev : nullptr, fb_cur,
                                        c->sym_fb + 2 * SYM_FB_LEN, c->stream, part);
               })))
            return rc;
        if ((rc = launch(c, 1, [&] { return launch_warm_select(as, c->stream, false); }))) return rc;
        if ((rc = launch(c, 4, [&] { return launch_route(as, c->stream); }))) return rc;
      } else {
        c->last_path = BOIDS_PATH_SCAN;
        CK(mset(c, c->sym_rcount, 0, sizeof(int32_t)));
        if ((rc = launch(c, 0, [&] { return launch_warm_scan(a, c->stream); }, 2))) return rc;
        if ((rc = launch(c, 1, [&] { return launch_warm_select(a, c->stream); }))) return rc;
        if ((rc = launch(c, 4, [&] { return launch_route(a, c->stream); }))) return rc;
      }
    } else {
      // cold step (no previous lists) or forced: the cluster kernel
      c->last_path = BOIDS_PATH_FUSED;
      int cl = c->cluster_opt;
      if ((rc = launch(c, 0, [&] { return launch_fused(a, cl, c->stream); }))) return rc;
    }
  }
  if (!c->shard) c->cur ^= 1;
  if (c->spatial) {  // the new positions decide migrants and halo copies (k_spatial.cu)
    CK(mset(c, c->sp_counts, 0, 2 * c->world * sizeof(int)));
    if ((rc = launch(c, 2, [&] {
           return launch_spatial_pack(c->buf[c->cur], c->buf[c->cur ^ 1], c->m, c->n, c->own, c->up4, c->side4, c->nbr, c->cnt, c->nbr8,
                                      c->acc4, c->sgrid, c->zb, c->world, c->rank, c->sp_reach, c->halo_out, c->cap_h,
                                      c->mig_out, c->cap_m, c->sp_counts, c->sp_overflow, c->halo_in, c->last_nh,
                                      c->kept, c->nkept, c->kept_bound, c->stream);
         })))
      return rc;
    c->kept_bound = c->n;  // refined by boids_spatial_outbox (it reads the count)
    c->last_nh = 0;
  }
  c->warm = true;
  c->steering_valid = c->record_steering;
  c->step_index++;
  c->steps_taken++;
  return BOIDS_OK;
}

// boids_step's CUDA-graph path: warm single-rank steps without profiling or
// think frequency replay a captured graph of the step's launches (the host
// launch cost of 4-6 kernels and memsets per step becomes one graph launch; the
// PDL edges are captured as programmatic graph edges).  The launch sequence of
// a step is fixed by host-side state: whether the spatial query order is
// rebuilt this step, the k_sym feedback-record parity and the ping-pong buffer
// parity; together with dt they key the cache.  A replay first advances that
// host state by a dry run of one_step (nothing enqueued), exactly as the
// captured run did.  Results never depend on the path taken.
// Profiling (BOIDS_OPT_PROFILE) works inside graphs: the event records that
// bracket a profiled launch are captured as event-record nodes, and every replay
// points them at fresh events first (cudaGraphExecEventRecordNodeSetEvent), so
// each replayed launch is timed like an eager one.
bool graph_ok(const boids_ctx* c) {
  const bool grid = c->p.search_mode == BOIDS_GRID;
  return c->use_graphs && !c->shard && !c->spatial && c->p.think_every == 1 && c->phase == nullptr && c->steps_taken >= 2 &&
         (grid || (c->warm && c->kernel == BOIDS_KERNEL_FUSED));
}

void clear_graphs(boids_ctx* c) {
  for (auto& g : c->graphs) {
    cudaGraphExecDestroy(g.exec);
    cudaGraphDestroy(g.graph);
  }
  c->graphs.clear();
}

int graph_step(boids_ctx* c, float dt) {
  const bool resort = c->since_sort < 0 || c->since_sort >= c->resort_every;
  const uint32_t key = (resort ? 1u : 0u) | ((uint32_t)c->sym_fb_par << 1) | ((uint32_t)c->cur << 2);
  for (auto& g : c->graphs)
    if (g.key == key && g.dt == dt) {
      c->dry = true;
      const int rc = one_step(c, dt);
      c->dry = false;
      if (rc) return rc;
      for (auto& pr : g.prof) {
        cudaEvent_t ea = get_event(c), eb = get_event(c);
        CK(cudaGraphExecEventRecordNodeSetEvent(g.exec, pr.a, ea));
        CK(cudaGraphExecEventRecordNodeSetEvent(g.exec, pr.b, eb));
        c->recs.push_back({pr.cls, ea, eb});
      }
      CK(cudaGraphLaunch(g.exec, c->stream));
      c->graph_launches++;
      return BOIDS_OK;
    }
  if (c->graphs.size() >= 16) clear_graphs(c);  // e.g. a caller cycling through many dt values
  if (!c->cap_stream) CK(cudaStreamCreateWithFlags(&c->cap_stream, cudaStreamNonBlocking));
  cudaStream_t orig = c->stream;
  c->stream = c->cap_stream;
  cudaError_t e = cudaStreamBeginCapture(c->cap_stream, cudaStreamCaptureModeRelaxed);
  if (e != cudaSuccess) {
    c->stream = orig;
    CK(e);
  }
  const size_t rec0 = c->recs.size();
  c->capturing = true;
  const int rc = one_step(c, dt);
  c->capturing = false;
  cudaGraph_t g = nullptr;
  e = cudaStreamEndCapture(c->cap_stream, &g);
  c->stream = orig;
  if (rc) {
    if (g) cudaGraphDestroy(g);
    return rc;
  }
  CK(e);
  // the event-record nodes of the profiled launches of this step (if any)
  std::vector<boids_ctx::GraphEntry::Prof> prof;
  if (c->recs.size() > rec0) {
    size_t nn = 0;
    CK(cudaGraphGetNodes(g, nullptr, &nn));
    std::vector<cudaGraphNode_t> nodes(nn);
    CK(cudaGraphGetNodes(g, nodes.data(), &nn));
    auto node_of = [&](cudaEvent_t ev) -> cudaGraphNode_t {
      for (auto nd : nodes) {
        cudaGraphNodeType t;
        cudaEvent_t x = nullptr;
        if (cudaGraphNodeGetType(nd, &t) == cudaSuccess && t == cudaGraphNodeTypeEventRecord &&
            cudaGraphEventRecordNodeGetEvent(nd, &x) == cudaSuccess && x == ev)
          return nd;
      }
      return nullptr;
    };
    for (size_t i = rec0; i < c->recs.size(); ++i) {
      const auto& r = c->recs[i];
      prof.push_back({r.cls, node_of(r.a), node_of(r.b)});
      if (!prof.back().a || !prof.back().b) {
        cudaGraphDestroy(g);
        return fail(BOIDS_ECUDA, "graph capture: profiling event node not found");
      }
    }
  }
  cudaGraphExec_t exec = nullptr;
  e = cudaGraphInstantiate(&exec, g, 0);
  if (e != cudaSuccess) cudaGraphDestroy(g);
  CK(e);
  c->graphs.push_back({key, dt, exec, g, prof});
  CK(cudaGraphLaunch(exec, c->stream));
  c->graph_launches++;
  return BOIDS_OK;
}

}  // namespace

bool boids::pdl_enabled() {
  static const bool v = [] {
    const char* e = getenv("BOIDS_PDL");
    return !(e && atoi(e) == 0);
  }();
  return v;
}

bool boids::pdl_env(const char* name) {
  const char* e = getenv(name);
  return !(e && atoi(e) == 0);
}

int boids::carveout_pct() {
  static const int v = [] {
    const char* e = getenv("BOIDS_CARVEOUT");
    return e ? atoi(e) : 100;
  }();
  return v;
}

namespace {

int check_dt(float dt) {
  if (!std::isfinite(dt) || dt < 0.f) return fail(BOIDS_EINVAL, "dt must be finite and >= 0");
  return BOIDS_OK;
}

void to_aos(const std::vector<float4>& v, int64_t count, float* out, bool w) {
  for (int64_t i = 0; i < count; ++i) {
    if (w) {
      out[i] = v[i].w;
    } else {
      out[3 * i] = v[i].x;
      out[3 * i + 1] = v[i].y;
      out[3 * i + 2] = v[i].z;
    }
  }
}

}  // namespace

extern "C" {

BOIDS_API void boids_default_params(boids_params* out) {
  if (!out) return;
  out->search_radius = 9.0f;
  out->w_separation = 12.0f;
  out->w_alignment = 8.0f;
  out->w_cohesion = 8.0f;
  out->max_force = 27.0f;
  out->max_speed = 9.0f;
  out->mass = 1.0f;
  out->world_radius = 50.0f;
  out->init_radius = 20.0f;
  out->init_speed_frac = 0.3f;
  out->max_neighbors = 7;
  out->search_mode = BOIDS_BRUTE;
  out->init_mode = BOIDS_INIT_OPENSTEER;
  out->think_every = 1;
  out->steer_mode = BOIDS_STEER_THESIS;
}

BOIDS_API int boids_create(int64_t n, const boids_params* p, uint64_t seed, boids_ctx** out) {
  return create_impl(n, p, seed, 0, 1, false, out);
}

BOIDS_API int boids_create_shard(int64_t n, const boids_params* p, uint64_t seed, int32_t rank,
                       int32_t world, boids_ctx** out) {
  return create_impl(n, p, seed, rank, world, true, out);
}

// ---- sym-shards: boids_symshard_prep / _search / _finish (include/boids.h) ----
static int ss_check(boids_ctx* c) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->shard || c->p.search_mode != BOIDS_BRUTE || c->p.think_every != 1 || c->kernel != BOIDS_KERNEL_FUSED)
    return fail(BOIDS_EINVAL, "sym-shards: a brute-force shard handle (think_every 1, default kernels)");
  if (!c->warm) return fail(BOIDS_EINVAL, "sym-shards step warm handles: run the first step with boids_step_shard");
  return BOIDS_OK;
}

static int ss_alloc(boids_ctx* c) {
  if (c->ss_lim_send) return BOIDS_OK;
  const int64_t slots = (int64_t)c->world * c->m;
  const size_t hcap = (size_t)slots * SS_HITS * sizeof(unsigned long long);
  cudaError_t e;
  if ((e = cudaMalloc((void**)&c->ss_lim_send, c->m * sizeof(float))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_lim_full, slots * sizeof(float))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_hits, hcap)) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_recv, hcap)) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_hitcnt, slots * sizeof(int32_t))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_rcnt, slots * sizeof(int32_t))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_gperm, slots * sizeof(int32_t))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_gbcnt, c->loc_grid.cells * sizeof(int32_t))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_gbstart, (c->loc_grid.cells + 1) * sizeof(int32_t))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->ss_spos, slots * sizeof(float4))) != cudaSuccess ||
      (!c->sym_sp && (e = cudaMalloc((void**)&c->sym_sp, sym_capacity(slots) * sizeof(float4))) != cudaSuccess) ||
      (!c->sym_idx && (e = cudaMalloc((void**)&c->sym_idx, sym_capacity(slots) * sizeof(int32_t))) != cudaSuccess) ||
      (!c->sym_fb &&
       (e = cudaMalloc((void**)&c->sym_fb, (2 * SYM_FB_LEN + SYM_FB_MAX_CTAS + 1) * sizeof(long long))) != cudaSuccess)) {
    (void)cudaGetLastError();
    return fail(BOIDS_ENOMEM, std::string("sym-shard buffers: ") + cudaGetErrorString(e));
  }
  CK(cudaMemsetAsync(c->ss_gbcnt, 0, c->loc_grid.cells * sizeof(int32_t), c->stream));
  CK(cudaMemsetAsync(c->sym_fb, 0, 2 * SYM_FB_LEN * sizeof(long long), c->stream));
  CK(cudaMemsetAsync(c->ss_lim_full, 0, slots * sizeof(float), c->stream));
  return BOIDS_OK;
}

BOIDS_API int boids_symshard_prep(boids_ctx* c) {
  int rc = ss_check(c);
  if (rc) return rc;
  DeviceGuard g(c->dev);
  if ((rc = ss_alloc(c))) return rc;
  StepArgs a = make_args(c, 0.f);
  a.routed = c->routed;
  const int64_t slots = (int64_t)c->world * c->m;
  // the global Morton order, identical on every rank (cells sorted by index): the
  // limits' window bound looks agents up in it, and the search walks it
  if (c->ss_since_sort < 0 || c->ss_since_sort >= c->resort_every) {
    if ((rc = launch(c, 2, [&] {
           cudaError_t e = launch_bin(a.full, c->m, a.sdiv, 0, slots, c->loc_grid, c->cellrank, c->ss_gbcnt,
                                      c->ss_gbstart, c->ss_spos, c->ss_gperm, 0, c->stream, nullptr);
           if (e == cudaSuccess) e = launch_ss_cellsort(c->ss_gperm, c->ss_gbstart, c->loc_grid.cells, c->stream);
           return e;
         }, 4)))
      return rc;
    c->ss_since_sort = 0;
    c->steps_sorted++;
  }
  c->ss_since_sort++;
  CK(cudaMemsetAsync(c->sym_rcount, 0, sizeof(int32_t), c->stream));
  // class 4 (with the routing): the search class (0) holds one record per step, the triangle share
  return launch(c, 4, [&] { return launch_ss_lim(a, c->ss_lim_send, c->ss_gperm, c->ss_gbstart, c->n, c->stream); });
}

BOIDS_API int boids_symshard_search(boids_ctx* c) {
  int rc = ss_check(c);
  if (rc) return rc;
  if (!c->ss_lim_send) return fail(BOIDS_EINVAL, "boids_symshard_prep first");
  DeviceGuard g(c->dev);
  StepArgs a = make_args(c, 0.f);
  const int64_t slots = (int64_t)c->world * c->m;
  CK(cudaMemsetAsync(c->ss_hitcnt, 0, slots * sizeof(int32_t), c->stream));
  StepArgs as = a;
  as.hits = c->ss_hits;
  as.hitcnt = c->ss_hitcnt;
  as.hits_cap = SS_HITS;
  long long* fb_prev = c->sym_fb + (c->sym_fb_par ^ 1) * SYM_FB_LEN;
  long long* fb_cur = c->sym_fb + c->sym_fb_par * SYM_FB_LEN;
  c->sym_fb_par ^= 1;
  return launch(c, 0, [&] {
    return launch_ss_search(as, c->ss_gperm, c->n, c->ss_lim_full, c->sym_sp, c->sym_idx, c->balance ? fb_prev : nullptr,
                            fb_cur, c->sym_fb + 2 * SYM_FB_LEN, c->rank, c->world, c->stream);
  }, 2);
}

BOIDS_API int boids_symshard_finish(boids_ctx* c, float dt) {
  int rc = ss_check(c);
  if (rc) return rc;
  if ((rc = check_dt(dt))) return rc;
  if (!c->ss_lim_send) return fail(BOIDS_EINVAL, "boids_symshard_prep first");
  DeviceGuard g(c->dev);
  StepArgs a = make_args(c, dt);
  a.routed = c->routed;
  a.hits_cap = SS_HITS;
  if ((rc = launch(c, 1, [&] { return launch_ss_select(a, c->ss_recv, c->ss_rcnt, c->world, c->stream); }))) return rc;
  if ((rc = launch(c, 4, [&] { return launch_route(a, c->stream); }))) return rc;
  c->last_path = BOIDS_PATH_SYM;
  c->warm = true;
  c->steering_valid = c->record_steering;
  c->step_index++;
  c->steps_taken++;
  return BOIDS_OK;
}

BOIDS_API int boids_symshard_buffers(boids_ctx* c, void** lim_send, void** lim_full, void** hits, void** hitcnt,
                                     void** recv, void** rcnt, int32_t* hits_cap) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->shard || c->p.search_mode != BOIDS_BRUTE) return fail(BOIDS_EINVAL, "not a brute-force shard handle");
  DeviceGuard g(c->dev);
  int rc = ss_alloc(c);
  if (rc) return rc;
  if (lim_send) *lim_send = c->ss_lim_send;
  if (lim_full) *lim_full = c->ss_lim_full;
  if (hits) *hits = c->ss_hits;
  if (hitcnt) *hitcnt = c->ss_hitcnt;
  if (recv) *recv = c->ss_recv;
  if (rcnt) *rcnt = c->ss_rcnt;
  if (hits_cap) *hits_cap = SS_HITS;
  return BOIDS_OK;
}

BOIDS_API int boids_create_spatial(int64_t n, const boids_params* p, uint64_t seed, int32_t rank, int32_t world,
                                   boids_ctx** out) {
  if (!out) return fail(BOIDS_EINVAL, "out is NULL");
  *out = nullptr;
  if (!p) return fail(BOIDS_EINVAL, "params is NULL");
  if (p->search_mode != BOIDS_GRID) return fail(BOIDS_EINVAL, "spatial shards need search_mode = BOIDS_GRID");
  if (p->think_every != 1) return fail(BOIDS_EINVAL, "spatial shards need think_every = 1");
  if (world < 1 || world > 256 || rank < 0 || rank >= world) return fail(BOIDS_EINVAL, "bad rank/world");
  boids_ctx* c = nullptr;
  int rc = create_impl(n, p, seed, 0, 1, false, &c);
  if (rc) return rc;
  c->spatial = true;
  c->rank = rank;
  c->world = world;
  c->sp_reach = c->sgrid.reach;
  const int L = c->sgrid.dim[2];
  auto bad = [&](cudaError_t e) -> int {
    (void)cudaGetLastError();
    free_ctx(c);
    return fail(e == cudaErrorMemoryAllocation ? BOIDS_ENOMEM : BOIDS_ECUDA,
                std::string("create_spatial: ") + cudaGetErrorString(e));
  };
  // slab boundaries: equal shares of the initial agents over the cell layers z
  // (every rank holds all n initial agents and computes the same boundaries)
  int* hist = nullptr;
  cudaError_t e = cudaMalloc((void**)&hist, L * sizeof(int));
  if (e == cudaSuccess) e = cudaMemsetAsync(hist, 0, L * sizeof(int), c->stream);
  if (e == cudaSuccess) e = launch_zhist(c->buf[c->cur], n, c->sgrid, hist, c->stream);
  std::vector<int> h(L, 0);
  if (e == cudaSuccess) e = cudaMemcpyAsync(h.data(), hist, L * sizeof(int), cudaMemcpyDeviceToHost, c->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
  cudaFree(hist);
  if (e != cudaSuccess) return bad(e);
  c->zb_host.assign(world + 1, L);
  c->zb_host[0] = 0;
  int64_t cum = 0;
  int g = 1;
  for (int z = 0; z < L && g < world; ++z) {
    cum += h[z];
    while (g < world && cum * world >= (int64_t)g * n) c->zb_host[g++] = z + 1;
  }
  for (int k = 1; k <= world; ++k) c->zb_host[k] = std::max(c->zb_host[k], c->zb_host[k - 1]);
  // outbox capacities: the largest halo band of the initial distribution, doubled
  int64_t band = 0;
  for (int d = 0; d < world; ++d) {
    int64_t b = 0;
    for (int z = std::max(0, c->zb_host[d] - c->sp_reach); z < c->zb_host[d]; ++z) b += h[z];
    for (int z = c->zb_host[d + 1]; z < std::min(L, c->zb_host[d + 1] + c->sp_reach); ++z) b += h[z];
    band = std::max(band, b);
  }
  // binning and search over this rank's layers only (its slab and halo): the
  // cell tables and their scans shrink with the slab
  c->bgrid = make_slab_grid(c->sgrid, std::max(0, c->zb_host[rank] - c->sp_reach),
                            std::min(L, c->zb_host[rank + 1] + c->sp_reach));
  c->bqgrid = make_query_grid(c->bgrid);
  c->cap_h = std::max<int64_t>(4096, 2 * band);
  c->cap_m = std::max<int64_t>(4096, n / 16);
  c->cap_in_h = c->cap_h * std::max(1, world - 1);
  c->cap_in_m = c->cap_m * std::max(1, world - 1);
  const size_t hf = spatial_halo_f4() * sizeof(float4), mf = spatial_mig_f4() * sizeof(float4);
  if ((e = cudaMalloc((void**)&c->zb, (world + 1) * sizeof(int))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->own, std::max<int64_t>(1, n))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->halo_out, (size_t)world * c->cap_h * hf)) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->mig_out, (size_t)world * c->cap_m * mf)) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->halo_in, (size_t)c->cap_in_h * hf)) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->mig_in, (size_t)c->cap_in_m * mf)) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->sp_counts, 2 * world * sizeof(int))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->sp_overflow, sizeof(int))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->kept, std::max<int64_t>(1, n) * sizeof(int))) != cudaSuccess ||
      (e = cudaMalloc((void**)&c->nkept, sizeof(int))) != cudaSuccess)
    return bad(e);
  if ((e = cudaMemcpyAsync(c->zb, c->zb_host.data(), (world + 1) * sizeof(int), cudaMemcpyHostToDevice,
                           c->stream)) != cudaSuccess ||
      (e = cudaMemsetAsync(c->sp_counts, 0, 2 * world * sizeof(int), c->stream)) != cudaSuccess ||
      (e = cudaMemsetAsync(c->sp_overflow, 0, sizeof(int), c->stream)) != cudaSuccess ||
      (e = launch_spatial_init(c->buf[c->cur], c->buf[c->cur ^ 1], c->m, n, c->own, c->sgrid, c->zb, world, rank,
                               c->sp_reach, c->kept, c->nkept, c->stream)) != cudaSuccess ||
      (e = cudaStreamSynchronize(c->stream)) != cudaSuccess)
    return bad(e);
  c->kept_bound = n;
  c->last_nh = 0;
  *out = c;
  return BOIDS_OK;
}

BOIDS_API int boids_step_spatial(boids_ctx* c, float dt) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->spatial) return fail(BOIDS_EINVAL, "not a spatial handle");
  int rc = check_dt(dt);
  if (rc) return rc;
  DeviceGuard g(c->dev);
  return one_step(c, dt);
}

BOIDS_API int boids_spatial_outbox(boids_ctx* c, int32_t* halo_counts, int32_t* mig_counts, void** halo_out,
                                   void** mig_out, int64_t* cap_halo, int64_t* cap_mig) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->spatial) return fail(BOIDS_EINVAL, "not a spatial handle");
  DeviceGuard g(c->dev);
  std::vector<int> cnt(2 * c->world);
  int ovf = 0;
  CK(cudaMemcpyAsync(cnt.data(), c->sp_counts, cnt.size() * sizeof(int), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaMemcpyAsync(&ovf, c->sp_overflow, sizeof(int), cudaMemcpyDeviceToHost, c->stream));
  int nk = 0;
  CK(cudaMemcpyAsync(&nk, c->nkept, sizeof(int), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  c->kept_bound = nk;
  if (ovf) return fail(BOIDS_ENOMEM, "spatial outbox overflow (more halo/migrant records than capacity)");
  for (int d = 0; d < c->world; ++d) {
    if (halo_counts) halo_counts[d] = cnt[d];
    if (mig_counts) mig_counts[d] = cnt[c->world + d];
  }
  if (halo_out) *halo_out = c->halo_out;
  if (mig_out) *mig_out = c->mig_out;
  if (cap_halo) *cap_halo = c->cap_h;
  if (cap_mig) *cap_mig = c->cap_m;
  return BOIDS_OK;
}

BOIDS_API int boids_spatial_inbox(boids_ctx* c, void** halo_in, void** mig_in, int64_t* cap_halo_in,
                                  int64_t* cap_mig_in) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->spatial) return fail(BOIDS_EINVAL, "not a spatial handle");
  if (halo_in) *halo_in = c->halo_in;
  if (mig_in) *mig_in = c->mig_in;
  if (cap_halo_in) *cap_halo_in = c->cap_in_h;
  if (cap_mig_in) *cap_mig_in = c->cap_in_m;
  return BOIDS_OK;
}

BOIDS_API int boids_spatial_unpack(boids_ctx* c, int64_t n_halo, int64_t n_mig) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->spatial) return fail(BOIDS_EINVAL, "not a spatial handle");
  if (n_halo < 0 || n_mig < 0 || n_halo > c->cap_in_h || n_mig > c->cap_in_m)
    return fail(BOIDS_EINVAL, "record counts outside the inbox capacities");
  DeviceGuard g(c->dev);
  CK(launch_spatial_unpack(c->halo_in, n_halo, c->mig_in, n_mig, c->buf[c->cur], c->m, c->own, c->up4, c->side4,
                           c->nbr, c->cnt, c->nbr8, c->acc4, c->stream));
  c->last_nh = n_halo;  // these entries are cleared by the next pack (the inbox keeps their records)
  c->launches += (n_halo > 0) + (n_mig > 0);
  return BOIDS_OK;
}

BOIDS_API int boids_spatial_owned(boids_ctx* c, uint8_t* own) {
  if (!c || !own) return fail(BOIDS_EINVAL, "NULL argument");
  if (!c->spatial) return fail(BOIDS_EINVAL, "not a spatial handle");
  DeviceGuard g(c->dev);
  CK(cudaMemcpyAsync(own, c->own, c->n, cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return BOIDS_OK;
}

BOIDS_API int boids_spatial_bounds(boids_ctx* c, int32_t* zb, int32_t* reach) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->spatial) return fail(BOIDS_EINVAL, "not a spatial handle");
  if (zb)
    for (int k = 0; k <= c->world; ++k) zb[k] = c->zb_host[k];
  if (reach) *reach = c->sp_reach;
  return BOIDS_OK;
}

BOIDS_API int boids_set_stream(boids_ctx* c, void* stream) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  c->stream = (cudaStream_t)stream;
  return BOIDS_OK;
}

BOIDS_API int boids_set_option(boids_ctx* c, int32_t opt, int64_t v) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  DeviceGuard g(c->dev);
  CK(cudaStreamSynchronize(c->stream));  // captured graphs may still run: drop them only when done
  clear_graphs(c);
  switch (opt) {
    case BOIDS_OPT_GRAPH:
      c->use_graphs = v != 0;
      return BOIDS_OK;
    case BOIDS_OPT_SMALL:
      c->use_small = v != 0;
      return BOIDS_OK;
    case BOIDS_OPT_RECORD_STEERING:
      if (v && !c->force4) CK(cudaMalloc((void**)&c->force4, c->m * sizeof(float4)));
      c->record_steering = v != 0;
      return BOIDS_OK;
    case BOIDS_OPT_KERNEL:
      if (v != BOIDS_KERNEL_FUSED && v != BOIDS_KERNEL_SIMPLE && v != BOIDS_KERNEL_CLUSTER)
        return fail(BOIDS_EINVAL, "bad kernel");
      c->kernel = (int)v;
      return BOIDS_OK;
    case BOIDS_OPT_PROFILE:
      if (v < 0 || v > 2) return fail(BOIDS_EINVAL, "profile level must be 0, 1 or 2");
      c->profile = (int)v;
      return BOIDS_OK;
    case BOIDS_OPT_SYMMETRIC:
      c->symmetric = v != 0;
      return BOIDS_OK;
    case BOIDS_OPT_BALANCE:
      c->balance = v != 0;
      return BOIDS_OK;
    case BOIDS_OPT_VOTE_U:
      if (v != 4 && v != 8) return fail(BOIDS_EINVAL, "vote width must be 4 or 8");
      c->vote_u = (int)v;
      return BOIDS_OK;
    case BOIDS_OPT_RESORT:
      if (v < 1) return fail(BOIDS_EINVAL, "resort interval must be >= 1");
      c->resort_every = (int)v;
      c->since_sort = -1;
      return BOIDS_OK;
    case BOIDS_OPT_PHASES:
      if (v && !c->phase) {
        CK(cudaMalloc((void**)&c->phase, (size_t)v * 8 * sizeof(unsigned long long)));
        CK(cudaMemset(c->phase, 0, (size_t)v * 8 * sizeof(unsigned long long)));
      }
      if (!v && c->phase) {
        cudaFree(c->phase);
        c->phase = nullptr;
      }
      return BOIDS_OK;
    case BOIDS_OPT_CLUSTER:
      if (v < 0 || v > 16 || (v & (v - 1))) return fail(BOIDS_EINVAL, "cluster must be 0 or a power of two <= 16");
      c->cluster_opt = (int)v;
      return BOIDS_OK;
    default:
      return fail(BOIDS_EINVAL, "unknown option");
  }
}

BOIDS_API int boids_step(boids_ctx* c, float dt, int32_t steps) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (c->shard) return fail(BOIDS_EINVAL, "shard handle: use boids_step_shard after the all-gather");
  if (c->spatial) return fail(BOIDS_EINVAL, "spatial handle: use boids_step_spatial + the record exchange");
  int rc = check_dt(dt);
  if (rc) return rc;
  if (steps < 0) return fail(BOIDS_EINVAL, "steps must be >= 0");
  DeviceGuard g(c->dev);
  for (int32_t t = 0; t < steps; ++t)
    if ((rc = graph_ok(c) ? graph_step(c, dt) : one_step(c, dt))) return rc;
  return BOIDS_OK;
}

BOIDS_API int boids_step_shard(boids_ctx* c, float dt) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->shard) return fail(BOIDS_EINVAL, "not a shard handle");
  int rc = check_dt(dt);
  if (rc) return rc;
  DeviceGuard g(c->dev);
  return one_step(c, dt);
}

BOIDS_API int boids_shard_buffers(boids_ctx* c, void** send, void** full, int64_t* slice_bytes) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->shard) return fail(BOIDS_EINVAL, "not a shard handle");
  if (send) *send = c->buf[1];
  if (full) *full = c->buf[0];
  if (slice_bytes) *slice_bytes = 2 * c->m * (int64_t)sizeof(float4);
  return BOIDS_OK;
}

// Host AoS <-> device float4 state goes through a device staging buffer of 13
// floats per agent ([pos3 | fwd3 | up3 | side3 | speed]) and one conversion
// kernel: the copies are plain DMA of the caller's arrays (pinned memory: full
// PCIe/C2C rate), no host-side conversion loops.
static int ensure_stage(boids_ctx* c) {
  if (!c->stage) {
    cudaError_t e = cudaMalloc((void**)&c->stage, (size_t)13 * (c->m > 0 ? c->m : 1) * sizeof(float));
    if (e != cudaSuccess) {
      (void)cudaGetLastError();
      return fail(BOIDS_ENOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
    }
  }
  return BOIDS_OK;
}

BOIDS_API int boids_get_state(boids_ctx* c, float* pos3, float* fwd3, float* up3, float* side3, float* speed) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  DeviceGuard g(c->dev);
  int rc = ensure_stage(c);
  if (rc) return rc;
  const int64_t k = c->nloc;
  float* st = c->stage;
  CK(launch_state_out(c->local(), c->m, c->up4, c->side4, k, st, c->stream));
  c->launches++;
  const size_t v = (size_t)k * 3 * sizeof(float);
  if (pos3) CK(cudaMemcpyAsync(pos3, st, v, cudaMemcpyDeviceToHost, c->stream));
  if (fwd3) CK(cudaMemcpyAsync(fwd3, st + 3 * k, v, cudaMemcpyDeviceToHost, c->stream));
  if (up3) CK(cudaMemcpyAsync(up3, st + 6 * k, v, cudaMemcpyDeviceToHost, c->stream));
  if (side3) CK(cudaMemcpyAsync(side3, st + 9 * k, v, cudaMemcpyDeviceToHost, c->stream));
  if (speed) CK(cudaMemcpyAsync(speed, st + 12 * k, k * sizeof(float), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return BOIDS_OK;
}

// The spatial query order (qperm) is a permutation of agent ids: after an upload
// with another id <-> space arrangement it no longer groups nearby queries
// (measured: C4 with Morton-renumbered ids 2.79 -> 3.60 ms/step until the next
// refresh), so boids_set_state has it rebuilt on the next step -- unless the
// upload keeps the arrangement (the usual case: the caller's copy of the last
// state, moved a little).  Test (k_order_check, on the device, reading the
// staged positions): 256 strided pairs of consecutive qperm entries; the order is
// kept if at least half of them are still within the search radius of each
// other.  Only a performance decision; its 8-byte result rides on set_state's
// own synchronisation.

BOIDS_API int boids_set_state(boids_ctx* c, const float* pos3, const float* fwd3, const float* up3,
                    const float* side3, const float* speed) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!pos3 || !fwd3 || !up3 || !speed) return fail(BOIDS_EINVAL, "pos3, fwd3, up3, speed required");
  DeviceGuard g(c->dev);
  int rc = ensure_stage(c);
  if (rc) return rc;
  const int64_t k = c->nloc;
  float* st = c->stage;
  const size_t v = (size_t)k * 3 * sizeof(float);
  CK(cudaMemcpyAsync(st, pos3, v, cudaMemcpyHostToDevice, c->stream));
  CK(cudaMemcpyAsync(st + 3 * k, fwd3, v, cudaMemcpyHostToDevice, c->stream));
  CK(cudaMemcpyAsync(st + 6 * k, up3, v, cudaMemcpyHostToDevice, c->stream));
  if (side3) CK(cudaMemcpyAsync(st + 9 * k, side3, v, cudaMemcpyHostToDevice, c->stream));
  CK(cudaMemcpyAsync(st + 12 * k, speed, k * sizeof(float), cudaMemcpyHostToDevice, c->stream));
  CK(launch_state_in(st, side3 != nullptr, k, c->local(), c->m, c->up4, c->side4, c->stream));
  c->launches++;
  if (c->spatial) {  // all n uploaded: own / halo / cleared again from the new positions
    CK(launch_spatial_init(c->local(), c->buf[c->cur ^ 1], c->m, c->n, c->own, c->sgrid, c->zb, c->world, c->rank,
                           c->sp_reach, c->kept, c->nkept, c->stream));
    c->kept_bound = c->n;
    c->last_nh = 0;
    c->launches++;
  }
  // The previous neighbour lists are KEPT: the warm bound they seed (the 7th
  // smallest current distance to 7-8 distinct existing agents) is an upper bound
  // on the 7th neighbour distance for ANY positions, so the next step stays exact;
  // a poor bound only costs time.  boids_get_neighbors still reports the lists of
  // the last step until the next step.
  int chk[2] = {0, 0};
  const bool check = c->since_sort >= 0 && c->qperm && k >= 64;
  if (check) {
    CK(launch_order_check(st, c->qperm, k, c->p.search_radius * c->p.search_radius, c->ocheck, c->stream));
    c->launches++;
    CK(cudaMemcpyAsync(chk, c->ocheck, sizeof(chk), cudaMemcpyDeviceToHost, c->stream));
  }
  CK(cudaStreamSynchronize(c->stream));
  if (c->since_sort >= 0 && !(check && chk[0] > 0 && 2 * chk[1] >= chk[0])) c->since_sort = -1;
  c->steering_valid = false;
  return BOIDS_OK;
}

BOIDS_API int boids_get_accel(boids_ctx* c, float* acc3) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!acc3) return fail(BOIDS_EINVAL, "acc3 is NULL");
  if (!c->acc4) return fail(BOIDS_EINVAL, "no acceleration state (steer_mode is not BOIDS_STEER_OPENSTEER)");
  DeviceGuard g(c->dev);
  // strided copy float4 -> packed float3 rows: the DMA engine converts the layout
  CK(cudaMemcpy2DAsync(acc3, 3 * sizeof(float), c->acc4, sizeof(float4), 3 * sizeof(float), (size_t)c->nloc,
                       cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return BOIDS_OK;
}

BOIDS_API int boids_set_accel(boids_ctx* c, const float* acc3) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!acc3) return fail(BOIDS_EINVAL, "acc3 is NULL");
  if (!c->acc4) return fail(BOIDS_EINVAL, "no acceleration state (steer_mode is not BOIDS_STEER_OPENSTEER)");
  DeviceGuard g(c->dev);
  CK(cudaMemcpy2DAsync(c->acc4, sizeof(float4), acc3, 3 * sizeof(float), 3 * sizeof(float), (size_t)c->nloc,
                       cudaMemcpyHostToDevice, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return BOIDS_OK;
}

BOIDS_API int boids_get_neighbors(boids_ctx* c, int32_t* idx7, int32_t* cnt) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  DeviceGuard g(c->dev);
  if (idx7) CK(cudaMemcpyAsync(idx7, c->nbr, c->nloc * 7 * sizeof(int32_t), cudaMemcpyDeviceToHost, c->stream));
  if (cnt) CK(cudaMemcpyAsync(cnt, c->cnt, c->nloc * sizeof(int32_t), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return BOIDS_OK;
}

BOIDS_API int boids_get_steering(boids_ctx* c, float* force3) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->steering_valid) return fail(BOIDS_EINVAL, "no recorded steering (set BOIDS_OPT_RECORD_STEERING before stepping)");
  if (!force3) return fail(BOIDS_EINVAL, "force3 is NULL");
  DeviceGuard g(c->dev);
  std::vector<float4> h((size_t)c->nloc);
  CK(cudaMemcpyAsync(h.data(), c->force4, c->nloc * sizeof(float4), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  to_aos(h, c->nloc, force3, false);
  return BOIDS_OK;
}

BOIDS_API int boids_sync(boids_ctx* c) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  DeviceGuard g(c->dev);
  CK(cudaStreamSynchronize(c->stream));
  CK(cudaGetLastError());
  return BOIDS_OK;
}

BOIDS_API int boids_info(boids_ctx* c, boids_info_t* o) {
  if (!c || !o) return fail(BOIDS_EINVAL, "NULL argument");
  o->n = c->n;
  o->lo = c->lo;
  o->hi = c->hi;
  o->slice = c->m;
  o->rank = c->rank;
  o->world = c->world;
  o->kernel = c->kernel;
  o->cluster = c->cluster_opt ? c->cluster_opt : fused_auto_cluster(c->ncand, c->nloc, c->sm_count);
  o->launches = c->launches;
  unsigned long long st[4] = {0, 0, 0, 0};
  CK(cudaMemcpyAsync(st, c->stats, sizeof(st), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  o->slow_groups = (int64_t)st[0];
  o->vote_groups = (int64_t)st[1];
  o->fallbacks = (int64_t)st[2];
  o->grid_pairs = (int64_t)st[3];
  o->step_index = c->step_index;
  o->last_path = c->last_path;
  o->reserved0 = 0;
  o->steps_sorted = c->steps_sorted;
  o->graph_launches = c->graph_launches;
  return BOIDS_OK;
}

BOIDS_API int boids_get_profile(boids_ctx* c, double* ms, int64_t* launches, int32_t reset) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  DeviceGuard g(c->dev);
  CK(cudaStreamSynchronize(c->stream));
  for (auto& r : c->recs) {
    float t = 0.f;
    CK(cudaEventElapsedTime(&t, r.a, r.b));
    c->prof_ms[r.cls] += t;
    c->prof_n[r.cls] += 1;
    c->pool.push_back(r.a);
    c->pool.push_back(r.b);
  }
  c->recs.clear();
  for (int k = 0; k < BOIDS_PROF_CLASSES; ++k) {
    if (ms) ms[k] = c->prof_ms[k];
    if (launches) launches[k] = c->prof_n[k];
    if (reset) {
      c->prof_ms[k] = 0;
      c->prof_n[k] = 0;
    }
  }
  return BOIDS_OK;
}

BOIDS_API int boids_get_phases(boids_ctx* c, uint64_t* out, int64_t count) {
  if (!c || !out) return fail(BOIDS_EINVAL, "NULL argument");
  if (!c->phase) return fail(BOIDS_EINVAL, "phases not enabled (BOIDS_OPT_PHASES)");
  DeviceGuard g(c->dev);
  CK(cudaMemcpyAsync(out, c->phase, count * sizeof(uint64_t), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return BOIDS_OK;
}

BOIDS_API int boids_bench_update(boids_ctx* c, float dt, int32_t reps, double* ms_per_launch) {
  if (!c || !ms_per_launch) return fail(BOIDS_EINVAL, "NULL argument");
  if (reps < 1) return fail(BOIDS_EINVAL, "reps must be >= 1");
  int rc = check_dt(dt);
  if (rc) return rc;
  DeviceGuard g(c->dev);
  const int64_t m = c->m;
  if (!c->ubench) CK(cudaMalloc((void**)&c->ubench, (size_t)5 * m * sizeof(float4)));
  StepArgs a = make_args(c, dt);
  float4* su = c->ubench + 2 * m;
  float4* ss = c->ubench + 3 * m;
  float4* sa = c->ubench + 4 * m;
  // the kernel updates the frame (and OpenSteer's smoothed acceleration) in place:
  // give it copies, so the handle's state is untouched
  CK(cudaMemcpyAsync(su, c->up4, m * sizeof(float4), cudaMemcpyDeviceToDevice, c->stream));
  CK(cudaMemcpyAsync(ss, c->side4, m * sizeof(float4), cudaMemcpyDeviceToDevice, c->stream));
  if (c->acc4) CK(cudaMemcpyAsync(sa, c->acc4, m * sizeof(float4), cudaMemcpyDeviceToDevice, c->stream));
  a.out = c->ubench;
  a.up4 = su;
  a.side4 = ss;
  a.acc4 = c->acc4 ? sa : nullptr;
  a.force4 = nullptr;
  cudaEvent_t e0 = get_event(c), e1 = get_event(c);
  double tot = 0.0;
  for (int32_t r = 0; r < reps; ++r) {
    CK(cudaEventRecord(e0, c->stream));
    CK(launch_update(a, c->stream));
    CK(cudaEventRecord(e1, c->stream));
    CK(cudaEventSynchronize(e1));
    float t = 0.f;
    CK(cudaEventElapsedTime(&t, e0, e1));
    tot += t;
    c->launches++;
  }
  c->pool.push_back(e0);
  c->pool.push_back(e1);
  *ms_per_launch = tot / reps;
  return BOIDS_OK;
}

BOIDS_API int boids_readback_begin(boids_ctx* c, float* host16) {
  if (!c || !host16) return fail(BOIDS_EINVAL, "NULL argument");
  DeviceGuard g(c->dev);
  if (!c->draw) {
    CK(cudaMalloc((void**)&c->draw, (size_t)(c->m > 0 ? c->m : 1) * 4 * sizeof(float4)));
    CK(cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&c->packed, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&c->landed, cudaEventDisableTiming));
  }
  if (c->rb_pending) CK(cudaEventSynchronize(c->landed));  // one in flight (the draw buffer is reused)
  // pack on the compute stream (ordered after the last step), copy on the copy stream
  CK(launch_pack_draw(c->local(), c->m, c->up4, c->side4, c->nloc, c->draw, c->stream));
  c->launches++;
  CK(cudaEventRecord(c->packed, c->stream));
  CK(cudaStreamWaitEvent(c->copy_stream, c->packed, 0));
  CK(cudaMemcpyAsync(host16, c->draw, c->nloc * 4 * sizeof(float4), cudaMemcpyDeviceToHost, c->copy_stream));
  CK(cudaEventRecord(c->landed, c->copy_stream));
  c->rb_pending = true;
  return BOIDS_OK;
}

BOIDS_API int boids_readback_wait(boids_ctx* c) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (!c->rb_pending) return BOIDS_OK;
  DeviceGuard g(c->dev);
  CK(cudaEventSynchronize(c->landed));
  c->rb_pending = false;
  return BOIDS_OK;
}

BOIDS_API int boids_get_think_state(boids_ctx* c, int64_t* step_index, float* fstore3) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  DeviceGuard g(c->dev);
  if (step_index) *step_index = c->step_index;
  if (fstore3) {
    std::vector<float4> h((size_t)c->nloc);
    CK(cudaMemcpyAsync(h.data(), c->fstore, c->nloc * sizeof(float4), cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    to_aos(h, c->nloc, fstore3, false);
  }
  return BOIDS_OK;
}

BOIDS_API int boids_set_think_state(boids_ctx* c, int64_t step_index, const float* fstore3) {
  if (!c) return fail(BOIDS_EINVAL, "NULL handle");
  if (step_index < 0) return fail(BOIDS_EINVAL, "step_index must be >= 0");
  DeviceGuard g(c->dev);
  c->step_index = step_index;
  if (fstore3) {
    std::vector<float4> h((size_t)c->nloc);
    for (int64_t i = 0; i < c->nloc; ++i)
      h[i] = make_float4(fstore3[3 * i], fstore3[3 * i + 1], fstore3[3 * i + 2], 0.f);
    CK(cudaMemcpyAsync(c->fstore, h.data(), c->nloc * sizeof(float4), cudaMemcpyHostToDevice, c->stream));
    CK(cudaStreamSynchronize(c->stream));
  }
  return BOIDS_OK;
}

BOIDS_API void boids_destroy(boids_ctx* c) { free_ctx(c); }

BOIDS_API const char* boids_last_error(void) { return g_err.c_str(); }

}  // extern "C"
