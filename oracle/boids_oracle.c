/*
 * boids_oracle.c -- plain, slow, single-threaded CPU oracle for one Boids step.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing in the product path (the package
 * paper_conf_ipps_breitbart09_b200/, its CUDA library, its Python binding)
 * may include, link, load or execute this file.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * use it.  It shares no code, header, table or constant generator with the
 * CUDA path; its parameter defaults are restated here from DESIGN.md Table C1.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:<line>"):
 *   - neighbour search: Listing 5.2 (sec 5.2.1) and Listing 6.3
 *     (sec 6.3.1), literally: scan every agent A in index order, keep
 *     up to 7 within the search radius, once 7 are held replace the farthest
 *     held one B when A is closer.  Readings Q2-Q6 of DESIGN.md: the test is
 *     d2 < r2 with r2 = fl(r*r); "closer" is the total order on (d2, index);
 *     self is excluded by index; the result is sorted ascending by (d2, idx).
 *   - steering: Listing 5.1 (flocking = weighted sum of normalised
 *     behaviours), Listing 5.3 (separation),
 *     Listing 5.4 (cohesion), Listing 5.5 (alignment, mis-titled
 *     cohesion() in the text).
 *   - modification substage (sec 5.3, sec 6.2.3):
 *     clamp force, integrate velocity/position, regenerate local space,
 *     spherical wrap "at the diametric opposite point" (sec 5.1).
 *     The arithmetic is DESIGN.md reading Q10 (the paper gives no formula).
 *   - synchronous (Jacobi) update: every output of step t is computed from
 *     the state of step t only (two substages; two kernels).
 *   - initial state: DESIGN.md Appendix B (the paper is silent).
 *   - steer_mode 1 (the thesis's device code "is based on
 *     the CPU version of OpenSteer"): OpenSteer 0.8.2's own flocking
 *     instead of Listings 5.3-5.5 -- per-behaviour neighbourhood filters
 *     (inBoidNeighborhood), averaged behaviours, adjustRawSteeringForce and
 *     acceleration smoothing (blendIntoAccumulator) in the modification.
 *     Restated from OpenSteer [ext], not from the paper: DESIGN.md Q20-Q24.
 *
 * Arithmetic (DESIGN.md Appendix A): IEEE binary32, round to nearest even,
 * every operation individually rounded, no fused multiply-add, evaluated in
 * the written order.  Build with: gcc -O2 -ffp-contract=off -fno-fast-math.
 *
 * Pins (tests/test_oracle_*.py): brute-force sort on tiny flocks, tie and
 * boundary cases, invariants, closed-form steering/modification cases, the
 * wrap example, scipy cKDTree on tie-free inputs, the local-space handedness
 * (closed forms, the triple-product identity up' = n(u - (u.f')f'), det sign).  Parity unpinned: that the
 * DESIGN.md Table C1 constants and the Q10 modification arithmetic are what
 * the thesis actually ran (the paper prints neither).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_K 7 /* "We only consider the 7 nearest neighbors" P:364 */

typedef struct oracle_params {
  float search_radius;  /* Table C1: 9.0   [ext, reading Q1] */
  float w_separation;   /* 12 */
  float w_alignment;    /* 8  */
  float w_cohesion;     /* 8  */
  float max_force;      /* 27 */
  float max_speed;      /* 9  */
  float mass;           /* 1  */
  float world_radius;   /* 50 */
  float init_radius;    /* 20 */
  float init_speed_frac;/* 0.3 */
  int32_t max_neighbors;/* 7 */
  int32_t search_mode;  /* ignored by the oracle: every mode has one answer */
  int32_t init_mode;    /* 0 = ball of init_radius, 1 = ball of world_radius */
  int32_t think_every;  /* think frequency k; 1 = every agent thinks every step */
  int32_t steer_mode;   /* 0 = the thesis's Listings 5.1-5.5 + reading Q10 (default);
                           1 = OpenSteer 0.8.2 flocking [ext] (readings Q20-Q24) */
} oracle_params;

void oracle_default_params(oracle_params* p) {
  p->search_radius = 9.0f;
  p->w_separation = 12.0f;
  p->w_alignment = 8.0f;
  p->w_cohesion = 8.0f;
  p->max_force = 27.0f;
  p->max_speed = 9.0f;
  p->mass = 1.0f;
  p->world_radius = 50.0f;
  p->init_radius = 20.0f;
  p->init_speed_frac = 0.3f;
  p->max_neighbors = ORACLE_K;
  p->search_mode = 0;
  p->init_mode = 0;
  p->think_every = 1;
  p->steer_mode = 0;
}

/* ---------------- Appendix A vector helpers (each op rounded) ------------ */
typedef struct { float x, y, z; } v3;

static v3 v3_make(float x, float y, float z) { v3 r; r.x = x; r.y = y; r.z = z; return r; }
static v3 v3_load(const float* a, int64_t i) { return v3_make(a[3 * i], a[3 * i + 1], a[3 * i + 2]); }
static void v3_store(float* a, int64_t i, v3 v) { a[3 * i] = v.x; a[3 * i + 1] = v.y; a[3 * i + 2] = v.z; }
static v3 v3_add(v3 a, v3 b) { return v3_make(a.x + b.x, a.y + b.y, a.z + b.z); }
static v3 v3_sub(v3 a, v3 b) { return v3_make(a.x - b.x, a.y - b.y, a.z - b.z); }
static v3 v3_scale(v3 a, float s) { return v3_make(a.x * s, a.y * s, a.z * s); } /* a (x) s */
static v3 v3_divs(v3 a, float s) { return v3_make(a.x / s, a.y / s, a.z / s); }  /* a (/) s */
/* dot(a,b) = ((a.x*b.x) + (a.y*b.y)) + (a.z*b.z) */
static float v3_dot(v3 a, v3 b) {
  float xx = a.x * b.x;
  float yy = a.y * b.y;
  float zz = a.z * b.z;
  float s = xx + yy;
  return s + zz;
}
static float v3_len(v3 a) { return sqrtf(v3_dot(a, a)); }
/* normalize: m = len(a); m > 0 ? a (/) m : a   (so normalize(0) = 0, Q9) */
static v3 v3_normalize(v3 a) {
  float m = v3_len(a);
  return m > 0.0f ? v3_divs(a, m) : a;
}
static v3 v3_cross(v3 a, v3 b) {
  return v3_make(a.y * b.z - a.z * b.y, a.z * b.x - a.x * b.z, a.x * b.y - a.y * b.x);
}
/* truncateLength: l2 = dot(a,a); l2 <= L*L ? a : a (x) (L / sqrt(l2)) */
static v3 v3_trunc(v3 a, float L) {
  float l2 = v3_dot(a, a);
  float LL = L * L;
  if (l2 <= LL) return a;
  float s = L / sqrtf(l2);
  return v3_scale(a, s);
}

/* ---------------- Appendix B initial state ------------------------------- */
#define SM64_GAMMA 0x9E3779B97F4A7C15ull
static uint64_t sm64_mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
/* splitmix64(x): the first output of a SplitMix64 generator seeded with x. */
static uint64_t sm64(uint64_t x) { return sm64_mix(x + SM64_GAMMA); }
static float draw_coord(uint64_t* s) {
  *s += SM64_GAMMA;
  uint64_t out = sm64_mix(*s);
  float u = (float)(out >> 40) * 5.9604644775390625e-08f; /* 2^-24, exact */
  float two_u = u * 2.0f;
  return two_u - 1.0f;
}
/* OpenSteer-style rejection in the cube [-1,1)^3 until dot < 1. */
static v3 draw_ball(uint64_t* s) {
  for (;;) {
    float x = draw_coord(s);
    float y = draw_coord(s);
    float z = draw_coord(s);
    v3 v = v3_make(x, y, z);
    if (v3_dot(v, v) < 1.0f) return v;
  }
}

void oracle_init(int64_t n, const oracle_params* p, uint64_t seed, float* pos3, float* fwd3,
                 float* up3, float* side3, float* speed) {
  float R = p->init_mode == 1 ? p->world_radius : p->init_radius;
  float sp = p->init_speed_frac * p->max_speed;
  for (int64_t i = 0; i < n; ++i) {
    uint64_t s = sm64(seed ^ sm64((uint64_t)i));
    v3 b = draw_ball(&s);
    v3 pos = v3_scale(b, R);
    v3 f = v3_normalize(draw_ball(&s));
    v3 up0 = v3_make(0.0f, 1.0f, 0.0f);
    v3 side = v3_normalize(v3_cross(f, up0));
    v3 up = v3_cross(side, f);
    v3_store(pos3, i, pos);
    v3_store(fwd3, i, f);
    v3_store(up3, i, up);
    v3_store(side3, i, side);
    speed[i] = sp;
  }
}

/* ---------------- Listing 5.2 / 6.3 neighbour search ---------------------- */
/* key order: (d2, index) lexicographic -- reading Q4 */
static int key_less(float da, int32_t ia, float db, int32_t ib) {
  return da < db || (da == db && ia < ib);
}

/* d = pi (-) pj ; d2 = ((dx*dx) + (dy*dy)) + (dz*dz)   (reading Q3, no FMA) */
static float dist2(v3 pi, v3 pj) {
  v3 d = v3_sub(pi, pj);
  return v3_dot(d, d);
}

/* One agent i against all n agents, literally as Listing 5.2. */
void oracle_search_one(int64_t n, const float* pos3, float radius, int64_t i, int32_t* idx7,
                       int32_t* cnt_out) {
  float r2 = radius * radius;
  float nd[ORACLE_K];
  int32_t ni[ORACLE_K];
  int cnt = 0;
  v3 me = v3_load(pos3, i);
  for (int64_t j = 0; j < n; ++j) {
    v3 a = v3_load(pos3, j);
    float d2 = dist2(me, a);
    if (d2 < r2 && j != i) {             /* Listing 6.3 line 7 */
      if (cnt < ORACLE_K) {              /* "neighbors found < 7": add A */
        nd[cnt] = d2;
        ni[cnt] = (int32_t)j;
        ++cnt;
      } else {                           /* B := neighbour with the biggest distance */
        int b = 0;
        for (int k = 1; k < ORACLE_K; ++k)
          if (key_less(nd[b], ni[b], nd[k], ni[k])) b = k;
        if (key_less(d2, (int32_t)j, nd[b], ni[b])) { /* distance(Me,B) > distance(Me,A) */
          nd[b] = d2;
          ni[b] = (int32_t)j;
        }
      }
    }
  }
  /* Reading Q5: report ascending by (d2, idx), -1 padded. Insertion sort. */
  for (int a = 1; a < cnt; ++a) {
    float kd = nd[a];
    int32_t ki = ni[a];
    int b = a - 1;
    while (b >= 0 && key_less(kd, ki, nd[b], ni[b])) {
      nd[b + 1] = nd[b];
      ni[b + 1] = ni[b];
      --b;
    }
    nd[b + 1] = kd;
    ni[b + 1] = ki;
  }
  for (int k = 0; k < ORACLE_K; ++k) idx7[k] = k < cnt ? ni[k] : -1;
  *cnt_out = cnt;
}

void oracle_search(int64_t n, const float* pos3, float radius, int32_t* idx7, int32_t* cnt) {
  for (int64_t i = 0; i < n; ++i) oracle_search_one(n, pos3, radius, i, idx7 + 7 * i, cnt + i);
}

static void oracle_steer_one_os(const float* pos3, const float* fwd3, int64_t i, const int32_t* idx7,
                                int32_t cnt, const oracle_params* p, float* force3);

/* ---------------- Listings 5.1, 5.3, 5.4, 5.5 steering -------------------- */
void oracle_steer_one(const float* pos3, const float* fwd3, int64_t i, const int32_t* idx7,
                      int32_t cnt, const oracle_params* p, float* force3) {
  if (p->steer_mode == 1) {
    oracle_steer_one_os(pos3, fwd3, i, idx7, cnt, p, force3);
    return;
  }
  v3 me = v3_load(pos3, i);
  v3 fme = v3_load(fwd3, i);
  v3 sep = v3_make(0.0f, 0.0f, 0.0f);
  v3 coh = v3_make(0.0f, 0.0f, 0.0f);
  v3 ali = v3_make(0.0f, 0.0f, 0.0f);
  for (int k = 0; k < cnt; ++k) {               /* neighbours in key order (Q8) */
    int64_t j = idx7[k];
    v3 o = v3_sub(v3_load(pos3, j), me);        /* A.position - me.position */
    float L = v3_len(o);
    if (L > 0.0f) {                             /* division-by-zero guard (Q6) */
      v3 nrm = v3_divs(o, L);                   /* distance.normalize() */
      v3 t = v3_divs(nrm, L);                   /* ... / distance.length() */
      sep = v3_sub(sep, t);                     /* steering -= ... (Listing 5.3) */
    }
    coh = v3_add(coh, o);                       /* Listing 5.4 line 8 */
    ali = v3_add(ali, v3_load(fwd3, j));        /* Listing 5.5 line 7 */
  }
  ali = v3_sub(ali, v3_scale(fme, (float)cnt)); /* Listing 5.5 line 10 */
  /* Listing 5.1: weightA*normalize(separation) + weightB*normalize(alignment)
   *              + weightC*normalize(cohesion), summed left to right. */
  v3 sw = v3_scale(v3_normalize(sep), p->w_separation);
  v3 aw = v3_scale(v3_normalize(ali), p->w_alignment);
  v3 cw = v3_scale(v3_normalize(coh), p->w_cohesion);
  v3 F = v3_add(v3_add(sw, aw), cw);
  v3_store(force3, 0, F);
}

/* ---------------- steer_mode 1: OpenSteer 0.8.2 flocking [ext] -------------
 * Boid::steerToFlock with SteerLibrary's steerForSeparation / Alignment /
 * Cohesion over the same <= 7 neighbours (the thesis's list), each behaviour
 * keeping only the neighbours inBoidNeighborhood(minDistance = 3 * radius
 * (radius 0.5), maxDistance, cosMaxAngle) accepts (Q20-Q22). */
#define OS_MIN_DIST 1.5f   /* 3 * SimpleVehicle radius 0.5 */
#define OS_SEP_R 5.0f
#define OS_SEP_COS (-0.707f)
#define OS_ALI_R 7.5f
#define OS_ALI_COS 0.7f
#define OS_COH_R 9.0f
#define OS_COH_COS (-0.15f)

/* inBoidNeighborhood: inside minDistance -> yes; beyond maxDistance -> no;
 * else forward . (offset / |offset|) > cosMaxAngle. */
static int os_in_hood(v3 o, float d2, v3 fme, float min_d, float max_d, float cos_max) {
  if (d2 < min_d * min_d) return 1;
  if (d2 > max_d * max_d) return 0;
  v3 unit = v3_divs(o, sqrtf(d2));
  return v3_dot(fme, unit) > cos_max;
}

static void oracle_steer_one_os(const float* pos3, const float* fwd3, int64_t i, const int32_t* idx7,
                                int32_t cnt, const oracle_params* p, float* force3) {
  v3 me = v3_load(pos3, i);
  v3 fme = v3_load(fwd3, i);
  v3 sep = v3_make(0.0f, 0.0f, 0.0f), ali = sep, coh = sep;
  int ns = 0, na = 0, nc = 0;
  for (int k = 0; k < cnt; ++k) {               /* neighbours in key order (Q8) */
    int64_t j = idx7[k];
    v3 pj = v3_load(pos3, j);
    v3 o = v3_sub(pj, me);                      /* offset = other.position - position */
    float d2 = v3_dot(o, o);                    /* offset.lengthSquared() */
    if (os_in_hood(o, d2, fme, OS_MIN_DIST, OS_SEP_R, OS_SEP_COS) && d2 > 0.0f) {
      sep = v3_add(sep, v3_divs(o, -d2));       /* steering += offset / -distanceSquared */
      ++ns;
    }
    if (os_in_hood(o, d2, fme, OS_MIN_DIST, OS_ALI_R, OS_ALI_COS)) {
      ali = v3_add(ali, v3_load(fwd3, j));      /* steering += other.forward() */
      ++na;
    }
    if (os_in_hood(o, d2, fme, OS_MIN_DIST, OS_COH_R, OS_COH_COS)) {
      coh = v3_add(coh, pj);                    /* steering += other.position() */
      ++nc;
    }
  }
  if (ns > 0) sep = v3_normalize(v3_divs(sep, (float)ns));
  if (na > 0) ali = v3_normalize(v3_sub(v3_divs(ali, (float)na), fme));
  if (nc > 0) coh = v3_normalize(v3_sub(v3_divs(coh, (float)nc), me));
  v3 sw = v3_scale(sep, p->w_separation);
  v3 aw = v3_scale(ali, p->w_alignment);
  v3 cw = v3_scale(coh, p->w_cohesion);
  v3 F = v3_add(v3_add(sw, aw), cw);
  v3_store(force3, 0, F);
}

/* x^20 as ((x^2)^2)^2)^2 * x^4, each product rounded (reading Q23 for pow(range, 20)). */
static float os_pow20(float x) {
  float x2 = x * x, x4 = x2 * x2, x8 = x4 * x4, x16 = x8 * x8;
  return x16 * x4;
}

/* SimpleVehicle::adjustRawSteeringForce (Q23): below 0.2 maxSpeed the force is
 * kept within a cone around forward (vecLimitDeviationAngleUtility, inside). */
static v3 os_adjust_raw(v3 F, float speed, v3 fwd, const oracle_params* p) {
  float max_adj = 0.2f * p->max_speed;
  if (speed > max_adj || (F.x == 0.0f && F.y == 0.0f && F.z == 0.0f)) return F;
  float range = speed / max_adj;
  float cosine = 1.0f + (-1.0f - 1.0f) * os_pow20(range); /* interpolate(pow(range,20), 1, -1) */
  float L = v3_len(F);
  if (L == 0.0f) return F;
  v3 dir = v3_divs(F, L);
  if (v3_dot(dir, fwd) >= cosine) return F;
  v3 perp = v3_sub(F, v3_scale(fwd, v3_dot(F, fwd)));  /* source.perpendicularComponent(basis) */
  v3 uperp = v3_normalize(perp);
  float perp_dist = sqrtf(1.0f - cosine * cosine);
  v3 c0 = v3_scale(fwd, cosine);
  v3 c1 = v3_scale(uperp, perp_dist);
  return v3_scale(v3_add(c0, c1), L);
}

/* ---------------- modification substage (reading Q10-Q13) ----------------- */
/* acc3: steer_mode 1 only -- the agent's smoothed acceleration, read and
 * updated in place (OpenSteer's _smoothedAcceleration; only the agent itself
 * uses it, so the in-place update keeps the step synchronous). */
void oracle_modify_one(const float* p_in, const float* f_in, const float* u_in, const float* s_in,
                       float speed, const float* F_in, const oracle_params* p, float dt,
                       float* p_out, float* f_out, float* u_out, float* s_out, float* speed_out,
                       float* acc3) {
  v3 pos = v3_make(p_in[0], p_in[1], p_in[2]);
  v3 f = v3_make(f_in[0], f_in[1], f_in[2]);
  v3 u = v3_make(u_in[0], u_in[1], u_in[2]);
  v3 s = v3_make(s_in[0], s_in[1], s_in[2]);
  v3 F = v3_make(F_in[0], F_in[1], F_in[2]);
  if (p->steer_mode == 1) F = os_adjust_raw(F, speed, f, p);  /* Q23 */
  v3 Fc = v3_trunc(F, p->max_force);           /* clamp force */
  v3 a = v3_divs(Fc, p->mass);                 /* a = F / m  (length = acceleration) */
  if (p->steer_mode == 1) {                    /* blendIntoAccumulator (Q24) */
    v3 sm = v3_load(acc3, 0);
    if (dt > 0.0f) {
      float rate = 9.0f * dt;                  /* clip(9 dt, 0.15, 0.4) */
      rate = rate < 0.15f ? 0.15f : (rate > 0.4f ? 0.4f : rate);
      sm = v3_add(sm, v3_scale(v3_sub(a, sm), rate));  /* interpolate(rate, smoothed, new) */
      v3_store(acc3, 0, sm);
    }
    a = sm;
  }
  v3 v = v3_scale(f, speed);                   /* velocity = forward * speed */
  v3 v1 = v3_add(v, v3_scale(a, dt));          /* integrate velocity */
  v3 v2 = v3_trunc(v1, p->max_speed);          /* clamp speed */
  float sp = v3_len(v2);
  v3 p1 = v3_add(pos, v3_scale(v2, dt));       /* integrate position */
  if (sp > 0.0f) {                             /* regenerate local space */
    f = v3_divs(v2, sp);
    s = v3_normalize(v3_cross(f, u));
    u = v3_cross(s, f);
  }
  float L = v3_len(p1);                        /* spherical wrap (Q12) */
  if (L > p->world_radius) {
    v3 t = v3_scale(v3_scale(v3_divs(p1, L), p->world_radius), -2.0f);
    p1 = v3_add(p1, t);
  }
  p_out[0] = p1.x; p_out[1] = p1.y; p_out[2] = p1.z;
  f_out[0] = f.x; f_out[1] = f.y; f_out[2] = f.z;
  u_out[0] = u.x; u_out[1] = u.y; u_out[2] = u.z;
  s_out[0] = s.x; s_out[1] = s.y; s_out[2] = s.z;
  *speed_out = sp;
}

/* One agent of one synchronous step: search + steer + modify, from state S_t. */
static void step_agent(int64_t n, const oracle_params* p, float dt, const float* pos3,
                       const float* fwd3, const float* up3, const float* side3,
                       const float* speed, int64_t i, float* pos_o, float* fwd_o, float* up_o,
                       float* side_o, float* speed_o, int32_t* idx7, int32_t* cnt,
                       float* force3, float* acc3) {
  oracle_search_one(n, pos3, p->search_radius, i, idx7, cnt);
  oracle_steer_one(pos3, fwd3, i, idx7, *cnt, p, force3);
  oracle_modify_one(pos3 + 3 * i, fwd3 + 3 * i, up3 + 3 * i, side3 + 3 * i, speed[i], force3, p,
                    dt, pos_o, fwd_o, up_o, side_o, speed_o, acc3);
}

/* Whole step S_t -> S_{t+1}; outputs must not alias inputs (Jacobi update). */
/* acc3 (n,3): steer_mode 1 smoothed accelerations, updated in place (ignored otherwise). */
void oracle_step(int64_t n, const oracle_params* p, float dt, const float* pos3,
                 const float* fwd3, const float* up3, const float* side3, const float* speed,
                 float* pos_o, float* fwd_o, float* up_o, float* side_o, float* speed_o,
                 int32_t* idx7, int32_t* cnt, float* force3, float* acc3) {
  for (int64_t i = 0; i < n; ++i)
    step_agent(n, p, dt, pos3, fwd3, up3, side3, speed, i, pos_o + 3 * i, fwd_o + 3 * i,
               up_o + 3 * i, side_o + 3 * i, speed_o + i, idx7 + 7 * i, cnt + i, force3 + 3 * i,
               acc3 + 3 * i);
}

/* Sampled step: only the m agents listed in `agents` (outputs indexed 0..m-1). */
void oracle_step_sample(int64_t n, const oracle_params* p, float dt, const float* pos3,
                        const float* fwd3, const float* up3, const float* side3,
                        const float* speed, int64_t m, const int64_t* agents, float* pos_o,
                        float* fwd_o, float* up_o, float* side_o, float* speed_o,
                        int32_t* idx7, int32_t* cnt, float* force3, float* acc3) {
  for (int64_t k = 0; k < m; ++k)  /* acc3 (m,3): the sampled agents' accelerations, in/out */
    step_agent(n, p, dt, pos3, fwd3, up3, side3, speed, agents[k], pos_o + 3 * k, fwd_o + 3 * k,
               up_o + 3 * k, side_o + 3 * k, speed_o + k, idx7 + 7 * k, cnt + k, force3 + 3 * k,
               acc3 + 3 * k);
}

/* One synchronous step with think frequency k = p->think_every (sec 5.3:
 * "the simulation substage of a specific agent is executed every ten simulation
 * time steps.  In one simulation time step only 1/10th of the agents execute the
 * simulation substage").  Readings (Q15): agent i thinks at step t iff
 * (i + t) mod k == 0; a thinking agent searches + steers and stores its steering
 * vector in fstore; a non-thinking agent keeps its neighbour list and uses its
 * stored vector (zero before its first think); every agent runs the
 * modification substage.  idx7/cnt/fstore are in/out; force3 = F used. */
void oracle_step_think(int64_t n, const oracle_params* p, float dt, int64_t t, const float* pos3,
                       const float* fwd3, const float* up3, const float* side3, const float* speed,
                       float* pos_o, float* fwd_o, float* up_o, float* side_o, float* speed_o,
                       int32_t* idx7, int32_t* cnt, float* fstore3, float* force3, float* acc3) {
  int64_t k = p->think_every < 1 ? 1 : p->think_every;
  for (int64_t i = 0; i < n; ++i) {
    if ((i + t) % k == 0) {
      oracle_search_one(n, pos3, p->search_radius, i, idx7 + 7 * i, cnt + i);
      oracle_steer_one(pos3, fwd3, i, idx7 + 7 * i, cnt[i], p, fstore3 + 3 * i);
    }
    force3[3 * i] = fstore3[3 * i];
    force3[3 * i + 1] = fstore3[3 * i + 1];
    force3[3 * i + 2] = fstore3[3 * i + 2];
    oracle_modify_one(pos3 + 3 * i, fwd3 + 3 * i, up3 + 3 * i, side3 + 3 * i, speed[i], force3 + 3 * i, p,
                      dt, pos_o + 3 * i, fwd_o + 3 * i, up_o + 3 * i, side_o + 3 * i, speed_o + i,
                      acc3 + 3 * i);
  }
}

/* oracle_step_think evaluated only for the m agents listed in `agents` (each
 * thinker searched against all n): the same per-agent rule (reading
 * Q15), for checking large flocks on a sample.  fstore3/force3/acc3/idx7/cnt
 * and the outputs are per sampled agent (row s belongs to agents[s]). */
void oracle_step_think_sample(int64_t n, const oracle_params* p, float dt, int64_t t, const float* pos3,
                              const float* fwd3, const float* up3, const float* side3, const float* speed,
                              int64_t m, const int64_t* agents, float* pos_o, float* fwd_o, float* up_o,
                              float* side_o, float* speed_o, int32_t* idx7, int32_t* cnt, float* fstore3,
                              float* force3, float* acc3) {
  int64_t k = p->think_every < 1 ? 1 : p->think_every;
  for (int64_t s = 0; s < m; ++s) {
    int64_t i = agents[s];
    if ((i + t) % k == 0) {
      oracle_search_one(n, pos3, p->search_radius, i, idx7 + 7 * s, cnt + s);
      oracle_steer_one(pos3, fwd3, i, idx7 + 7 * s, cnt[s], p, fstore3 + 3 * s);
    }
    force3[3 * s] = fstore3[3 * s];
    force3[3 * s + 1] = fstore3[3 * s + 1];
    force3[3 * s + 2] = fstore3[3 * s + 2];
    oracle_modify_one(pos3 + 3 * i, fwd3 + 3 * i, up3 + 3 * i, side3 + 3 * i, speed[i], force3 + 3 * s, p,
                      dt, pos_o + 3 * s, fwd_o + 3 * s, up_o + 3 * s, side_o + 3 * s, speed_o + s,
                      acc3 + 3 * s);
  }
}

/* Many synchronous steps (S_t -> S_{t+steps}); state arrays updated in place. */
int oracle_run(int64_t n, const oracle_params* p, float dt, int32_t steps, float* pos3,
               float* fwd3, float* up3, float* side3, float* speed, float* acc3) {
  size_t v = (size_t)n * 3 * sizeof(float);
  float* buf = (float*)malloc(4 * v + (size_t)n * sizeof(float) + (size_t)n * 7 * sizeof(int32_t) +
                              (size_t)n * sizeof(int32_t) + v);
  if (!buf) return -4;
  float* po = buf;
  float* fo = po + 3 * n;
  float* uo = fo + 3 * n;
  float* so = uo + 3 * n;
  float* spo = so + 3 * n;
  int32_t* idx = (int32_t*)(spo + n);
  int32_t* cnt = idx + 7 * n;
  float* F = (float*)(cnt + n);
  for (int32_t t = 0; t < steps; ++t) {
    oracle_step(n, p, dt, pos3, fwd3, up3, side3, speed, po, fo, uo, so, spo, idx, cnt, F, acc3);
    memcpy(pos3, po, v);
    memcpy(fwd3, fo, v);
    memcpy(up3, uo, v);
    memcpy(side3, so, v);
    memcpy(speed, spo, (size_t)n * sizeof(float));
  }
  free(buf);
  return 0;
}
