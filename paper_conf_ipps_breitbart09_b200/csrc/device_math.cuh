// device_math.cuh -- fp32 vector helpers with the DESIGN.md Appendix A contract:
// every operation individually rounded to nearest even (explicit __f*_rn
// intrinsics, which nvcc never contracts into FMA), evaluated in the written
// order.  The library is also compiled with --fmad=false as a backstop.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace boids {

struct V3 {
  float x, y, z;
};

__device__ __forceinline__ V3 v3(float x, float y, float z) { return V3{x, y, z}; }
__device__ __forceinline__ V3 v3(float4 a) { return V3{a.x, a.y, a.z}; }
__device__ __forceinline__ V3 add(V3 a, V3 b) {
  return v3(__fadd_rn(a.x, b.x), __fadd_rn(a.y, b.y), __fadd_rn(a.z, b.z));
}
__device__ __forceinline__ V3 sub(V3 a, V3 b) {
  return v3(__fsub_rn(a.x, b.x), __fsub_rn(a.y, b.y), __fsub_rn(a.z, b.z));
}
__device__ __forceinline__ V3 scale(V3 a, float s) {
  return v3(__fmul_rn(a.x, s), __fmul_rn(a.y, s), __fmul_rn(a.z, s));
}
__device__ __forceinline__ V3 divs(V3 a, float s) {
  return v3(__fdiv_rn(a.x, s), __fdiv_rn(a.y, s), __fdiv_rn(a.z, s));
}
// dot(a,b) = ((a.x*b.x) + (a.y*b.y)) + (a.z*b.z)
__device__ __forceinline__ float dot(V3 a, V3 b) {
  float xx = __fmul_rn(a.x, b.x);
  float yy = __fmul_rn(a.y, b.y);
  float zz = __fmul_rn(a.z, b.z);
  return __fadd_rn(__fadd_rn(xx, yy), zz);
}
__device__ __forceinline__ float len(V3 a) { return __fsqrt_rn(dot(a, a)); }
__device__ __forceinline__ V3 normalize(V3 a) {
  float m = len(a);
  return m > 0.0f ? divs(a, m) : a;
}
__device__ __forceinline__ V3 cross(V3 a, V3 b) {
  return v3(__fsub_rn(__fmul_rn(a.y, b.z), __fmul_rn(a.z, b.y)),
            __fsub_rn(__fmul_rn(a.z, b.x), __fmul_rn(a.x, b.z)),
            __fsub_rn(__fmul_rn(a.x, b.y), __fmul_rn(a.y, b.x)));
}
__device__ __forceinline__ V3 trunc_len(V3 a, float L) {
  float l2 = dot(a, a);
  float LL = __fmul_rn(L, L);
  if (l2 <= LL) return a;
  float s = __fdiv_rn(L, __fsqrt_rn(l2));
  return scale(a, s);
}

// Search distance: d = pi - pj; d2 = ((dx*dx) + (dy*dy)) + (dz*dz), no FMA (reading Q3).
__device__ __forceinline__ float dist2(float px, float py, float pz, float4 c) {
  float dx = __fsub_rn(px, c.x);
  float dy = __fsub_rn(py, c.y);
  float dz = __fsub_rn(pz, c.z);
  return __fadd_rn(__fadd_rn(__fmul_rn(dx, dx), __fmul_rn(dy, dy)), __fmul_rn(dz, dz));
}

// ---- (d2, index) keys: the total order of reading Q4 as one unsigned 64-bit
// integer.  d2 >= 0, so its IEEE bit pattern orders like the value.
typedef unsigned long long key_t;
constexpr key_t KEY_EMPTY = 0x7F800000FFFFFFFFull;  // (+inf, 0xFFFFFFFF): after every real key

__device__ __forceinline__ key_t make_key(float d2, int j) {
  return ((key_t)__float_as_uint(d2) << 32) | (unsigned)j;
}
__device__ __forceinline__ float key_d2(key_t k) { return __uint_as_float((unsigned)(k >> 32)); }
__device__ __forceinline__ int key_idx(key_t k) { return (int)(unsigned)(k & 0xFFFFFFFFull); }

// Insert k into the ascending 7-list (keeps the 7 smallest).  Branch-free on
// statically indexed registers: new[s] = k < old[s-1] ? old[s-1] : min(k, old[s]).
__device__ __forceinline__ void insert7(key_t (&L)[7], key_t k) {
#pragma unroll
  for (int s = 6; s >= 1; --s) {
    key_t a = L[s - 1];
    key_t b = L[s] < k ? L[s] : k;
    L[s] = k < a ? a : b;
  }
  L[0] = L[0] < k ? L[0] : k;
}

__device__ __forceinline__ void cex(key_t& a, key_t& b) {
  key_t lo = a < b ? a : b;
  key_t hi = a < b ? b : a;
  a = lo;
  b = hi;
}

// A := the 7 smallest keys of A u B, ascending (A, B ascending 7-lists).
// Half-cleaner min(A[s], B[6-s]) keeps the 7 smallest as a bitonic sequence;
// a 0 sentinel in front keeps it bitonic at length 8; an 8-wide bitonic merge
// network sorts it and the sentinel (the minimum) is dropped.
__device__ __forceinline__ void merge7(key_t (&A)[7], const key_t (&B)[7]) {
  key_t S[8];
  S[0] = 0ull;
#pragma unroll
  for (int s = 0; s < 7; ++s) S[s + 1] = A[s] < B[6 - s] ? A[s] : B[6 - s];
#pragma unroll
  for (int i = 0; i < 4; ++i) cex(S[i], S[i + 4]);
  cex(S[0], S[2]); cex(S[1], S[3]); cex(S[4], S[6]); cex(S[5], S[7]);
  cex(S[0], S[1]); cex(S[2], S[3]); cex(S[4], S[5]); cex(S[6], S[7]);
#pragma unroll
  for (int s = 0; s < 7; ++s) A[s] = S[s + 1];
}

// A := the 8 smallest keys of A u B, ascending (half-cleaner + 8-wide bitonic merge).
__device__ __forceinline__ void merge8(key_t (&A)[8], const key_t (&B)[8]) {
  key_t S[8];
#pragma unroll
  for (int s = 0; s < 8; ++s) S[s] = A[s] < B[7 - s] ? A[s] : B[7 - s];
#pragma unroll
  for (int i = 0; i < 4; ++i) cex(S[i], S[i + 4]);
  cex(S[0], S[2]); cex(S[1], S[3]); cex(S[4], S[6]); cex(S[5], S[7]);
  cex(S[0], S[1]); cex(S[2], S[3]); cex(S[4], S[5]); cex(S[6], S[7]);
#pragma unroll
  for (int s = 0; s < 8; ++s) A[s] = S[s];
}
__device__ __forceinline__ void insert8(key_t (&L)[8], key_t k) {
#pragma unroll
  for (int s = 7; s >= 1; --s) {
    const key_t x = L[s - 1];
    const key_t y = L[s] < k ? L[s] : k;
    L[s] = k < x ? x : y;
  }
  L[0] = L[0] < k ? L[0] : k;
}

// ---- Appendix B: SplitMix64 streams --------------------------------------
constexpr uint64_t SM64_GAMMA = 0x9E3779B97F4A7C15ull;
__host__ __device__ __forceinline__ uint64_t sm64_mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__host__ __device__ __forceinline__ uint64_t sm64(uint64_t x) { return sm64_mix(x + SM64_GAMMA); }

}  // namespace boids
