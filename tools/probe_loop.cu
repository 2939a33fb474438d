// Probe of the fused kernel's hot loop in isolation (development aid, not part of libboids):
// Q queries/thread, candidates broadcast from a shared tile, per-query inclusive
// limits, FMNMX tree + warp vote per U candidates.  PACKED: subtract + square in
// FADD2/FMUL2 on query pairs (scalar FADD sums -- never fused), else scalar.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 --fmad=false tools/probe_loop.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int PACKED, int Q, int U>
__global__ void __launch_bounds__(128) loop(const float4* __restrict__ qpos, const float4* __restrict__ cand,
                                            int ncand, float lim0, unsigned* out) {
  __shared__ float4 tile[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) tile[i] = cand[i];
  __syncthreads();
  float px[Q], py[Q], pz[Q], lim[Q];
  for (int q = 0; q < Q; ++q) {
    float4 p = qpos[(blockIdx.x * blockDim.x + threadIdx.x) * Q + q];
    px[q] = p.x; py[q] = p.y; pz[q] = p.z; lim[q] = lim0 * (1.f + 0.01f * q);
  }
  float limc = lim[0];
  for (int q = 1; q < Q; ++q) limc = fmaxf(limc, lim[q]);
  unsigned hits = 0;
  for (int rep = 0; rep < ncand / 1024; ++rep) {
#pragma unroll 2
    for (int c = 0; c < 1024; c += U) {
      float4 cc[U];
#pragma unroll
      for (int u = 0; u < U; ++u) cc[u] = tile[c + u];
      float d[Q][U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (PACKED == 2) {
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            float2 dxy = __fadd2_rn(make_float2(px[q], py[q]), make_float2(-cc[u].x, -cc[u].y));
            float2 sq = __fmul2_rn(dxy, dxy);
            float dz = __fsub_rn(pz[q], cc[u].z);
            d[q][u] = __fadd_rn(__fadd_rn(sq.x, sq.y), __fmul_rn(dz, dz));
          }
        } else if (PACKED) {
#pragma unroll
          for (int qp = 0; qp < Q / 2; ++qp) {
            float2 X = make_float2(px[2 * qp], px[2 * qp + 1]);
            float2 Y = make_float2(py[2 * qp], py[2 * qp + 1]);
            float2 Z = make_float2(pz[2 * qp], pz[2 * qp + 1]);
            float2 dx = __fadd2_rn(X, make_float2(-cc[u].x, -cc[u].x));
            float2 dy = __fadd2_rn(Y, make_float2(-cc[u].y, -cc[u].y));
            float2 dz = __fadd2_rn(Z, make_float2(-cc[u].z, -cc[u].z));
            float2 xx = __fmul2_rn(dx, dx), yy = __fmul2_rn(dy, dy), zz = __fmul2_rn(dz, dz);
            d[2 * qp][u] = __fadd_rn(__fadd_rn(xx.x, yy.x), zz.x);
            d[2 * qp + 1][u] = __fadd_rn(__fadd_rn(xx.y, yy.y), zz.y);
          }
        } else {
#pragma unroll
          for (int q = 0; q < Q; ++q) {
            float dx = __fsub_rn(px[q], cc[u].x), dy = __fsub_rn(py[q], cc[u].y), dz = __fsub_rn(pz[q], cc[u].z);
            d[q][u] = __fadd_rn(__fadd_rn(__fmul_rn(dx, dx), __fmul_rn(dy, dy)), __fmul_rn(dz, dz));
          }
        }
      }
      float m = d[0][0];
#pragma unroll
      for (int q = 0; q < Q; ++q)
#pragma unroll
        for (int u = 0; u < U; ++u)
          if (q || u) m = fminf(m, d[q][u]);
      if (__any_sync(0xffffffffu, m <= limc)) {
#pragma unroll
        for (int q = 0; q < Q; ++q)
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (d[q][u] <= lim[q]) { hits++; lim[q] = fminf(lim[q], d[q][u] * 0.999f); }
        limc = lim[0];
#pragma unroll
        for (int q = 1; q < Q; ++q) limc = fmaxf(limc, lim[q]);
      }
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = hits;
}

template <int PACKED, int Q, int U>
void run(const float4* qpos, const float4* cand, unsigned* out, int clk, int warps_per_sm, const char* name) {
  int blocks = 148 * warps_per_sm / 4, ncand = 16384;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float ms = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(e0);
    loop<PACKED, Q, U><<<blocks, 128>>>(qpos, cand, ncand, 1e-3f, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
  }
  cudaEventElapsedTime(&ms, e0, e1);
  double pairs = (double)blocks * 128 * Q * ncand;
  printf("%-8s Q=%d U=%d warps/SM=%2d: %.3f ms  lane-op frac %.3f\n", name, Q, U, warps_per_sm, ms,
         8 * pairs / (ms * 1e-3) / (148.0 * 128 * clk * 1e3));
}

int main() {
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int nq = 148 * 32 * 128 * 8;
  float4 *qpos, *cand;
  unsigned* out;
  cudaMalloc(&qpos, nq * sizeof(float4));
  cudaMalloc(&cand, 1024 * sizeof(float4));
  cudaMalloc(&out, 148 * 32 * 128 * sizeof(unsigned));
  float4* h = new float4[nq];
  for (int i = 0; i < nq; ++i) h[i] = make_float4((i % 97) * 0.37f, (i % 89) * 0.41f, (i % 83) * 0.43f, 0);
  cudaMemcpy(qpos, h, nq * sizeof(float4), cudaMemcpyHostToDevice);
  for (int i = 0; i < 1024; ++i) h[i] = make_float4((i % 61) * 0.6f + 0.1f, (i % 59) * 0.6f + 0.2f, (i % 53) * 0.6f + 0.3f, 0);
  cudaMemcpy(cand, h, 1024 * sizeof(float4), cudaMemcpyHostToDevice);
  for (int w : {16, 24, 32}) {
    run<0, 4, 4>(qpos, cand, out, clk, w, "scalar");
    run<1, 8, 4>(qpos, cand, out, clk, w, "packedQ");
    run<2, 4, 4>(qpos, cand, out, clk, w, "packedXY");
    run<2, 4, 8>(qpos, cand, out, clk, w, "packedXY");
    run<2, 8, 4>(qpos, cand, out, clk, w, "packedXY");
    run<2, 2, 8>(qpos, cand, out, clk, w, "packedXY");
  }
  return 0;
}
