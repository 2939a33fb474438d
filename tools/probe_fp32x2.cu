// Microbenchmark: FP32 pipe throughput of scalar FADD/FMUL vs packed FADD2/FMUL2
// on sm_100a, and of the candidate distance pattern (packed sub/mul + scalar add).
// Development probe (not part of libboids).  nvcc -gencode arch=compute_100a,code=sm_100a -O3 --fmad=false
#include <cstdio>
#include <cuda_runtime.h>

#define ITERS 4096
template <int MODE>
__global__ void k(float* out, float s) {
  float a[8];
  float2 b[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { a[i] = threadIdx.x * 1e-3f + i; b[i] = make_float2(a[i], a[i] + 0.5f); }
  float c = s, d = 1.0000001f;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (MODE == 0) a[i] = __fadd_rn(a[i], c);            // 1 lane-op / instr
      if (MODE == 1) a[i] = __fmul_rn(a[i], d);
      if (MODE == 2) b[i] = __fadd2_rn(b[i], make_float2(c, c));  // 2 lane-ops / instr
      if (MODE == 3) b[i] = __fmul2_rn(b[i], make_float2(d, d));
    }
  }
  float r = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) r += a[i] + b[i].x + b[i].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = r;
}

// the distance pattern: Q queries x candidates from smem.  MODE 0 scalar,
// 1 packed sub+mul / scalar add, 2 packed sub / scalar mul+add.
template <int MODE, int Q>
__global__ void kd(float* out, int reps) {
  __shared__ float4 cand[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) cand[i] = make_float4(i * 0.01f, i * 0.02f, i * 0.03f, 0);
  __syncthreads();
  float2 px[Q / 2], py[Q / 2], pz[Q / 2];
  for (int q = 0; q < Q / 2; ++q) {
    px[q] = make_float2(threadIdx.x * 1e-3f, q * 0.7f);
    py[q] = make_float2(threadIdx.x * 2e-3f + 0.3f, q * 0.3f + 0.1f);
    pz[q] = make_float2(threadIdx.x * 3e-3f + 0.7f, q * 0.5f + 0.2f);
  }
  float lim = 1e-4f;
  int hits = 0;
  for (int r = 0; r < reps; ++r) {
#pragma unroll 4
    for (int c = 0; c < 256; ++c) {
      float4 v = cand[c];
      bool h = false;
#pragma unroll
      for (int q = 0; q < Q / 2; ++q) {
        if (MODE == 1) {
          float2 dx = __fadd2_rn(px[q], make_float2(-v.x, -v.x));
          float2 dy = __fadd2_rn(py[q], make_float2(-v.y, -v.y));
          float2 dz = __fadd2_rn(pz[q], make_float2(-v.z, -v.z));
          float2 xx = __fmul2_rn(dx, dx), yy = __fmul2_rn(dy, dy), zz = __fmul2_rn(dz, dz);
          float d0 = __fadd_rn(__fadd_rn(xx.x, yy.x), zz.x);
          float d1 = __fadd_rn(__fadd_rn(xx.y, yy.y), zz.y);
          h |= d0 < lim; h |= d1 < lim;
        } else if (MODE == 2) {
          float2 dx = __fadd2_rn(px[q], make_float2(-v.x, -v.x));
          float2 dy = __fadd2_rn(py[q], make_float2(-v.y, -v.y));
          float2 dz = __fadd2_rn(pz[q], make_float2(-v.z, -v.z));
          float d0 = __fadd_rn(__fadd_rn(__fmul_rn(dx.x, dx.x), __fmul_rn(dy.x, dy.x)), __fmul_rn(dz.x, dz.x));
          float d1 = __fadd_rn(__fadd_rn(__fmul_rn(dx.y, dx.y), __fmul_rn(dy.y, dy.y)), __fmul_rn(dz.y, dz.y));
          h |= d0 < lim; h |= d1 < lim;
        } else {
          for (int e = 0; e < 2; ++e) {
            float x = __fsub_rn(e ? px[q].y : px[q].x, v.x), y = __fsub_rn(e ? py[q].y : py[q].x, v.y),
                  z = __fsub_rn(e ? pz[q].y : pz[q].x, v.z);
            float d = __fadd_rn(__fadd_rn(__fmul_rn(x, x), __fmul_rn(y, y)), __fmul_rn(z, z));
            h |= d < lim;
          }
        }
      }
      if (__any_sync(0xffffffffu, h)) hits++;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = hits;
}

template <int MODE, int Q>
void run_kd(float* out, int clk, cudaEvent_t e0, cudaEvent_t e1, int warps_per_sm) {
  int blocks = 148 * warps_per_sm / 4, reps = 64 * 4 / Q;
  float ms = 0;
  for (int rep = 0; rep < 2; ++rep) {
    cudaEventRecord(e0);
    kd<MODE, Q><<<blocks, 128>>>(out, reps);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
  }
  cudaEventElapsedTime(&ms, e0, e1);
  double pairs = (double)blocks * 128 * reps * 256 * Q;
  const char* nm[3] = {"scalar", "packed sub+mul", "packed sub"};
  printf("dist %-15s Q=%d warps/SM=%2d: %.3f ms, %.1f Gpairs/s, lane-op frac %.3f\n", nm[MODE], Q, warps_per_sm, ms,
         pairs / ms / 1e6, 8 * pairs / (ms * 1e-3) / (148.0 * 128 * clk * 1e3));
}

int main() {
  float* out;
  cudaMalloc(&out, 148 * 64 * 256 * sizeof(float));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int dev;
  cudaGetDevice(&dev);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  int blocks = 148 * 8, threads = 256;
  const char* names[4] = {"FADD", "FMUL", "FADD2", "FMUL2"};
  for (int mode = 0; mode < 4; ++mode) {
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      if (mode == 0) k<0><<<blocks, threads>>>(out, 1e-7f);
      if (mode == 1) k<1><<<blocks, threads>>>(out, 1e-7f);
      if (mode == 2) k<2><<<blocks, threads>>>(out, 1e-7f);
      if (mode == 3) k<3><<<blocks, threads>>>(out, 1e-7f);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
    }
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    double instr = (double)blocks * threads / 32 * ITERS * 8;
    double lane_ops = (double)blocks * threads * ITERS * 8 * (mode >= 2 ? 2 : 1);
    printf("%-6s %.3f ms  warp-instr/cycle/SM %.3f  lane-ops/cycle/SM %.1f (clock %.0f MHz assumed max)\n", names[mode],
           ms, instr / (ms * 1e-3) / 148 / (clk * 1e3), lane_ops / (ms * 1e-3) / 148 / (clk * 1e3), clk / 1e3);
  }
  for (int w : {8, 16, 32}) {
    run_kd<0, 2>(out, clk, e0, e1, w);
    run_kd<0, 4>(out, clk, e0, e1, w);
    run_kd<1, 2>(out, clk, e0, e1, w);
    run_kd<1, 4>(out, clk, e0, e1, w);
    run_kd<2, 4>(out, clk, e0, e1, w);
  }
  return 0;
}
