// Minimal TMA bulk-copy ring (full/empty mbarriers) for compute-sanitizer racecheck:
// does the tool report hazards on a textbook-ordered ring?  Development probe.
#include <cstdio>
#include "../paper_conf_ipps_breitbart09_b200/csrc/tma.cuh"
using namespace boids;
constexpr int CT = 256, S = 2, NT = 128;
__global__ void ring(const float4* src, int tiles, float* out) {
  __shared__ __align__(16) float4 buf[S][CT];
  __shared__ uint64_t full[S], empty[S];
  int tid = threadIdx.x, lane = tid & 31;
  if (tid == 0) {
    for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], NT / 32); }
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int t = 0; t < S && t < tiles; ++t) {
      mbar_arrive_expect_tx(&full[t], CT * 16);
      tma_load_1d(buf[t], src + t * CT, CT * 16, &full[t]);
    }
  float acc = 0;
  for (int t = 0; t < tiles; ++t) {
    int s = t % S;
    mbar_wait(&full[s], (t / S) & 1);
    for (int c = 0; c < CT; ++c) acc += buf[s][c].x;
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);
    if (tid == 0 && t + S < tiles) {
      mbar_wait(&empty[s], (t / S) & 1);
      fence_proxy_async_smem();
      mbar_arrive_expect_tx(&full[s], CT * 16);
      tma_load_1d(buf[s], src + (t + S) * CT, CT * 16, &full[s]);
    }
  }
  out[tid] = acc;
}
int main() {
  const int tiles = 16;
  float4* src; float* out;
  cudaMalloc(&src, tiles * CT * 16); cudaMalloc(&out, NT * 4);
  cudaMemset(src, 0, tiles * CT * 16);
  ring<<<1, NT>>>(src, tiles, out);
  printf("sync %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
