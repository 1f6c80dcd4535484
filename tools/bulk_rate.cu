// Microbenchmark: issue cost of 2 KB cp.async.bulk global->shared copies (the attention loader's
// per-page K/V blocks), one CTA per SM, source in L2.  Copies per round: 32 (= one K+V tile
// pair of 8 pages x 2 chunks x {K,V}); reports cycles to ISSUE a round and to COMPLETE it.
//   mode 0: one warp, lanes 0-7 each issue 4 copies (the kernel's current scheme)
//   mode 1: one warp, lane 0 issues all 32
//   mode 2: four warps, lane 0 of each issues 8
//   mode 3: eight warps, lane 0 of each issues 4
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_asplos_0017wzlxszh0w26_b200/csrc tools/bulk_rate.cu -o tools/bulk_rate
#include <cstdio>
#include <cstdint>
#include "ptx.cuh"
using namespace bat;

template <int MODE>
__global__ void __launch_bounds__(256, 1) k(const char* src, long long* out, int rounds) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t bar;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
  }
  __syncthreads();
  const char* base = src + (blockIdx.x % 16) * 65536;  // 16 distinct 64 KB source areas, L2-resident
  long long t_issue = 0, t0 = clock64();
  for (int r = 0; r < rounds; ++r) {
    if (threadIdx.x == 0) ptx::mbar_expect_tx(&bar, 32 * 2048);
    __syncthreads();
    const long long ti = clock64();
    if (MODE == 0) {
      if (warp == 0 && lane < 8)
        for (int c = 0; c < 4; ++c)
          ptx::bulk_g2s(smem + (lane * 4 + c) * 2048, base + ((lane * 7 + c * 3) % 32) * 2048, 2048, &bar);
    } else if (MODE == 1) {
      if (warp == 0 && lane == 0)
        for (int c = 0; c < 32; ++c) ptx::bulk_g2s(smem + c * 2048, base + ((c * 7) % 32) * 2048, 2048, &bar);
    } else if (MODE == 2) {
      if (warp < 4 && lane == 0)
        for (int c = 0; c < 8; ++c)
          ptx::bulk_g2s(smem + (warp * 8 + c) * 2048, base + (((warp * 8 + c) * 7) % 32) * 2048, 2048, &bar);
    } else {
      if (lane == 0)
        for (int c = 0; c < 4; ++c)
          ptx::bulk_g2s(smem + (warp * 4 + c) * 2048, base + (((warp * 4 + c) * 7) % 32) * 2048, 2048, &bar);
    }
    if (threadIdx.x == 0) t_issue += clock64() - ti;
    ptx::mbar_wait(&bar, r & 1);
    __syncthreads();
  }
  const long long t1 = clock64();
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    out[0] = t1 - t0;
    out[1] = t_issue;
  }
}

int main() {
  char* src;
  long long* d;
  cudaMalloc(&src, 16 * 65536 + 65536);
  cudaMemset(src, 1, 16 * 65536 + 65536);
  cudaMalloc(&d, 16);
  const int rounds = 2000;
  auto run = [&](auto kern, const char* name) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
    kern<<<148, 256, 70000>>>(src, d, rounds);
    kern<<<148, 256, 70000>>>(src, d, rounds);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[2];
    cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
    printf("%-40s %s  cycles/round %.0f  (issue by thread 0's group %.0f)  -> %.1f B/clk/SM\n", name,
           cudaGetErrorString(e), double(h[0]) / rounds, double(h[1]) / rounds, 65536.0 * rounds / double(h[0]));
  };
  run(k<0>, "1 warp, lanes 0-7 x 4 copies");
  run(k<1>, "1 warp, lane 0 x 32 copies");
  run(k<2>, "4 warps, lane 0 x 8 copies");
  run(k<3>, "8 warps, lane 0 x 4 copies");
  return 0;
}
