// Microbenchmark: global(L2-resident) -> shared throughput per SM at grid = 148, 64 KB per round
// (one K + V tile pair of the attention kernel), with 1 or 2 rounds in flight.
//   bulk S: cp.async.bulk copies of S bytes issued by lane 0 of `nw` warps
//   ldgsts: cp.async 16-byte copies by 256 threads
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_asplos_0017wzlxszh0w26_b200/csrc tools/load_rate.cu -o tools/load_rate
#include <cstdio>
#include <cstdint>
#include "ptx.cuh"
using namespace bat;

constexpr int ROUND = 65536;

__global__ void __launch_bounds__(256, 1) kbulk(const char* src, long long* out, int rounds, int sz, int nw, int inflight,
                                                int spread) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t bar[2];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar[0], 1);
    ptx::mbar_init(&bar[1], 1);
    ptx::fence_mbar_init();
  }
  __syncthreads();
  // spread = 1: every CTA reads its own 1 MB area; spread = 0: 16 CTAs share each area (hot lines)
  const char* base = src + (spread ? blockIdx.x : blockIdx.x % 8) * (1 << 20);
  const int n = ROUND / sz;
  long long t0 = clock64();
  for (int r = 0; r < rounds + inflight - 1; ++r) {
    if (r < rounds) {
      const int b = r & 1;
      if (threadIdx.x == 0) ptx::mbar_expect_tx(&bar[b], ROUND);
      __syncthreads();
      if (warp < nw && lane == 0)
        for (int c = warp; c < n; c += nw)
          ptx::bulk_g2s(smem + b * ROUND * (inflight - 1) + c * sz,
                        base + ((r * 7 + c * 13) % (1048576 / sz)) * sz, sz, &bar[b]);
    }
    const int rw = r - (inflight - 1);
    if (rw >= 0) {
      ptx::mbar_wait(&bar[rw & 1], (rw >> 1) & 1);
      __syncthreads();
    }
  }
  const long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}

__global__ void __launch_bounds__(256, 1) kldgsts(const char* src, long long* out, int rounds) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const char* base = src + blockIdx.x * (1 << 20);
  long long t0 = clock64();
  for (int r = 0; r < rounds; ++r) {
    const char* s = base + ((r * 7) % 16) * ROUND;
    for (int i = threadIdx.x; i < ROUND / 16; i += 256) {
      const uint32_t d = ptx::smem_u32(smem + i * 16);
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(s + i * 16));
    }
    asm volatile("cp.async.commit_group;");
    asm volatile("cp.async.wait_group 0;");
    __syncthreads();
  }
  const long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}

int main() {
  char* src;
  long long* d;
  const size_t bytes = size_t(148) << 20;
  cudaMalloc(&src, bytes);
  cudaMemset(src, 1, bytes);
  cudaMalloc(&d, 148 * 8);
  const int rounds = 400;
  long long h[148];
  auto report = [&](const char* name) {
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double mx = 0, sum = 0;
    for (int i = 0; i < 148; ++i) {
      mx = h[i] > mx ? h[i] : mx;
      sum += h[i];
    }
    printf("%-44s %s cycles/round mean %.0f max %.0f -> %.1f B/clk/SM\n", name, cudaGetErrorString(e),
           sum / 148 / rounds, mx / rounds, double(ROUND) * rounds / (sum / 148));
  };
  cudaFuncSetAttribute(kbulk, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * ROUND);
  cudaFuncSetAttribute(kldgsts, cudaFuncAttributeMaxDynamicSharedMemorySize, ROUND);
  char name[128];
  for (int spread = 1; spread >= 0; --spread)
    for (int inflight = 1; inflight <= 2; ++inflight)
      for (int sz : {2048, 4096, 8192, 16384})
        for (int nw : {1, 3, 8}) {
          kbulk<<<148, 256, 2 * ROUND>>>(src, d, 20, sz, nw, inflight, spread);
          kbulk<<<148, 256, 2 * ROUND>>>(src, d, rounds, sz, nw, inflight, spread);
          snprintf(name, sizeof(name), "bulk %5d B x%2d warps inflight %d %s", sz, nw, inflight,
                   spread ? "own" : "shared");
          report(name);
        }
  kldgsts<<<148, 256, ROUND>>>(src, d, 20);
  kldgsts<<<148, 256, ROUND>>>(src, d, rounds);
  report("cp.async 16 B x 256 threads");
  return 0;
}
