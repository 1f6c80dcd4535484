// Microbenchmark: does shared-memory traffic from concurrent bulk copies (the attention loader's
// K/V stream) slow tcgen05.mma?  One thread issues M=128 N=128 K=16 MMAs back to back (SS: both
// operands from smem = 128 B/clk of smem reads at full rate; TS: A from TMEM, B from smem) while
// three other warps keep 4 KB bulk copies global(L2) -> smem in flight.  One CTA per SM.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_asplos_0017wzlxszh0w26_b200/csrc tools/mma_smem.cu -o tools/mma_smem
#include <cstdio>
#include <cstdint>
#include "ptx.cuh"
using namespace bat;

template <bool TS, bool COPIES>
__global__ void __launch_bounds__(128, 1) k(const char* src, long long* out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t bar, cbar[3];
  __shared__ uint32_t tbase;
  __shared__ volatile int stop;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    for (int i = 0; i < 3; ++i) ptx::mbar_init(&cbar[i], 1);
    ptx::fence_mbar_init();
    stop = 0;
  }
  if (warp == 0) ptx::tmem_alloc(&tbase, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = tbase;
  if (warp == 0 && lane == 0) {
    const uint64_t da = ptx::desc_sw128(ptx::smem_u32(smem), 16, 1024);
    const uint64_t db = ptx::desc_sw128(ptx::smem_u32(smem + 32768), TS ? 16384 : 16, 1024);
    constexpr uint32_t idesc = ptx::idesc_bf16(128, 128, 0, TS ? 1 : 0);
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
      for (int kk = 0; kk < 8; ++kk) {
        if (TS) ptx::mma_ts(tmem + 256, tmem + kk * 8, db + kk * 128, idesc, 1u);
        else ptx::mma_ss(tmem, da + (kk & 3) * 2 + (kk >> 2) * 1024, db + (kk & 3) * 2 + (kk >> 2) * 1024, idesc, 1u);
      }
    }
    ptx::mma_commit(&bar);
    ptx::mbar_wait(&bar, 0);
    long long t1 = clock64();
    stop = 1;
    if (blockIdx.x == 0) out[0] = t1 - t0;
  } else if (COPIES && warp >= 1 && lane == 0) {
    const char* base = src + (blockIdx.x % 8) * (1 << 20);
    uint8_t* dst = smem + 65536 + (warp - 1) * 16384;
    long long bytes = 0, t0 = clock64();
    for (int r = 0; !stop; ++r) {
      ptx::mbar_expect_tx(&cbar[warp - 1], 16384);
      for (int c = 0; c < 4; ++c)
        ptx::bulk_g2s(dst + c * 4096, base + ((r * 5 + c * 3 + warp * 7) % 256) * 4096, 4096, &cbar[warp - 1]);
      ptx::mbar_wait(&cbar[warp - 1], r & 1);
      bytes += 16384;
    }
    long long t1 = clock64();
    if (blockIdx.x == 0) out[warp] = bytes * 1000 / (t1 - t0);
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) ptx::tmem_dealloc(tmem, 512);
}

template <bool TS, bool C>
void run(const char* src, long long* d, const char* name) {
  cudaFuncSetAttribute(k<TS, C>, cudaFuncAttributeMaxDynamicSharedMemorySize, 120000);
  const int iters = 4000;
  cudaMemset(d, 0, 32);
  k<TS, C><<<148, 128, 120000>>>(src, d, iters);
  k<TS, C><<<148, 128, 120000>>>(src, d, iters);
  long long h[4];
  cudaMemcpy(h, d, 32, cudaMemcpyDeviceToHost);
  printf("%-28s %.1f cycles/MMA (ideal 64), copies %.1f B/clk  %s\n", name, double(h[0]) / (iters * 8),
         (h[1] + h[2] + h[3]) / 1000.0, cudaGetErrorString(cudaGetLastError()));
}
int main() {
  char* src;
  cudaMalloc(&src, 8 << 20);
  cudaMemset(src, 1, 8 << 20);
  long long* d;
  cudaMalloc(&d, 32);
  run<false, false>(src, d, "SS alone");
  run<false, true>(src, d, "SS + bulk copies");
  run<true, false>(src, d, "TS alone");
  run<true, true>(src, d, "TS + bulk copies");
  return 0;
}
