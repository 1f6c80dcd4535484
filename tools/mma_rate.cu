// Microbenchmark: cycles per tcgen05.mma (kind::f16, cta_group::1, M=128) for SS / TS forms and
// several N, issued back to back by one thread, one CTA per SM (all SMs busy).
#include <cstdio>
#include <cstdint>
#include "../paper_conf_asplos_0017wzlxszh0w26_b200/csrc/ptx.cuh"
using namespace bat;
template <int N, bool TS>
__global__ void __launch_bounds__(128, 1) k(long long* out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x / 32;
  if (threadIdx.x == 0) { ptx::mbar_init(&bar, 1); ptx::fence_mbar_init(); }
  if (warp == 0) ptx::tmem_alloc(&tbase, 512);
  ptx::tc_fence_before(); __syncthreads(); ptx::tc_fence_after();
  const uint32_t tmem = tbase;
  if (threadIdx.x == 0) {
    const uint64_t da = ptx::desc_sw128(ptx::smem_u32(smem), 16, 1024);
    const uint64_t db = ptx::desc_sw128(ptx::smem_u32(smem + 32768), TS ? 16384 : 16, 1024);
    constexpr uint32_t idesc = ptx::idesc_bf16(128, N, 0, TS ? 1 : 0);
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
    if (blockIdx.x == 0) out[0] = t1 - t0;
  }
  ptx::tc_fence_before(); __syncthreads();
  if (warp == 0) ptx::tmem_dealloc(tmem, 512);
}
template <int N, bool TS>
void run(long long* d, const char* name) {
  cudaFuncSetAttribute(k<N, TS>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000);
  const int iters = 2000;
  k<N, TS><<<148, 128, 100000>>>(d, iters);
  k<N, TS><<<148, 128, 100000>>>(d, iters);
  long long c; cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
  double per = double(c) / (iters * 8);
  printf("%-22s N=%3d: %.1f cycles/MMA (ideal %d)  %s\n", name, N, per, 128 * N / 256, cudaGetErrorString(cudaGetLastError()));
}
// the attention kernel's pattern per half-tile pair: 2 x (PV: 4 TS N=128 + 2 commits;
// S: 8 SS N=64 + 2 commits)
template <bool COMMITS>
__global__ void __launch_bounds__(128, 1) kp(long long* out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t bar[8];
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x / 32;
  if (threadIdx.x == 0) { for (int i = 0; i < 8; ++i) ptx::mbar_init(&bar[i], 1); ptx::fence_mbar_init(); }
  if (warp == 0) ptx::tmem_alloc(&tbase, 512);
  ptx::tc_fence_before(); __syncthreads(); ptx::tc_fence_after();
  const uint32_t tmem = tbase;
  if (threadIdx.x == 0) {
    const uint64_t da = ptx::desc_sw128(ptx::smem_u32(smem), 16, 1024);
    const uint64_t db = ptx::desc_sw128(ptx::smem_u32(smem + 32768), 16, 1024);
    const uint64_t dv = ptx::desc_sw128(ptx::smem_u32(smem + 65536), 16384, 1024);
    constexpr uint32_t is = ptx::idesc_bf16(128, 64, 0, 0), ip = ptx::idesc_bf16(128, 128, 0, 1);
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      for (int g = 0; g < 2; ++g) {
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) ptx::mma_ts(tmem + 256 + g * 128, tmem + g * 128 + kk * 8, dv + kk * 128, ip, 1u);
        if (COMMITS) { ptx::mma_commit(&bar[0]); ptx::mma_commit(&bar[1]); }
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) ptx::mma_ss(tmem + g * 128 + 64, da + (kk & 3) * 2 + (kk >> 2) * 1024, db + (kk & 3) * 2 + (kk >> 2) * 1024, is, kk ? 1u : 0u);
        if (COMMITS) { ptx::mma_commit(&bar[2]); ptx::mma_commit(&bar[3]); }
      }
    }
    ptx::mma_commit(&bar[4]);
    ptx::mbar_wait(&bar[4], 0);
    long long t1 = clock64();
    if (blockIdx.x == 0) out[0] = t1 - t0;
  }
  ptx::tc_fence_before(); __syncthreads();
  if (warp == 0) ptx::tmem_dealloc(tmem, 512);
}
template <bool C>
void runp(long long* d) {
  cudaFuncSetAttribute(kp<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, 120000);
  const int iters = 1000;
  kp<C><<<148, 128, 120000>>>(d, iters);
  kp<C><<<148, 128, 120000>>>(d, iters);
  long long c; cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
  printf("attention pattern (commits=%d): %.0f cycles per half-tile pair (ideal 1280)  %s\n", int(C), double(c) / iters, cudaGetErrorString(cudaGetLastError()));
}
int main() {
  long long* d; cudaMalloc(&d, 8);
  run<128, false>(d, "SS (Q.K^T form)");
  run<64, false>(d, "SS (Q.K^T form)");
  run<256, false>(d, "SS");
  run<128, true>(d, "TS (P.V form, B MN)");
  run<64, true>(d, "TS (P.V form, B MN)");
  runp<false>(d);
  runp<true>(d);
  return 0;
}
