// Microbenchmark: do TMEM loads (tcgen05.ld 32x32b) and MUFU ex2 overlap across warps?
// 16 warps, each owning 64 fp32 TMEM columns x its 32 lanes; per round a warp loads its 64
// values (2 x .x32, one wait), takes 56 ex2 + 8 FMA-pipe ops on them, sums, and stores 32
// packed columns back (the attention softmax's per-tile work).  Modes: 0 = full, 1 = load +
// store only (no math), 2 = math only (registers, no TMEM traffic).  Prints clk per round
// (one round = 16 warps x 32 lanes x 64 elements = one 128-row x 128-key tile PAIR of S).
#include <cstdio>
#include <cuda_runtime.h>
#include "../paper_conf_asplos_0017wzlxszh0w26_b200/csrc/ptx.cuh"
using namespace bat;

__device__ __forceinline__ float ex2f(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }

__global__ void __launch_bounds__(544, 1) k(int mode, int rounds, long long* out, float* sink) {
  __shared__ uint32_t tbase;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 16) ptx::tmem_alloc(&tbase, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 16) { __syncthreads(); ptx::tmem_dealloc(tbase, 512); return; }
  const uint32_t t = tbase + ((warp & 3) * 32 << 16) + (warp >> 2) * 128 + ((warp >> 2) & 1) * 0;
  const uint32_t tS = t + 0;  // 64 columns at (warp / 4) * 128
  float acc = 0.f;
  uint32_t r[2][32];
#pragma unroll
  for (int i = 0; i < 32; ++i) { r[0][i] = __float_as_uint(-0.01f * i); r[1][i] = __float_as_uint(-0.02f * i); }
  __syncwarp();
  long long t0 = clock64();
  for (int it = 0; it < rounds; ++it) {
    if (mode != 2) {
      ptx::tmem_ld32(tS, r[0]);
      ptx::tmem_ld32(tS + 32, r[1]);
      ptx::tmem_ld_wait();
    }
    uint32_t pk[16];
    if (mode != 1) {
#pragma unroll
      for (int c = 0; c < 2; ++c)
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          float a = __uint_as_float(r[c][2 * i]) * 0.1f - 1.0f, b = __uint_as_float(r[c][2 * i + 1]) * 0.1f - 1.0f;
          float e0 = ex2f(a), e1 = (i < 2) ? fmaf(b, fmaf(b, 0.24f, 0.69f), 1.0f) : ex2f(b);
          acc += e0 + e1;
          if (c == 0) pk[i] = ptx::pack_bf16x2(e0, e1);
          else pk[i] ^= ptx::pack_bf16x2(e0, e1);
        }
    } else {
#pragma unroll
      for (int i = 0; i < 16; ++i) pk[i] = r[0][i] ^ r[1][i];
    }
    if (mode != 2) {
      ptx::tmem_st16(tS, pk);
      ptx::tmem_st16(tS + 16, pk);
      ptx::tmem_st_wait();
    } else {
#pragma unroll
      for (int i = 0; i < 16; ++i) { r[0][i] ^= pk[i]; r[1][i + 16] += pk[i]; }
    }
  }
  long long t1 = clock64();
  if (lane == 0) out[warp] = t1 - t0;
  sink[threadIdx.x] = acc;
  ptx::tc_fence_before();
  __syncthreads();
}

int main() {
  long long* d; float* s;
  cudaMalloc(&d, 16 * sizeof(long long));
  cudaMalloc(&s, 1024 * sizeof(float));
  const int rounds = 2000;
  const char* names[3] = {"ld+math+st", "ld+st only", "math only"};
  for (int mode = 0; mode < 3; ++mode) {
    for (int rep = 0; rep < 2; ++rep) k<<<1, 544>>>(mode, rounds, d, s);
    cudaDeviceSynchronize();
    long long h[16];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < 16; ++i) mx = h[i] > mx ? h[i] : mx;
    printf("%-12s %.0f clk per round (16 warps x 64 elements per lane = one 128x128 S tile pair)\n", names[mode], double(mx) / rounds);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
