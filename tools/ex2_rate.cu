// Microbenchmark: MUFU throughput of ex2.approx.f32 vs ex2.approx.f16x2 (two results per lane)
// vs ex2.approx.ftz.bf16x2, 512 threads per SM, all SMs, independent chains (8 per thread).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/ex2_rate.cu -o tools/ex2_rate
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>

template <int MODE>
__global__ void __launch_bounds__(512, 1) k(float* sink, long long* cyc, int iters) {
  uint32_t r[8];
  float f[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    f[i] = -0.001f * (threadIdx.x + i);
    r[i] = 0xB800B800u + i;  // f16x2 / bf16x2 small negatives
  }
  __syncthreads();
  const long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (MODE == 0) asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(f[i]));
      if (MODE == 1) asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(r[i]));
      if (MODE == 2) asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(r[i]));
    }
  }
  __syncthreads();
  const long long t1 = clock64();
  float s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += f[i] + __uint_as_float(r[i]);
  if (s == 1234.5f) sink[threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
  float* sink;
  long long* cyc;
  cudaMalloc(&sink, 4096);
  cudaMalloc(&cyc, 148 * 8);
  const int iters = 4096;
  const char* names[3] = {"ex2.approx.ftz.f32", "ex2.approx.f16x2", "ex2.approx.ftz.bf16x2"};
  for (int mode = 0; mode < 3; ++mode) {
    for (int rep = 0; rep < 2; ++rep) {
      if (mode == 0) k<0><<<148, 512>>>(sink, cyc, iters);
      if (mode == 1) k<1><<<148, 512>>>(sink, cyc, iters);
      if (mode == 2) k<2><<<148, 512>>>(sink, cyc, iters);
    }
    cudaError_t e = cudaDeviceSynchronize();
    long long h;
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    const double instr = 512.0 * 8 * iters;  // thread-instructions per SM
    const double per = mode == 0 ? 1.0 : 2.0;
    printf("%-24s %s: %.2f instr/clk/SM -> %.2f exp2/clk/SM\n", names[mode], cudaGetErrorString(e), instr / h,
           instr * per / h);
  }
  return 0;
}
