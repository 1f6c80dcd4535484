// Microbenchmark: throughput of the attention softmax's per-element arithmetic (row_exp_opt of
// k_attn.cu minus TMEM: FFMA2 scale/shift, FMNMX3 running max, 2x MUFU.EX2, FADD2 row sum,
// F2FP bf16 pack) on register data, NWARP warps per SM, all SMs.  Variants drop one instruction
// class at a time to find what, besides MUFU (16 ex2/clk/SM = 1,024 clk per 16,384 elements),
// sets the ~1.5k clk a 128 x 128 tile's softmax takes (tools/chain_ds.cu).
// Reports clk per 16,384 elements (one 128 x 128 tile) per SM.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/sm_mix.cu -o tools/sm_mix
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint64_t pk2(float a, float b) {
  uint64_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ void up2(uint64_t v, float& a, float& b) { asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v)); }
__device__ __forceinline__ uint64_t ffma2(uint64_t a, uint64_t b, uint64_t c) {
  uint64_t d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ uint64_t fadd2(uint64_t a, uint64_t b) {
  uint64_t d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ float ex2(float x) {
  float y;
  asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ uint32_t pack_bf16x2(float lo, float hi) {
  uint32_t r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ float fmax3(float a, float b, float c) {
  float d;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
  return d;
}

// MODE bits: 1 = no F2FP (xor the fp32 bits instead), 2 = no FMNMX3, 4 = no FADD2 sum,
//            8 = no MUFU (FFMA2 only)
template <int MODE>
__global__ void __launch_bounds__(512, 1) k(uint32_t* sink, long long* cyc, int iters) {
  uint32_t r[64];
#pragma unroll
  for (int i = 0; i < 64; ++i) r[i] = __float_as_uint(-0.001f * float((threadIdx.x * 7 + i * 13) & 255));
  __syncthreads();
  const long long t0 = clock64();
  uint32_t pkx = 0;
  float xm0 = -1e30f, xm1 = -1e30f;
  uint64_t acc0 = pk2(0.f, 0.f), acc1 = acc0;
  for (int it = 0; it < iters; ++it) {
    const uint64_t sc2 = pk2(0.7f, 0.7f), nm2 = pk2(-0.0001f * it, -0.0001f * it);
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      const uint64_t xv = ffma2(pk2(__uint_as_float(r[2 * i]), __uint_as_float(r[2 * i + 1])), sc2, nm2);
      float x0, x1;
      up2(xv, x0, x1);
      if (!(MODE & 2)) {
        if (i & 1) xm1 = fmax3(xm1, x0, x1);
        else xm0 = fmax3(xm0, x0, x1);
      }
      float p0 = x0, p1 = x1;
      if (!(MODE & 8)) {
        p0 = ex2(x0);
        p1 = ex2(x1);
      }
      if (!(MODE & 4)) {
        if (i & 1) acc1 = fadd2(acc1, pk2(p0, p1));
        else acc0 = fadd2(acc0, pk2(p0, p1));
      }
      if (MODE & 1) pkx ^= __float_as_uint(p0) ^ __float_as_uint(p1);
      else pkx ^= pack_bf16x2(p0, p1);
    }
  }
  const long long t1 = clock64();
  float a0, a1, b0, b1;
  up2(acc0, a0, a1);
  up2(acc1, b0, b1);
  sink[blockIdx.x * blockDim.x + threadIdx.x] = pkx ^ __float_as_uint(a0 + a1 + b0 + b1 + xm0 + xm1);
  if (threadIdx.x == 0 && blockIdx.x == 0) cyc[0] = t1 - t0;
}

int main() {
  uint32_t* sink;
  long long* cyc;
  cudaMalloc(&sink, 148 * 512 * 4);
  cudaMalloc(&cyc, 8);
  const int iters = 2000;
  auto run = [&](auto kern, const char* name, int threads) {
    kern<<<148, threads>>>(sink, cyc, iters);
    cudaError_t e = cudaDeviceSynchronize();
    long long c;
    cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    const double elems = double(iters) * 64 * threads;  // per SM
    printf("%-40s %3d warps  %s  clk per 16,384 elements %.0f\n", name, threads / 32, cudaGetErrorString(e),
           double(c) / elems * 16384);
  };
  for (int t : {128, 256, 512}) {
    run(k<0>, "full mix (FFMA2 FMNMX3 2xEX2 FADD2 F2FP)", t);
    run(k<1>, "no F2FP", t);
    run(k<2>, "no FMNMX3", t);
    run(k<4>, "no FADD2", t);
    run(k<7>, "EX2 + FFMA2 only", t);
    run(k<8>, "no EX2", t);
  }
  return 0;
}
