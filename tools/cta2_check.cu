// Stand-alone check of the CTA-pair (cta_group::2) MMA operand split the pair attention kernel
// relies on, against a host reference:
//   S = Q K^T : SS, M = 256 (CTA r holds Q rows [128r, 128r+128) at the same smem address),
//               N = 128 keys (CTA r holds keys [64r, 64r+64) — K-major, 128-byte swizzle);
//   O = P V   : TS, P = bf16(S / 64) written by each CTA into its own TMEM, V MN-major with
//               CTA r holding d-columns [64r, 64r+64) of all 128 keys.
// Both CTAs read their 128 rows of S and O from TMEM; the leader issues every MMA and commits
// with multicast to both CTAs' barriers; P readiness is signalled to the leader by remote arrives.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_asplos_0017wzlxszh0w26_b200/csrc tools/cta2_check.cu -o tools/cta2_check
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <vector>

#include <cuda_bf16.h>
#include "ptx.cuh"
using namespace bat;

constexpr int D = 128;

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(256, 1)
    pair_check(const __nv_bfloat16* Q, const __nv_bfloat16* K, const __nv_bfloat16* V, float* Sout, float* Oout) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;            // [2 chunks][128 rows][64]  32 KB
  uint8_t* sK = smem + 32768;    // [2 chunks][64 keys][64]   16 KB
  uint8_t* sV = smem + 49152;    // [128 keys][64 d]          16 KB
  __shared__ uint64_t bar_s, bar_p, bar_o;
  __shared__ uint32_t tbase;
  const uint32_t rank = ptx::cluster_ctarank();
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  // operands into shared memory (generic stores, 128-byte swizzle by hand)
  for (int e = threadIdx.x; e < 128 * 16; e += blockDim.x) {  // Q: row, 16-byte unit
    const int r = e / 16, u = e % 16, c = u / 8;
    const uint4 v = *reinterpret_cast<const uint4*>(Q + (size_t)(128 * rank + r) * D + u * 8);
    *reinterpret_cast<uint4*>(sQ + c * 16384 + ptx::swz128(r, u % 8)) = v;
  }
  for (int e = threadIdx.x; e < 64 * 16; e += blockDim.x) {  // K half
    const int r = e / 16, u = e % 16, c = u / 8;
    const uint4 v = *reinterpret_cast<const uint4*>(K + (size_t)(64 * rank + r) * D + u * 8);
    *reinterpret_cast<uint4*>(sK + c * 8192 + ptx::swz128(r, u % 8)) = v;
  }
  for (int e = threadIdx.x; e < 128 * 8; e += blockDim.x) {  // V: key row, 16-byte unit of my d half
    const int r = e / 8, u = e % 8;
    const uint4 v = *reinterpret_cast<const uint4*>(V + (size_t)r * D + 64 * rank + u * 8);
    *reinterpret_cast<uint4*>(sV + ptx::swz128(r, u)) = v;
  }
  ptx::fence_proxy_async_smem();
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar_s, 1);
    ptx::mbar_init(&bar_p, 8);
    ptx::mbar_init(&bar_o, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 0) ptx::tmem_alloc2(&tbase, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem = tbase;
  if (rank == 0 && threadIdx.x == 0) {
    constexpr uint32_t IS = ptx::idesc_bf16(256, 128, 0, 0);
    const uint32_t q = ptx::smem_u32(sQ), k = ptx::smem_u32(sK);
    for (int kk = 0; kk < D / 16; ++kk)
      ptx::mma2_ss(tmem, ptx::desc_sw128(q + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024),
                   ptx::desc_sw128(k + (kk >> 2) * 8192 + (kk & 3) * 32, 16, 1024), IS, kk ? 1u : 0u);
    ptx::mma2_commit(&bar_s, 3);
  }
  if (warp < 4) {
    ptx::mbar_wait(&bar_s, 0);
    ptx::tc_fence_after();
    const int row = warp * 32 + lane;
    const uint32_t lb = uint32_t(warp * 32) << 16;
    for (int c = 0; c < 4; ++c) {
      uint32_t r[32];
      ptx::tmem_ld32(tmem + lb + c * 32, r);
      ptx::tmem_ld_wait();
      for (int i = 0; i < 32; ++i) Sout[(size_t)(128 * rank + row) * 128 + c * 32 + i] = __uint_as_float(r[i]);
      uint32_t pk[16];
      for (int i = 0; i < 16; ++i)
        pk[i] = ptx::pack_bf16x2(__uint_as_float(r[2 * i]) / 64.0f, __uint_as_float(r[2 * i + 1]) / 64.0f);
      uint32_t full[32];
      for (int i = 0; i < 32; ++i) full[i] = i < 16 ? pk[i] : 0u;
      ptx::tmem_st32(tmem + lb + 128 + c * 16, full);  // P at columns [128, 192), 16 per 32 keys
      ptx::tmem_st_wait();
    }
    ptx::tc_fence_before();
    __syncwarp();
    if (lane == 0) ptx::mbar_arrive_cluster(ptx::mapa(ptx::smem_u32(&bar_p), 0));
  }
  if (rank == 0 && threadIdx.x == 32) {
    ptx::mbar_wait(&bar_p, 0);
    ptx::tc_fence_after();
    constexpr uint32_t IP = ptx::idesc_bf16(256, 128, 0, 1);
    const uint32_t v = ptx::smem_u32(sV);
    for (int kk = 0; kk < 8; ++kk)
      ptx::mma2_ts(tmem + 256, tmem + 128 + kk * 8, ptx::desc_sw128(v + kk * 2048, 16384, 1024), IP, kk ? 1u : 0u);
    ptx::mma2_commit(&bar_o, 3);
  }
  if (warp < 4) {
    ptx::mbar_wait(&bar_o, 0);
    ptx::tc_fence_after();
    const int row = warp * 32 + lane;
    const uint32_t lb = uint32_t(warp * 32) << 16;
    for (int c = 0; c < 4; ++c) {
      uint32_t r[32];
      ptx::tmem_ld32(tmem + lb + 256 + c * 32, r);
      ptx::tmem_ld_wait();
      for (int i = 0; i < 32; ++i) Oout[(size_t)(128 * rank + row) * 128 + c * 32 + i] = __uint_as_float(r[i]);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::cluster_sync();
  if (warp == 0) ptx::tmem_dealloc2(tmem, 512);
}

static float bf(float x) { return __bfloat162float(__float2bfloat16(x)); }

int main() {
  std::vector<__nv_bfloat16> hq(256 * D), hk(128 * D), hv(128 * D);
  std::vector<float> fq(256 * D), fk(128 * D), fv(128 * D);
  uint32_t st = 12345;
  auto rnd = [&]() { st = st * 1664525u + 1013904223u; return (int((st >> 9) % 2001) - 1000) / 1000.0f; };
  for (int i = 0; i < 256 * D; ++i) { fq[i] = bf(rnd()); hq[i] = __float2bfloat16(fq[i]); }
  for (int i = 0; i < 128 * D; ++i) { fk[i] = bf(rnd()); hk[i] = __float2bfloat16(fk[i]); }
  for (int i = 0; i < 128 * D; ++i) { fv[i] = bf(rnd()); hv[i] = __float2bfloat16(fv[i]); }
  __nv_bfloat16 *dq, *dk, *dv;
  float *ds, *dout;
  cudaMalloc(&dq, hq.size() * 2); cudaMalloc(&dk, hk.size() * 2); cudaMalloc(&dv, hv.size() * 2);
  cudaMalloc(&ds, 256 * 128 * 4); cudaMalloc(&dout, 256 * 128 * 4);
  cudaMemcpy(dq, hq.data(), hq.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dk, hk.data(), hk.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dv, hv.data(), hv.size() * 2, cudaMemcpyHostToDevice);
  cudaFuncSetAttribute(pair_check, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
  pair_check<<<2, 256, 70000>>>(dq, dk, dv, ds, dout);
  cudaError_t e = cudaDeviceSynchronize();
  printf("kernel: %s\n", cudaGetErrorString(e));
  std::vector<float> S(256 * 128), O(256 * 128);
  cudaMemcpy(S.data(), ds, S.size() * 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(O.data(), dout, O.size() * 4, cudaMemcpyDeviceToHost);
  double es = 0, eo = 0, ms = 0, mo = 0;
  std::vector<float> P(256 * 128);
  for (int m = 0; m < 256; ++m)
    for (int n = 0; n < 128; ++n) {
      double a = 0;
      for (int k = 0; k < D; ++k) a += double(fq[m * D + k]) * fk[n * D + k];
      es = fmax(es, fabs(a - S[m * 128 + n]));
      ms = fmax(ms, fabs(a));
      P[m * 128 + n] = bf(S[m * 128 + n] / 64.0f);  // from the device S: isolates the PV check
    }
  for (int m = 0; m < 256; ++m)
    for (int n = 0; n < 128; ++n) {
      double a = 0;
      for (int k = 0; k < 128; ++k) a += double(P[m * 128 + k]) * fv[k * D + n];
      eo = fmax(eo, fabs(a - O[m * 128 + n]));
      mo = fmax(mo, fabs(a));
    }
  printf("S = Q K^T  max|err| %.3e (max|S| %.2f)\nO = P V    max|err| %.3e (max|O| %.2f)\n%s\n", es, ms, eo, mo,
         (es < 1e-3 * ms && eo < 1e-3 * mo) ? "PASS" : "FAIL");
  return 0;
}
