// Microbenchmark for the round-2 attention softmax layout: the two-q-tile chain
//   S_q = Q_q K^T (8 SS MMAs) -> softmax (ONE thread per row, all 128 columns: row max first,
//   lazy reference max, exp2 on MUFU + a share on the FMA pipe, P as bf16 into S's first 64
//   TMEM columns) -> O_q += P_q V (8 TS MMAs) -> the next S_q
// with one 4-warp softmax team per q-tile (no cross-thread row agreement), no loaders / masks.
// Reports clk per k-tile pair (tensor work per pair: 2048 clk).  Compare tools/chain_rate.cu
// (round-1 layout: two threads per row, 2,753 clk).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I paper_conf_asplos_0017wzlxszh0w26_b200/csrc -I include tools/fa4_chain.cu -o tools/fa4_chain
#include <cstdio>
#include <cuda_bf16.h>
#include "ptx.cuh"
#include "attn_math.cuh"

namespace bat {
namespace {

// P = exp2(s * scale - m) for 128 columns held in registers; POLY of the 64 pairs on the FMA
// pipe; bf16 pairs stored to TMEM columns [0, 64) in four 16-column chunks as they are ready
template <int POLY, bool MASKED>
__device__ __forceinline__ float softmax_row(uint32_t tS, uint32_t (&s)[128], float& m_ref, float scale,
                                             const uint32_t (&vis)[4]) {
  if (MASKED) {
#pragma unroll
    for (int i = 0; i < 128; ++i) s[i] = ((vis[i >> 5] >> (i & 31)) & 1u) ? s[i] : 0xff800000u;
  }
  float m0 = -INFINITY, m1 = -INFINITY, m2 = -INFINITY, m3 = -INFINITY;
#pragma unroll
  for (int i = 0; i < 128; i += 8) {
    m0 = fmax3(m0, __uint_as_float(s[i]), __uint_as_float(s[i + 1]));
    m1 = fmax3(m1, __uint_as_float(s[i + 2]), __uint_as_float(s[i + 3]));
    m2 = fmax3(m2, __uint_as_float(s[i + 4]), __uint_as_float(s[i + 5]));
    m3 = fmax3(m3, __uint_as_float(s[i + 6]), __uint_as_float(s[i + 7]));
  }
  const float mt = fmaxf(fmaxf(m0, m1), fmaxf(m2, m3)) * scale;
  if (mt > m_ref + 8.0f) m_ref = mt;  // lazy: P <= 2^8 otherwise
  const float mr = m_ref == -INFINITY ? 0.0f : m_ref;
  const uint64_t sc2 = pk2(scale, scale), nm2 = pk2(-mr, -mr);
  uint64_t acc0 = pk2(0.f, 0.f), acc1 = acc0;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    uint32_t pk[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      const int i = c * 16 + j;  // pair index
      const uint64_t x = ffma2(pk2(__uint_as_float(s[2 * i]), __uint_as_float(s[2 * i + 1])), sc2, nm2);
      uint64_t e;
      if ((i & 63) < POLY && (!MASKED)) {
        e = exp2_poly2(x);
      } else {
        float x0, x1;
        up2(x, x0, x1);
        e = pk2(ex2(x0), ex2(x1));
      }
      if (j & 1) acc1 = fadd2(acc1, e);
      else acc0 = fadd2(acc0, e);
      float p0, p1;
      up2(e, p0, p1);
      pk[j] = ptx::pack_bf16x2(p0, p1);
    }
    ptx::tmem_st16(tS + c * 16, pk);
  }
  float a0, a1, b0, b1;
  up2(acc0, a0, a1);
  up2(acc1, b0, b1);
  return (a0 + a1) + (b0 + b1);
}

template <int POLY>
__global__ void __launch_bounds__(384, 1) chain(long long* out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t s_full[2], p_full[2];
  __shared__ uint32_t tbase;
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();
  if (threadIdx.x == 0) {
    for (int q = 0; q < 2; ++q) {
      ptx::mbar_init(&s_full[q], 1);
      ptx::mbar_init(&p_full[q], 4);
    }
    ptx::fence_mbar_init();
  }
  for (int i = threadIdx.x; i < 131072 / 16; i += blockDim.x) reinterpret_cast<uint4*>(smem)[i] = make_uint4(0, 0, 0, 0);
  ptx::fence_proxy_async_smem();
  if (warp == 0) ptx::tmem_alloc(&tbase, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = tbase;
  if (warp == 0) {
    const uint32_t sq = ptx::smem_u32(smem), sk = sq + 65536, sv = sq + 98304;
    constexpr uint32_t IS = ptx::idesc_bf16(128, 128, 0, 0), IP = ptx::idesc_bf16(128, 128, 0, 1);
    auto issue_s = [&](int q) {
#pragma unroll
      for (int kk = 0; kk < 8; ++kk)
        ptx::mma_ss_elect(tmem + q * 128, ptx::desc_sw128(sq + q * 32768 + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024),
                          ptx::desc_sw128(sk + (kk >> 2) * 1024 + (kk & 3) * 32, 16, 2048), IS, kk ? 1u : 0u);
      ptx::mma_commit_elect(&s_full[q]);
    };
    auto issue_pv = [&](int q) {
#pragma unroll
      for (int i = 0; i < 8; ++i)
        ptx::mma_ts_elect(tmem + 256 + q * 128, tmem + q * 128 + i * 8, ptx::desc_sw128(sv + i * 4096, 1024, 2048), IP, 1u);
    };
    const long long t0 = clock64();
    issue_s(0);
    issue_s(1);
    for (int i = 0; i < iters; ++i)
      for (int q = 0; q < 2; ++q) {
        ptx::mbar_wait(&p_full[q], i & 1);
        ptx::tc_fence_after();
        issue_pv(q);
        if (i + 1 < iters) issue_s(q);
      }
    ptx::mma_commit_elect(&s_full[0]);
    ptx::mbar_wait(&s_full[0], iters & 1);
    const long long t1 = clock64();
    if (lane == 0 && blockIdx.x == 0) out[0] = t1 - t0;
  } else if (warp >= 4) {
    const int q = (warp - 4) >> 2;
    const uint32_t sub = warp & 3;
    const uint32_t tS = tmem + q * 128 + ((sub * 32) << 16);
    float m_ref = -INFINITY, acc = 0.0f;
    const uint32_t vis[4] = {~0u, ~0u, ~0u, ~0u};
    for (int i = 0; i < iters; ++i) {
      ptx::mbar_wait(&s_full[q], i & 1);
      ptx::tc_fence_after();
      uint32_t s[128];
      ptx::tmem_ld32(tS, *reinterpret_cast<uint32_t(*)[32]>(s));
      ptx::tmem_ld32(tS + 32, *reinterpret_cast<uint32_t(*)[32]>(s + 32));
      ptx::tmem_ld32(tS + 64, *reinterpret_cast<uint32_t(*)[32]>(s + 64));
      ptx::tmem_ld32(tS + 96, *reinterpret_cast<uint32_t(*)[32]>(s + 96));
      ptx::tmem_ld_wait();
      acc += softmax_row<POLY, false>(tS, s, m_ref, 0.01f, vis);
      ptx::tmem_st_wait();
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&p_full[q]);
    }
    if (acc == 12345.0f) out[1] = 1;
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) ptx::tmem_dealloc(tmem, 512);
}

}  // namespace
}  // namespace bat

int main() {
  using namespace bat;
  long long* d;
  cudaMalloc(&d, 8 * sizeof(long long));
  const int iters = 400;
  const size_t smem = 131072;
  auto run = [&](auto kern, int poly) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    for (int rep = 0; rep < 2; ++rep) {
      cudaMemset(d, 0, 8 * sizeof(long long));
      kern<<<148, 384, smem>>>(d, iters);
      cudaError_t e = cudaDeviceSynchronize();
      long long h[8];
      cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
      if (rep) printf("1 thread/row, 2 q-tiles, %2d of 64 pairs on the FMA pipe: %s  clk per k-tile pair %.0f (tensor 2048)\n",
                      poly, cudaGetErrorString(e), double(h[0]) / iters);
    }
  };
  run(chain<0>, 0);
  run(chain<8>, 8);
  run(chain<16>, 16);
  run(chain<24>, 24);
  run(chain<32>, 32);
  return 0;
}
