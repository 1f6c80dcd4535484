// Microbenchmark: ONE q-tile per CTA with S double-buffered in TMEM (S_{x+1} = Q K_{x+1}^T is
// computed while the softmax of tile x runs; MMA order S_0 S_1 | PV_0 S_2 | PV_1 S_3 | ...), the
// softmax of every tile done by a team of NW warps: NW / 4 warps per TMEM lane quarter, each
// owning 128 / (NW / 4) columns of its 32 rows (row_exp_opt of k_attn.cu; the column slices of a
// row agree on the fast path through smem + a named barrier).  No loaders / masks / work items:
// how fast can the per-tile cycle go when the chain S -> softmax -> P.V -> S is broken by the
// second S buffer, as a function of the team size?  clk per tile; tensor work per tile 1,024 clk.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr
//        -I paper_conf_asplos_0017wzlxszh0w26_b200/csrc -I include tools/chain_ds.cu -o tools/chain_ds -lcuda
#include "../paper_conf_asplos_0017wzlxszh0w26_b200/csrc/k_attn.cu"

namespace bat {
void count_launch(int) {}
void set_smem_attr_raw(const void*, int) {}
namespace {

template <int NW, bool RANDOM_DATA>
__global__ void __launch_bounds__(640, 1) chain_ds(long long* out, int iters) {
  constexpr int SL = NW / 4;          // column slices per row
  constexpr int COLS = 128 / SL;      // S columns per thread
  constexpr int NC = COLS / 32;       // 32-column chunks per thread
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t s_full[2], p_full[2];
  __shared__ uint32_t tbase;
  __shared__ int okx[2][4][4][SL];
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();
  if (threadIdx.x == 0) {
    for (int q = 0; q < 2; ++q) {
      ptx::mbar_init(&s_full[q], 1);
      ptx::mbar_init(&p_full[q], NW);
    }
    ptx::fence_mbar_init();
  }
  for (int i = threadIdx.x; i < 131072 / 16; i += blockDim.x) {
    if (RANDOM_DATA) {
      uint32_t w[4];
      for (int j = 0; j < 4; ++j) {
        uint32_t x = (i * 4 + j) * 2654435761u;
        x ^= x >> 13; x *= 0x5bd1e995u; x ^= x >> 15;
        const float a = (float(x & 0xffff) / 32768.0f) - 1.0f, b = (float(x >> 16) / 32768.0f) - 1.0f;
        w[j] = ptx::pack_bf16x2(a, b);
      }
      reinterpret_cast<uint4*>(smem)[i] = make_uint4(w[0], w[1], w[2], w[3]);
    } else {
      reinterpret_cast<uint4*>(smem)[i] = make_uint4(0, 0, 0, 0);
    }
  }
  ptx::fence_proxy_async_smem();
  if (warp == 1) ptx::tmem_alloc(&tbase, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = tbase;
  if (warp == 1) {
    const uint32_t sq = ptx::smem_u32(smem), sk = sq + 65536, sv = sq + 98304;
    constexpr uint32_t IS = ptx::idesc_bf16(128, 128, 0, 0), IP = ptx::idesc_bf16(128, 128, 0, 1);
    auto issue_s = [&](int b) {
#pragma unroll
      for (int kk = 0; kk < 8; ++kk)
        ptx::mma_ss_elect(tmem + b * 128, ptx::desc_sw128(sq + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024),
                          ptx::desc_sw128(sk + (kk >> 2) * 1024 + (kk & 3) * 32, 16, 2048), IS, kk ? 1u : 0u);
      ptx::mma_commit_elect(&s_full[b]);
    };
    // P of slice j (keys [COLS j, COLS j + COLS)) at S columns [COLS j, COLS j + COLS / 2)
    auto issue_pv = [&](int b) {
#pragma unroll
      for (int j = 0; j < SL; ++j)
#pragma unroll
        for (int i = 0; i < COLS / 16; ++i)
          ptx::mma_ts_elect(tmem + 256, tmem + b * 128 + j * COLS + i * 8,
                            ptx::desc_sw128(sv + ((j * COLS + i * 16) / 64) * 16384 + ((j * COLS + i * 16) % 64 / 16) * 4096, 1024, 2048),
                            IP, 1u);
    };
    const long long t0 = clock64();
    issue_s(0);
    issue_s(1);
    for (int i = 0; i < iters; ++i) {
      ptx::mbar_wait(&p_full[i & 1], (i >> 1) & 1);
      ptx::tc_fence_after();
      issue_pv(i & 1);
      if (i + 2 < iters) issue_s(i & 1);
    }
    ptx::mma_commit_elect(&s_full[0]);
    ptx::mbar_wait(&s_full[0], (iters >> 1) & 1);
    const long long t1 = clock64();
    if (lane == 0 && blockIdx.x == 0) out[0] = t1 - t0;
  } else if (warp >= 4 && warp < 4 + NW) {
    const uint32_t sub = warp & 3;
    const int j = (warp - 4) >> 2;  // column slice
    const uint32_t lane_base = (sub * 32) << 16;
    const uint64_t sc2 = pk2(0.01f, 0.01f), nm2 = pk2(-1.0f, -1.0f);
    float acc = 0.0f;
    long long soft = 0;
    for (int i = 0; i < iters; ++i) {
      const int b = i & 1;
      ptx::mbar_wait(&s_full[b], (i >> 1) & 1);
      const long long ts = clock64();
      ptx::tc_fence_after();
      const uint32_t tS = tmem + b * 128 + j * COLS + lane_base;
      uint32_t vis[NC];
#pragma unroll
      for (int c = 0; c < NC; ++c) vis[c] = ~0u;
      float lsum = 0.0f;
      auto agree = [&](bool ok) {
        if (SL == 1) return ok;
        if (lane == 0) okx[b][sub][0][j] = ok;
        ptx::bar_sync(1 + sub, 32 * SL);
        bool all = ok;
#pragma unroll
        for (int o = 0; o < SL; ++o) all = all && okx[b][sub][0][o] != 0;
        return all;
      };
      row_exp_opt<false>(tS, vis, sc2, nm2, INFINITY, lsum, agree);
      acc += lsum;
      ptx::tmem_st_wait();
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&p_full[b]);
      soft += clock64() - ts;
    }
    if (acc == 12345.0f) out[1] = 1;
    if (warp == 4 && lane == 0 && blockIdx.x == 0) out[3] = soft;
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) ptx::tmem_dealloc(tmem, 512);
}

}  // namespace
}  // namespace bat

int main() {
  using namespace bat;
  long long* d;
  cudaMalloc(&d, 8 * sizeof(long long));
  const int iters = 400;
  const size_t smem = 131072;
  auto run = [&](auto kern, const char* name) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    cudaMemset(d, 0, 8 * sizeof(long long));
    kern<<<148, 640, smem>>>(d, iters);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[8];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("%-52s %s  clk per tile %.0f (tensor 1024); softmax S->P %.0f clk\n", name, cudaGetErrorString(e),
           double(h[0]) / iters, double(h[3]) / iters);
  };
  run(chain_ds<4, false>, "double S, 4-warp team (1 thread per row, 128 cols)");
  run(chain_ds<8, false>, "double S, 8-warp team (64 cols per thread)");
  run(chain_ds<16, false>, "double S, 16-warp team (32 cols per thread)");
  run(chain_ds<8, true>, "double S, 8-warp team, random data");
  run(chain_ds<16, true>, "double S, 16-warp team, random data");
  return 0;
}
