// Microbenchmark: cycles per softmax fast-path pass (row_exp_opt of k_attn.cu: TMEM ld of S,
// exp2 with MUFU / polynomial split, bf16 P stored back to TMEM) for the warp layouts the
// attention kernel can use, one 640-thread CTA per SM (all SMs busy).
//   mode 0: one q-tile, rows split in two key halves (8 warps, 64 columns each, pair barrier)
//   mode 1: two q-tiles, split halves (16 warps)
//   mode 2: one q-tile, full rows (4 warps, 128 columns)
//   mode 3: two q-tiles, full rows (8 warps)
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr
//        -I paper_conf_asplos_0017wzlxszh0w26_b200/csrc -I include tools/softmax_rate.cu -o tools/softmax_rate -lcuda
#include "../paper_conf_asplos_0017wzlxszh0w26_b200/csrc/k_attn.cu"

namespace bat {
namespace {

template <int MODE>
__global__ void __launch_bounds__(640, 1) softmax_rate(long long* out, int iters, float* sink) {
  __shared__ uint32_t tbase;
  __shared__ int okx[2][2][4];
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();
  if (warp == 1) ptx::tmem_alloc(&tbase, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = tbase;
  const uint32_t sub = warp & 3;
  const uint32_t lane_base = (sub * 32) << 16;
  if (warp >= 4 && warp < 8) {  // fill S0, S1 (columns 0..255) with scores in [-8, 4)
    uint32_t r[32];
    for (int c = 0; c < 8; ++c) {
#pragma unroll
      for (int i = 0; i < 32; ++i) r[i] = __float_as_uint(-8.0f + 12.0f * float((lane * 37 + i * 11 + c * 5) % 97) / 97.0f);
      ptx::tmem_st32(tmem + lane_base + c * 32, r);
    }
    ptx::tmem_st_wait();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  bool active;
  int q, h;
  if (MODE == 0) { active = (warp >= 4 && warp < 8) || (warp >= 12 && warp < 16); q = 0; h = warp >= 12; }
  else if (MODE == 1) { active = warp >= 4; q = ((warp - 4) >> 2) & 1; h = (warp - 4) >> 3; }
  else if (MODE == 2) { active = warp >= 4 && warp < 8; q = 0; h = 0; }
  else { active = warp >= 4 && warp < 12; q = (warp - 4) >> 2; h = 0; }
  float acc = 0.0f;
  long long t0 = 0, t1 = 0;
  if (active) {
    const uint64_t sc2 = pk2(1.0f, 1.0f), nm2 = pk2(-4.0f, -4.0f);
    t0 = clock64();
    for (int it = 0; it < iters; ++it) {
      float lsum = 0.0f;
      if (MODE <= 1) {
        uint32_t vis[2] = {~0u, ~0u};
        const uint32_t tS = tmem + q * 128 + h * 64 + lane_base;
        auto agree = [&](bool ok) {
          if (lane == 0) okx[q][h][sub] = ok;
          ptx::bar_sync(1 + q * 4 + sub, 64);
          return ok && okx[q][h ^ 1][sub] != 0;
        };
        row_exp_opt<false>(tS, vis, sc2, nm2, INFINITY, lsum, agree);
      } else {
        uint32_t vis[4] = {~0u, ~0u, ~0u, ~0u};
        const uint32_t tS = tmem + q * 128 + lane_base;
        row_exp_opt<false>(tS, vis, sc2, nm2, INFINITY, lsum, [](bool ok) { return ok; });
      }
      ptx::tmem_st_wait();
      acc += lsum;
      // restore the S columns the P overwrote (keeps the pass identical every iteration)
    }
    t1 = clock64();
  }
  if (active && lane == 0 && blockIdx.x == 0) out[warp] = t1 - t0;
  if (acc == 12345.0f) sink[threadIdx.x] = acc;
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) ptx::tmem_dealloc(tmem, 512);
}

}  // namespace
}  // namespace bat

namespace bat { void count_launch(int) {} }
int main() {
  using namespace bat;
  long long* d;
  float* sink;
  cudaMalloc(&d, 32 * sizeof(long long));
  cudaMalloc(&sink, 640 * sizeof(float));
  const int iters = 2000;
  auto run = [&](auto kern, const char* name, int nwarps_cols) {
    cudaMemset(d, 0, 32 * sizeof(long long));
    kern<<<148, 640>>>(d, iters, sink);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[32];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < 32; ++i) mx = h[i] > mx ? h[i] : mx;
    printf("%-34s %s  cycles/pass %.0f  (%d columns per thread)\n", name, cudaGetErrorString(e), double(mx) / iters,
           nwarps_cols);
  };
  run(softmax_rate<0>, "1 q-tile, split halves (8 warps)", 64);
  run(softmax_rate<1>, "2 q-tiles, split halves (16 warps)", 64);
  run(softmax_rate<2>, "1 q-tile, full rows (4 warps)", 128);
  run(softmax_rate<3>, "2 q-tiles, full rows (8 warps)", 128);
  return 0;
}
