// Microbenchmark: does softmax TMEM traffic (tcgen05.ld of S / tcgen05.st of P by other warps)
// slow the tensor pipe?  One thread issues the attention kernel's per-q-tile MMA pattern
// (S = Q K^T: 8 SS N=128 MMAs into S0; O += P V: 8 TS N=128 MMAs reading P from S0) in a loop
// while the softmax warps run row_exp_opt on S1 (a disjoint TMEM region).  One CTA per SM.
//   mode 0: MMA only                       mode 1: MMA + 4 softmax warps (full rows)
//   mode 2: MMA + 8 softmax warps (halves)  mode 3: MMA + 4 warps doing only LDTM/STTM
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr
//        -I paper_conf_asplos_0017wzlxszh0w26_b200/csrc -I include tools/mma_contention.cu -o tools/mma_contention -lcuda
#include "../paper_conf_asplos_0017wzlxszh0w26_b200/csrc/k_attn.cu"

namespace bat {
void count_launch(int) {}
namespace {

template <int MODE>
__global__ void __launch_bounds__(640, 1) contention(long long* out, int iters, float* sink) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  __shared__ int okx[2][2][4];
  __shared__ volatile int stop;
  __shared__ volatile int go[4];
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
    stop = 0;
  }
  if (warp == 1) ptx::tmem_alloc(&tbase, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = tbase;
  const uint32_t sub = warp & 3;
  const uint32_t lane_base = (sub * 32) << 16;
  long long passes = 0;
  float acc = 0.0f;
  if (warp == 1 && lane == 0) {
    const uint64_t dq = ptx::desc_sw128(ptx::smem_u32(smem), 16, 1024);
    const uint64_t dk = ptx::desc_sw128(ptx::smem_u32(smem + 32768), 16, 1024);
    const uint64_t dv = ptx::desc_sw128(ptx::smem_u32(smem + 65536), 16384, 1024);
    constexpr uint32_t is = ptx::idesc_bf16(128, 128, 0, 0), ip = ptx::idesc_bf16(128, 128, 0, 1);
    const long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
      for (int kk = 0; kk < 8; ++kk) {
        const uint32_t off = (kk >> 2) * 1024 + (kk & 3) * 2;  // desc units of 16 B
        ptx::mma_ss(tmem, dq + off, dk + off, is, kk ? 1u : 0u);
      }
#pragma unroll
      for (int kk = 0; kk < 8; ++kk) ptx::mma_ts(tmem + 256, tmem + kk * 8, dv + kk * 128, ip, 1u);
    }
    ptx::mma_commit(&bar);
    ptx::mbar_wait(&bar, 0);
    const long long t1 = clock64();
    stop = 1;
    if (blockIdx.x == 0) out[0] = t1 - t0;
  } else if (warp >= 4) {
    bool active;
    int h = 0;
    if (MODE == 1 || MODE == 3) active = warp < 8;
    else if (MODE == 2) { active = warp < 8 || (warp >= 12 && warp < 16); h = warp >= 12; }
    else active = false;
    if (active) {
      const uint64_t sc2 = pk2(1.0f, 1.0f), nm2 = pk2(-4.0f, -4.0f);
      bool more = true;
      while (more) {
        float lsum = 0.0f;
        if (MODE == 2) {
          uint32_t vis[2] = {~0u, ~0u};
          auto agree = [&](bool ok) {
            if (lane == 0) okx[0][h][sub] = ok;
            ptx::bar_sync(1 + sub, 64);
            return ok && okx[0][h ^ 1][sub] != 0;
          };
          row_exp_opt<false>(tmem + 128 + h * 64 + lane_base, vis, sc2, nm2, INFINITY, lsum, agree);
        } else if (MODE == 1) {
          uint32_t vis[4] = {~0u, ~0u, ~0u, ~0u};
          row_exp_opt<false>(tmem + 128 + lane_base, vis, sc2, nm2, INFINITY, lsum, [](bool ok) { return ok; });
        } else {
          uint32_t r[32];
#pragma unroll
          for (int c = 0; c < 4; ++c) {
            ptx::tmem_ld32(tmem + 128 + lane_base + c * 32, r);
            ptx::tmem_ld_wait();
            lsum += __uint_as_float(r[lane & 31]);
          }
#pragma unroll
          for (int c = 0; c < 2; ++c) ptx::tmem_st32(tmem + 128 + lane_base + c * 32, r);
        }
        ptx::tmem_st_wait();
        acc += lsum;
        ++passes;
        if (MODE == 2) {  // the pair leaves together: h = 0 decides
          if (h == 0 && lane == 0) go[sub] = !stop;
          ptx::bar_sync(1 + sub, 64);
          more = go[sub] != 0;
        } else {
          more = !stop;
        }
      }
    }
    if (active && lane == 0 && blockIdx.x == 0 && warp == 4) out[1] = passes;
  }
  if (acc == 12345.0f) sink[threadIdx.x] = acc;
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) ptx::tmem_dealloc(tmem, 512);
}

}  // namespace
}  // namespace bat

int main() {
  using namespace bat;
  long long* d;
  float* sink;
  cudaMalloc(&d, 4 * sizeof(long long));
  cudaMalloc(&sink, 640 * sizeof(float));
  const int iters = 4000;
  auto run = [&](auto kern, const char* name) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000);
    cudaMemset(d, 0, 4 * sizeof(long long));
    kern<<<148, 640, 100000>>>(d, iters, sink);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[4];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("%-36s %s  MMA cycles per q-tile-tile %.0f (ideal 1024); softmax passes per q-tile-tile %.2f\n", name,
           cudaGetErrorString(e), double(h[0]) / iters, double(h[1]) / iters);
  };
  run(contention<0>, "MMA only");
  run(contention<1>, "MMA + softmax 4 warps (full rows)");
  run(contention<2>, "MMA + softmax 8 warps (halves)");
  run(contention<3>, "MMA + 4 warps LDTM/STTM only");
  return 0;
}
