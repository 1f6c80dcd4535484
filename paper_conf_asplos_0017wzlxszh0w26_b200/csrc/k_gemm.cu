// tcgen05 GEMM for the dense projections of every layer:
//   C[M,N] = A[M,K] * B[N,K]^T, A = bf16 activations (K-major), B = bf16 weights [N][K]
// with the layer's elementwise work fused into the epilogue:
//   EPI_BF16_BIAS  qkv = a*Wqkv^T + b             (bf16 out)
//   EPI_RESID_F32  h  += o*Wo^T  /  h += act*Wd^T (fp32 residual stream, in place)
//   EPI_SWIGLU     act = silu(x*Wg^T) * (x*Wu^T)  (the B tile holds 128 gate + 128 up rows)
// Persistent, warp-specialised: warp 0 issues TMA (2-D tensor maps, 128-byte swizzle) into a
// 4-stage ring; warp 1 (one thread) issues tcgen05.mma M=128 N=256 K=16 into a double-buffered
// TMEM accumulator (2 x 256 columns); warps 2-5 drain TMEM with tcgen05.ld and run the
// epilogue while the next tile accumulates.  Tiles are rasterised in groups of 8 M-tiles so
// concurrently running CTAs share weight tiles in L2.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "kernels.h"
#include "ptx.cuh"

namespace bat {
namespace {

constexpr int BM = 128, BN = 256, BK = 64, STAGES = 4;
constexpr int A_BYTES = BM * BK * 2;      // 16 KB
constexpr int B_BYTES = BN * BK * 2;      // 32 KB
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int GROUP_M = 8;
constexpr int NUM_THREADS = 192;
constexpr uint32_t IDESC = ptx::idesc_bf16(BM, BN, 0, 0);

struct __align__(8) GemmSmemBars {
  uint64_t full[STAGES], empty[STAGES], tfull[2], tempty[2];
  uint32_t tmem_base;
};

constexpr size_t kGemmSmem = 1024 /*align slack*/ + STAGES * STAGE_BYTES + sizeof(GemmSmemBars);

__device__ __forceinline__ void tile_coords(int t, int num_m, int num_n, int& m, int& n) {
  const int per_group = GROUP_M * num_n;
  const int g = t / per_group;
  const int r = t - g * per_group;
  const int rows = min(GROUP_M, num_m - g * GROUP_M);
  m = g * GROUP_M + r % rows;
  n = r / rows;
}

__device__ __forceinline__ float silu(float x) { return x / (1.0f + __expf(-x)); }

template <int EPI>
__global__ void __launch_bounds__(NUM_THREADS, 1)
gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
               GemmParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  GemmSmemBars* bars = reinterpret_cast<GemmSmemBars*>(smem + STAGES * STAGE_BYTES);
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();

  const int out_bn = (EPI == EPI_SWIGLU) ? BN / 2 : BN;  // output columns per tile
  const int num_m = (p.M + BM - 1) / BM;
  const int num_n = (p.N + out_bn - 1) / out_bn;
  const int num_tiles = num_m * num_n;
  const int num_kb = (p.K + BK - 1) / BK;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < STAGES; ++s) {
      ptx::mbar_init(&bars->full[s], 1);
      ptx::mbar_init(&bars->empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&bars->tfull[a], 1);
      ptx::mbar_init(&bars->tempty[a], 4);
    }
    ptx::fence_mbar_init();
    ptx::prefetch_tmap(&tmA);
    ptx::prefetch_tmap(&tmB);
  }
  if (warp == 1) ptx::tmem_alloc(&bars->tmem_base, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = bars->tmem_base;

  if (warp == 0) {
    if (lane == 0) {  // ---------------- TMA producer
      int stage = 0;
      uint32_t phase = 0;
      for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
        int m, n;
        tile_coords(t, num_m, num_n, m, n);
        for (int kb = 0; kb < num_kb; ++kb) {
          ptx::mbar_wait(&bars->empty[stage], phase ^ 1);
          uint8_t* sa = smem + stage * STAGE_BYTES;
          uint8_t* sb = sa + A_BYTES;
          ptx::mbar_expect_tx(&bars->full[stage], STAGE_BYTES);
          ptx::tma_load_2d(sa, &tmA, kb * BK, m * BM, &bars->full[stage]);
          if (EPI == EPI_SWIGLU) {
            ptx::tma_load_2d(sb, &tmB, kb * BK, n * (BN / 2), &bars->full[stage]);
            ptx::tma_load_2d(sb + B_BYTES / 2, &tmB, kb * BK, p.up_row0 + n * (BN / 2), &bars->full[stage]);
          } else {
            ptx::tma_load_2d(sb, &tmB, kb * BK, n * BN, &bars->full[stage]);
          }
          if (++stage == STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ---------------- MMA issuer (single thread)
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
        ptx::mbar_wait(&bars->tempty[acc], acc_phase ^ 1);
        ptx::tc_fence_after();
        const uint32_t d_tmem = tmem + acc * BN;
        for (int kb = 0; kb < num_kb; ++kb) {
          ptx::mbar_wait(&bars->full[stage], phase);
          ptx::tc_fence_after();
          const uint32_t sa = ptx::smem_u32(smem + stage * STAGE_BYTES);
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            uint64_t da = ptx::desc_sw128(sa + kk * 32, 16, 1024);
            uint64_t db = ptx::desc_sw128(sb + kk * 32, 16, 1024);
            ptx::mma_ss(d_tmem, da, db, IDESC, (kb | kk) ? 1u : 0u);
          }
          ptx::mma_commit(&bars->empty[stage]);
          if (++stage == STAGES) { stage = 0; phase ^= 1; }
        }
        ptx::mma_commit(&bars->tfull[acc]);
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {  // ------------------------------ epilogue warps 2..5
    const uint32_t sub = warp & 3;  // TMEM sub-partition this warp may access
    const int row_in_tile = sub * 32 + lane;
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
      int m, n;
      tile_coords(t, num_m, num_n, m, n);
      ptx::mbar_wait(&bars->tfull[acc], acc_phase);
      ptx::tc_fence_after();
      const uint32_t tbase = tmem + ((sub * 32) << 16) + acc * BN;
      const int row = m * BM + row_in_tile;
      const bool row_ok = row < p.M;
      if (EPI == EPI_SWIGLU) {
#pragma unroll 1
        for (int c = 0; c < BN / 2; c += 32) {
          uint32_t g[32], u[32];
          ptx::tmem_ld32(tbase + c, g);
          ptx::tmem_ld32(tbase + BN / 2 + c, u);
          ptx::tmem_ld_wait();
          const int col = n * (BN / 2) + c;
          if (row_ok && col < p.N) {
            uint32_t pk[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) {
              float g0 = __uint_as_float(g[2 * i]), g1 = __uint_as_float(g[2 * i + 1]);
              float u0 = __uint_as_float(u[2 * i]), u1 = __uint_as_float(u[2 * i + 1]);
              pk[i] = ptx::pack_bf16x2(silu(g0) * u0, silu(g1) * u1);
            }
            uint4* dst = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(p.out) + size_t(row) * p.ldo + col);
#pragma unroll
            for (int i = 0; i < 4; ++i) dst[i] = make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
          }
        }
      } else {
#pragma unroll 1
        for (int c = 0; c < BN; c += 32) {
          uint32_t r[32];
          ptx::tmem_ld32(tbase + c, r);
          ptx::tmem_ld_wait();
          const int col = n * BN + c;
          if (row_ok && col < p.N) {
            if (EPI == EPI_RESID_F32) {
              float4* dst = reinterpret_cast<float4*>(static_cast<float*>(p.out) + size_t(row) * p.ldo + col);
#pragma unroll
              for (int i = 0; i < 8; ++i) {
                float4 h = dst[i];
                h.x += __uint_as_float(r[4 * i]);
                h.y += __uint_as_float(r[4 * i + 1]);
                h.z += __uint_as_float(r[4 * i + 2]);
                h.w += __uint_as_float(r[4 * i + 3]);
                dst[i] = h;
              }
            } else {
              uint32_t pk[16];
#pragma unroll
              for (int i = 0; i < 16; ++i) {
                float v0 = __uint_as_float(r[2 * i]), v1 = __uint_as_float(r[2 * i + 1]);
                if (EPI == EPI_BF16_BIAS) {
                  v0 += __bfloat162float(p.bias[col + 2 * i]);
                  v1 += __bfloat162float(p.bias[col + 2 * i + 1]);
                }
                pk[i] = ptx::pack_bf16x2(v0, v1);
              }
              uint4* dst = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(p.out) + size_t(row) * p.ldo + col);
#pragma unroll
              for (int i = 0; i < 4; ++i) dst[i] = make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
            }
          }
        }
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&bars->tempty[acc]);
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) ptx::tmem_dealloc(tmem, 512);
}

}  // namespace

size_t gemm_smem_bytes() { return kGemmSmem; }

void launch_gemm(int epi, const CUtensorMap& tmA, const CUtensorMap& tmB, const GemmParams& p,
                 int num_sms, cudaStream_t stream) {
  const int out_bn = (epi == EPI_SWIGLU) ? BN / 2 : BN;
  const int tiles = ((p.M + BM - 1) / BM) * ((p.N + out_bn - 1) / out_bn);
  const int grid = tiles < num_sms ? tiles : num_sms;
  if (grid <= 0) return;
  switch (epi) {
#define BAT_GEMM_CASE(E)                                                                        \
  case E: {                                                                                     \
    static bool attr = false;                                                                   \
    if (!attr) {                                                                                \
      cudaFuncSetAttribute(gemm_tc_kernel<E>, cudaFuncAttributeMaxDynamicSharedMemorySize,     \
                           static_cast<int>(kGemmSmem));                                        \
      attr = true;                                                                              \
    }                                                                                           \
    gemm_tc_kernel<E><<<grid, NUM_THREADS, kGemmSmem, stream>>>(tmA, tmB, p);                  \
    break;                                                                                      \
  }
    BAT_GEMM_CASE(EPI_BF16)
    BAT_GEMM_CASE(EPI_BF16_BIAS)
    BAT_GEMM_CASE(EPI_RESID_F32)
    BAT_GEMM_CASE(EPI_SWIGLU)
#undef BAT_GEMM_CASE
  }
  count_launch();
}

}  // namespace bat
