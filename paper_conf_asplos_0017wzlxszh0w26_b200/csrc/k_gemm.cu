// tcgen05 GEMM for the dense projections of every layer:
//   C[M,N] = A[M,K] * B[N,K]^T, A = bf16 activations (K-major), B = bf16 weights [N][K]
// with the layer's elementwise work fused into the epilogue, written back through 128B-swizzled
// shared-memory staging and TMA (tile store, or TMA reduce-add for the fp32 residual stream):
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

constexpr int STG_BYTES = 4096;  // per-warp epilogue staging buffer: [32 rows][128 B], 128B-swizzled
constexpr int STG_OFF = STAGES * STAGE_BYTES;
constexpr size_t kGemmSmem = 1024 /*align slack*/ + STAGES * STAGE_BYTES + 4 * 2 * STG_BYTES + sizeof(GemmSmemBars);

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
               const __grid_constant__ CUtensorMap tmC, GemmParams p) {
  extern __shared__ uint8_t smem_raw[];
  // 1 KB-align by offsetting the __shared__ array itself (keeps the shared address space, so
  // the compiler emits LDS/STS rather than generic loads and stores)
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  GemmSmemBars* bars = reinterpret_cast<GemmSmemBars*>(smem + STG_OFF + 4 * 2 * STG_BYTES);
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
    ptx::prefetch_tmap(&tmC);
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
    // TMEM -> registers -> (bias / SwiGLU) -> 128B-swizzled smem staging -> TMA store (bf16)
    // or TMA reduce-add (fp32 residual).  Coalesced, asynchronous, double-buffered per warp.
    const uint32_t sub = warp & 3;  // TMEM sub-partition this warp may access
    uint8_t* stg = smem + STG_OFF + (warp - 2) * 2 * STG_BYTES;
    int sbuf = 0;
    auto stage_row = [&](uint8_t* buf, int chunk16, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
      ptx::st_shared_v4(buf + lane * 128 + ((chunk16 ^ (lane & 7)) << 4), a, b, c, d);
    };
    auto next_buf = [&]() -> uint8_t* {
      uint8_t* buf = stg + sbuf * STG_BYTES;
      if (lane == 0) ptx::bulk_wait_read<1>();  // the group that last used this buffer is done
      __syncwarp();
      return buf;
    };
    auto flush = [&](uint8_t* buf, int col, int row) {
      ptx::fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) {
        if (EPI == EPI_RESID_F32) ptx::tma_reduce_add_2d(&tmC, buf, col, row);
        else ptx::tma_store_2d(&tmC, buf, col, row);
        ptx::bulk_commit();
      }
      sbuf ^= 1;
    };
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
      int m, n;
      tile_coords(t, num_m, num_n, m, n);
      ptx::mbar_wait(&bars->tfull[acc], acc_phase);
      ptx::tc_fence_after();
      const uint32_t tbase = tmem + ((sub * 32) << 16) + acc * BN;
      const int row0 = m * BM + sub * 32;
      if constexpr (EPI == EPI_SWIGLU) {
#pragma unroll 1
        for (int c = 0; c < BN / 2; c += 64) {  // 64 output columns per staging buffer
          uint8_t* buf = next_buf();
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            uint32_t g[32], u[32];
            ptx::tmem_ld32(tbase + c + 32 * h, g);
            ptx::tmem_ld32(tbase + BN / 2 + c + 32 * h, u);
            ptx::tmem_ld_wait();
            uint32_t pk[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) {
              float g0 = __uint_as_float(g[2 * i]), g1 = __uint_as_float(g[2 * i + 1]);
              float u0 = __uint_as_float(u[2 * i]), u1 = __uint_as_float(u[2 * i + 1]);
              pk[i] = ptx::pack_bf16x2(silu(g0) * u0, silu(g1) * u1);
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) stage_row(buf, 4 * h + j, pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
          }
          flush(buf, n * (BN / 2) + c, row0);
        }
      } else if constexpr (EPI == EPI_RESID_F32) {
#pragma unroll 1
        for (int c = 0; c < BN; c += 32) {  // 32 fp32 columns per staging buffer
          uint8_t* buf = next_buf();
          uint32_t r[32];
          ptx::tmem_ld32(tbase + c, r);
          ptx::tmem_ld_wait();
#pragma unroll
          for (int j = 0; j < 8; ++j) stage_row(buf, j, r[4 * j], r[4 * j + 1], r[4 * j + 2], r[4 * j + 3]);
          flush(buf, n * BN + c, row0);
        }
      } else {
#pragma unroll 1
        for (int c = 0; c < BN; c += 64) {  // 64 bf16 columns per staging buffer
          uint8_t* buf = next_buf();
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            uint32_t r[32];
            ptx::tmem_ld32(tbase + c + 32 * h, r);
            ptx::tmem_ld_wait();
            const int col = n * BN + c + 32 * h;
            uint32_t pk[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) {
              float v0 = __uint_as_float(r[2 * i]), v1 = __uint_as_float(r[2 * i + 1]);
              if (EPI == EPI_BF16_BIAS && col + 2 * i + 1 < p.N) {
                v0 += __bfloat162float(p.bias[col + 2 * i]);
                v1 += __bfloat162float(p.bias[col + 2 * i + 1]);
              }
              pk[i] = ptx::pack_bf16x2(v0, v1);
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) stage_row(buf, 4 * h + j, pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
          }
          flush(buf, n * BN + c, row0);
        }
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&bars->tempty[acc]);
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
    }
    if (lane == 0) ptx::bulk_wait<0>();
    __syncwarp();
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) ptx::tmem_dealloc(tmem, 512);
}

}  // namespace

size_t gemm_smem_bytes() { return kGemmSmem; }

void launch_gemm(int epi, const CUtensorMap& tmA, const CUtensorMap& tmB, const CUtensorMap& tmC,
                 const GemmParams& p, int num_sms, cudaStream_t stream) {
  const int out_bn = (epi == EPI_SWIGLU) ? BN / 2 : BN;
  const int tiles = ((p.M + BM - 1) / BM) * ((p.N + out_bn - 1) / out_bn);
  const int grid = tiles < num_sms ? tiles : num_sms;
  if (grid <= 0) return;
  auto launch = [&](auto kern) {
    static const void* attr_done[16] = {nullptr};  // kernels whose smem attribute is set
    bool found = false;
    for (const void* f : attr_done) found |= (f == reinterpret_cast<const void*>(kern));
    if (!found) {
      cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(kGemmSmem));
      for (auto& f : attr_done)
        if (!f) { f = reinterpret_cast<const void*>(kern); break; }
    }
    kern<<<grid, NUM_THREADS, kGemmSmem, stream>>>(tmA, tmB, tmC, p);
  };
  switch (epi) {
    case EPI_BF16: launch(gemm_tc_kernel<EPI_BF16>); break;
    case EPI_BF16_BIAS: launch(gemm_tc_kernel<EPI_BF16_BIAS>); break;
    case EPI_RESID_F32: launch(gemm_tc_kernel<EPI_RESID_F32>); break;
    case EPI_SWIGLU: launch(gemm_tc_kernel<EPI_SWIGLU>); break;
  }
  count_launch();
}

}  // namespace bat
