// tcgen05 GEMM for the dense projections of every layer:
//   C[M,N] = A[M,K] * B[N,K]^T, A = bf16 activations (K-major), B = bf16 weights [N][K]
// with the layer's elementwise work fused into the epilogue, written back through 128B-swizzled
// shared-memory staging and TMA (tile store, or TMA reduce-add for the fp32 residual stream):
//   EPI_BF16_BIAS  qkv = a*Wqkv^T + b             (bf16 out)
//   EPI_RESID_F32  h  += o*Wo^T  /  h += act*Wd^T (fp32 residual stream, in place)
//   EPI_SWIGLU     act = silu(x*Wg^T) * (x*Wu^T)  (the B tile holds 128 gate + 128 up rows)
//
// Two persistent, warp-specialised kernels share the epilogue:
//  * gemm2_tc_kernel (M >= 256): a CTA PAIR (cluster of 2, tcgen05 cta_group::2) computes a
//    256 x 256 tile — each CTA stages its 128 rows of A and its 128 rows of B (half of N) per
//    64-deep k-block (32 KB, 6-stage ring), the pair leader's single thread issues
//    M=256 N=256 K=16 MMAs that read both CTAs' shared memory, and each CTA accumulates its 128
//    rows x 256 columns in its own TMEM (2 x 256 columns, double-buffered).  Per SM this halves
//    the B traffic from L2 and cuts the tensor core's shared-memory reads from 96 to 64 B/clk
//    against the 1-CTA 128 x 256 tile.
//  * gemm_tc_kernel (small M, e.g. the last layer's discriminant rows): one CTA per 128 x 256
//    tile, M=128 N=256 K=16 MMAs, 4-stage ring.
// In both, warp 0 issues TMA (2-D tensor maps, 128-byte swizzle), warp 1 issues the MMAs, and
// warps 2-5 drain TMEM with tcgen05.ld and run the epilogue while the next tile accumulates.
// Tiles are rasterised in groups of M-tiles (GROUP_M; 32 for SwiGLU) so concurrently running CTAs
// share operand tiles in L2.
#include <cuda.h>
#include <cstdlib>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "kernels.h"
#include "ptx.cuh"

namespace bat {
namespace {

constexpr int BN = 256, BK = 64, BROWS = 128;  // B is loaded in 128-row boxes
constexpr int A_BYTES = 128 * BK * 2;           // 16 KB: 128 rows of A per CTA
// default rasterisation group (M-tiles) of the QKV / O / down GEMMs: 1 = the N-tiles of one M-tile
// run back to back (down GEMM DRAM reads 1.43 GB at 8, 1.27 at 4, 1.12 at 1, 2.26 at 32 per launch,
// profiles/r1_gemm_raster.txt); BAT_GEMM_GROUP_M / _SWIGLU override
constexpr int GROUP_M = 1;
constexpr int GROUP_M_SWIGLU = 32;
constexpr int NUM_THREADS = 192;
constexpr int STG_BYTES = 4096;  // per-warp epilogue staging buffer: [32 rows][128 B], 128B-swizzled

// 1-CTA kernel: 128 x 256 tiles
constexpr int STAGES1 = 4;
constexpr int STAGE1_BYTES = A_BYTES + BN * BK * 2;  // 48 KB
constexpr int STG1_OFF = STAGES1 * STAGE1_BYTES;
// CTA-pair kernel: 256 x 256 tiles, each CTA 128 rows of A + 128 rows of B per stage
constexpr int STAGES2 = 6;
constexpr int STAGE2_BYTES = A_BYTES + BROWS * BK * 2;  // 32 KB
constexpr int STG2_OFF = STAGES2 * STAGE2_BYTES;

struct __align__(8) GemmSmemBars {
  uint64_t full[8], empty[8], tfull[2], tempty[2];
  uint32_t tmem_base;
};
constexpr size_t kGemmSmem1 = 1024 /*align slack*/ + STG1_OFF + 4 * 2 * STG_BYTES + sizeof(GemmSmemBars);
constexpr size_t kGemmSmem2 = 1024 /*align slack*/ + STG2_OFF + 4 * 2 * STG_BYTES + sizeof(GemmSmemBars);
static_assert(kGemmSmem1 <= 232448 && kGemmSmem2 <= 232448, "GEMM shared memory");

__device__ __forceinline__ void tile_coords(int t, int num_m, int num_n, int group_m, int& m, int& n) {
  const int per_group = group_m * num_n;
  const int g = t / per_group;
  const int r = t - g * per_group;
  const int rows = min(group_m, num_m - g * group_m);
  m = g * group_m + r % rows;
  n = r / rows;
}

__device__ __forceinline__ float silu(float x) { return x / (1.0f + __expf(-x)); }

// Epilogue of one accumulator (this warp's 32 TMEM lanes = output rows row0 .. row0 + 31):
// TMEM -> registers -> (bias / SwiGLU) -> 128B-swizzled smem staging -> TMA store (bf16) or
// TMA reduce-add (fp32 residual).  Coalesced, asynchronous, double-buffered per warp.
template <int EPI>
struct Epilogue {
  const CUtensorMap* tmC;
  const GemmParams* p;
  uint8_t* stg;  // this warp's 2 staging buffers
  uint32_t lane;
  int sbuf = 0;

  __device__ __forceinline__ void stage_row(uint8_t* buf, int chunk16, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    ptx::st_shared_v4(buf + lane * 128 + ((chunk16 ^ (lane & 7)) << 4), a, b, c, d);
  }
  __device__ __forceinline__ uint8_t* next_buf() {
    uint8_t* buf = stg + sbuf * STG_BYTES;
    if (lane == 0) ptx::bulk_wait_read<1>();  // the group that last used this buffer is done
    __syncwarp();
    return buf;
  }
  __device__ __forceinline__ void flush(uint8_t* buf, int col, int row) {
    ptx::fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
      if (EPI == EPI_RESID_F32) ptx::tma_reduce_add_2d(tmC, buf, col, row);
      else if (EPI == EPI_PART_F32) ptx::tma_store_2d(tmC, buf, col, row);
      else if (p->hints & 2) ptx::tma_store_2d_hint(tmC, buf, col, row, ptx::policy_evict_first());
      else ptx::tma_store_2d(tmC, buf, col, row);
      ptx::bulk_commit();
    }
    sbuf ^= 1;
  }
  // tbase: TMEM address of this warp's lanes, column 0 of the accumulator; n: output N-tile
  __device__ __forceinline__ void run(uint32_t tbase, int n, int row0) {
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
    } else if constexpr (EPI == EPI_RESID_F32 || EPI == EPI_PART_F32) {
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
            if (EPI == EPI_BF16_BIAS && col + 2 * i + 1 < p->N) {
              v0 += __bfloat162float(p->bias[col + 2 * i]);
              v1 += __bfloat162float(p->bias[col + 2 * i + 1]);
            }
            pk[i] = ptx::pack_bf16x2(v0, v1);
          }
#pragma unroll
          for (int j = 0; j < 4; ++j) stage_row(buf, 4 * h + j, pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
        }
        flush(buf, n * BN + c, row0);
      }
    }
  }
};

// B rows of output N-tile n, 128-row half h: SwiGLU tiles take 128 gate rows then 128 up rows
template <int EPI>
__device__ __forceinline__ int b_row(const GemmParams& p, int n, int h) {
  return (EPI == EPI_SWIGLU) ? (h ? p.up_row0 : 0) + n * (BN / 2) : n * BN + h * BROWS;
}

// ------------------------------------------------------------------- 1-CTA, 128 x 256 tiles
template <int EPI>
__global__ void __launch_bounds__(NUM_THREADS, 1)
gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
               const __grid_constant__ CUtensorMap tmC, GemmParams p) {
  extern __shared__ uint8_t smem_raw[];
  // 1 KB-align by offsetting the __shared__ array itself (keeps the shared address space, so
  // the compiler emits LDS/STS rather than generic loads and stores)
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  GemmSmemBars* bars = reinterpret_cast<GemmSmemBars*>(smem + STG1_OFF + 4 * 2 * STG_BYTES);
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();
  constexpr uint32_t IDESC = ptx::idesc_bf16(128, BN, 0, 0);

  const int out_bn = (EPI == EPI_SWIGLU) ? BN / 2 : BN;  // output columns per tile
  const int num_m = (p.M + 127) / 128;
  const int num_n = (p.N + out_bn - 1) / out_bn;
  const int num_tiles = num_m * num_n;
  const int num_kb = (p.K + BK - 1) / BK;
  const int ksplit = EPI == EPI_PART_F32 ? p.ksplit : 1;
  const int num_work = num_tiles * ksplit;  // (K slice, tile) work units, slice-major

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < STAGES1; ++s) {
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
      const uint64_t pol_b = ptx::policy_evict_last();
      int stage = 0;
      uint32_t phase = 0;
      for (int t = blockIdx.x; t < num_work; t += gridDim.x) {
        int m, n;
        tile_coords(t % num_tiles, num_m, num_n, p.group_m, m, n);
        const int ks = t / num_tiles;
        for (int kb = ks * num_kb / ksplit; kb < (ks + 1) * num_kb / ksplit; ++kb) {
          ptx::mbar_wait(&bars->empty[stage], phase ^ 1);
          uint8_t* sa = smem + stage * STAGE1_BYTES;
          uint8_t* sb = sa + A_BYTES;
          ptx::mbar_expect_tx(&bars->full[stage], STAGE1_BYTES);
          ptx::tma_load_2d(sa, &tmA, kb * BK, m * 128, &bars->full[stage]);
          if (p.hints & 1) {
            ptx::tma_load_2d_hint(sb, &tmB, kb * BK, b_row<EPI>(p, n, 0), &bars->full[stage], pol_b);
            ptx::tma_load_2d_hint(sb + BROWS * BK * 2, &tmB, kb * BK, b_row<EPI>(p, n, 1), &bars->full[stage], pol_b);
          } else {
            ptx::tma_load_2d(sb, &tmB, kb * BK, b_row<EPI>(p, n, 0), &bars->full[stage]);
            ptx::tma_load_2d(sb + BROWS * BK * 2, &tmB, kb * BK, b_row<EPI>(p, n, 1), &bars->full[stage]);
          }
          if (++stage == STAGES1) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ---------------- MMA issuer (single thread)
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int t = blockIdx.x; t < num_work; t += gridDim.x) {
        ptx::mbar_wait(&bars->tempty[acc], acc_phase ^ 1);
        ptx::tc_fence_after();
        const uint32_t d_tmem = tmem + acc * BN;
        const int ks = t / num_tiles, kb0 = ks * num_kb / ksplit;
        for (int kb = kb0; kb < (ks + 1) * num_kb / ksplit; ++kb) {
          ptx::mbar_wait(&bars->full[stage], phase);
          ptx::tc_fence_after();
          const uint32_t sa = ptx::smem_u32(smem + stage * STAGE1_BYTES);
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            uint64_t da = ptx::desc_sw128(sa + kk * 32, 16, 1024);
            uint64_t db = ptx::desc_sw128(sb + kk * 32, 16, 1024);
            ptx::mma_ss(d_tmem, da, db, IDESC, (kb != kb0 || kk) ? 1u : 0u);
          }
          ptx::mma_commit(&bars->empty[stage]);
          if (++stage == STAGES1) { stage = 0; phase ^= 1; }
        }
        ptx::mma_commit(&bars->tfull[acc]);
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {  // ------------------------------ epilogue warps 2..5
    const uint32_t sub = warp & 3;  // TMEM sub-partition this warp may access
    Epilogue<EPI> epi{&tmC, &p, smem + STG1_OFF + (warp - 2) * 2 * STG_BYTES, lane};
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int t = blockIdx.x; t < num_work; t += gridDim.x) {
      int m, n;
      tile_coords(t % num_tiles, num_m, num_n, p.group_m, m, n);
      const int slab = EPI == EPI_PART_F32 ? (t / num_tiles) * p.mpad : 0;
      ptx::mbar_wait(&bars->tfull[acc], acc_phase);
      ptx::tc_fence_after();
      epi.run(tmem + ((sub * 32) << 16) + acc * BN, n, slab + m * 128 + sub * 32);
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

// ------------------------------------------------------------ CTA pair, 256 x 256 tiles
template <int EPI>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(NUM_THREADS, 1)
gemm2_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                const __grid_constant__ CUtensorMap tmC, GemmParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  GemmSmemBars* bars = reinterpret_cast<GemmSmemBars*>(smem + STG2_OFF + 4 * 2 * STG_BYTES);
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();
  const uint32_t rank = ptx::cluster_ctarank();  // 0 = leader (issues the pair MMAs)
  constexpr uint32_t IDESC = ptx::idesc_bf16(256, BN, 0, 0);

  const int out_bn = (EPI == EPI_SWIGLU) ? BN / 2 : BN;
  const int num_m = (p.M + 255) / 256;
  const int num_n = (p.N + out_bn - 1) / out_bn;
  const int num_tiles = num_m * num_n;
  const int num_kb = (p.K + BK - 1) / BK;
  const int ksplit = EPI == EPI_PART_F32 ? p.ksplit : 1;
  const int num_work = num_tiles * ksplit;
  const int pair = blockIdx.x >> 1, n_pairs = gridDim.x >> 1;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < STAGES2; ++s) {
      ptx::mbar_init(&bars->full[s], 1);   // leader: its own arrive.expect_tx (both CTAs' bytes)
      ptx::mbar_init(&bars->empty[s], 1);  // pair commit (multicast to both CTAs)
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&bars->tfull[a], 1);   // pair commit
      ptx::mbar_init(&bars->tempty[a], 8);  // leader: the 4 epilogue warps of both CTAs
    }
    ptx::fence_mbar_init();
    ptx::prefetch_tmap(&tmA);
    ptx::prefetch_tmap(&tmB);
    ptx::prefetch_tmap(&tmC);
  }
  if (warp == 1) ptx::tmem_alloc2(&bars->tmem_base, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::cluster_sync();  // both CTAs' barriers exist before any remote signal
  ptx::tc_fence_after();
  const uint32_t tmem = bars->tmem_base;

  if (warp == 0) {
    if (lane == 0) {  // ---------------- TMA producer (both CTAs): my 128 rows of A and of B
      int stage = 0;
      uint32_t phase = 0;
      for (int t = pair; t < num_work; t += n_pairs) {
        int m, n;
        tile_coords(t % num_tiles, num_m, num_n, p.group_m, m, n);
        const int ks = t / num_tiles;
        for (int kb = ks * num_kb / ksplit; kb < (ks + 1) * num_kb / ksplit; ++kb) {
          ptx::mbar_wait(&bars->empty[stage], phase ^ 1);
          uint8_t* sa = smem + stage * STAGE2_BYTES;
          uint8_t* sb = sa + A_BYTES;
          const uint32_t full_leader = ptx::mapa(ptx::smem_u32(&bars->full[stage]), 0);
          if (rank == 0) ptx::mbar_expect_tx(&bars->full[stage], 2 * STAGE2_BYTES);
          ptx::tma_load_2d_pair(sa, &tmA, kb * BK, m * 256 + int(rank) * 128, full_leader);
          ptx::tma_load_2d_pair(sb, &tmB, kb * BK, b_row<EPI>(p, n, int(rank)), full_leader);
          if (++stage == STAGES2) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {  // ---------------- pair MMA issuer (leader, single thread)
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int t = pair; t < num_work; t += n_pairs) {
        ptx::mbar_wait(&bars->tempty[acc], acc_phase ^ 1);
        ptx::tc_fence_after();
        const uint32_t d_tmem = tmem + acc * BN;
        const int ks = t / num_tiles, kb0 = ks * num_kb / ksplit;
        for (int kb = kb0; kb < (ks + 1) * num_kb / ksplit; ++kb) {
          ptx::mbar_wait(&bars->full[stage], phase);
          ptx::tc_fence_after();
          const uint32_t sa = ptx::smem_u32(smem + stage * STAGE2_BYTES);
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            uint64_t da = ptx::desc_sw128(sa + kk * 32, 16, 1024);
            uint64_t db = ptx::desc_sw128(sb + kk * 32, 16, 1024);
            ptx::mma2_ss(d_tmem, da, db, IDESC, (kb != kb0 || kk) ? 1u : 0u);
          }
          ptx::mma2_commit(&bars->empty[stage], 3);
          if (++stage == STAGES2) { stage = 0; phase ^= 1; }
        }
        ptx::mma2_commit(&bars->tfull[acc], 3);
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {  // ------------------------------ epilogue warps 2..5 (both CTAs): my 128 rows
    const uint32_t sub = warp & 3;
    Epilogue<EPI> epi{&tmC, &p, smem + STG2_OFF + (warp - 2) * 2 * STG_BYTES, lane};
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int t = pair; t < num_work; t += n_pairs) {
      int m, n;
      tile_coords(t % num_tiles, num_m, num_n, p.group_m, m, n);
      const int slab = EPI == EPI_PART_F32 ? (t / num_tiles) * p.mpad : 0;
      ptx::mbar_wait(&bars->tfull[acc], acc_phase);
      ptx::tc_fence_after();
      epi.run(tmem + ((sub * 32) << 16) + acc * BN, n, slab + m * 256 + int(rank) * 128 + sub * 32);
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive_cluster(ptx::mapa(ptx::smem_u32(&bars->tempty[acc]), 0));
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
    }
    if (lane == 0) ptx::bulk_wait<0>();
    __syncwarp();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::cluster_sync();  // no CTA leaves while its peer's MMAs / signals may still target it
  if (warp == 1) ptx::tmem_dealloc2(tmem, 512);
}

}  // namespace

size_t gemm_smem_bytes() { return kGemmSmem2 > kGemmSmem1 ? kGemmSmem2 : kGemmSmem1; }

static int env_group(const char* name) {
  const char* v = std::getenv(name);
  return v && std::atoi(v) > 0 ? std::atoi(v) : 0;
}

void launch_gemm(int epi, const CUtensorMap& tmA, const CUtensorMap& tmB, const CUtensorMap& tmC,
                 const GemmParams& p_in, int num_sms, cudaStream_t stream) {
  static const int g_all = env_group("BAT_GEMM_GROUP_M"), g_swiglu = env_group("BAT_GEMM_GROUP_SWIGLU");
  static const int hints = env_group("BAT_GEMM_HINTS");
  GemmParams p = p_in;
  if (!p.hints) p.hints = hints;
  // SwiGLU (1-CTA, 128-row tiles, 55 MB of gate/up weights re-streamed once per group): groups of
  // 32 M-tiles with evict_last weight loads read 574 MB of DRAM per launch instead of 705 MB at
  // equal speed (profiles/r1_gemm_raster.txt)
  if (p.group_m <= 0)
    p.group_m = epi == EPI_SWIGLU ? (g_swiglu ? g_swiglu : GROUP_M_SWIGLU) : (g_all ? g_all : GROUP_M);
  if (epi == EPI_SWIGLU && !std::getenv("BAT_GEMM_HINTS")) p.hints |= 1;
  const int out_bn = (epi == EPI_SWIGLU) ? BN / 2 : BN;
  const int n_tiles = (p.N + out_bn - 1) / out_bn;
  // the SwiGLU GEMM stays on 1-CTA tiles: measured in the bench step, its pair version ran
  // slower (1.18 vs 1.24 PFLOP/s) although both tie when timed alone
  const int ks = epi == EPI_PART_F32 ? p.ksplit : 1;
  if (p.M >= 256 && num_sms >= 2 && epi != EPI_SWIGLU) {
    const int tiles = ((p.M + 255) / 256) * n_tiles * ks;
    const int pairs = tiles < num_sms / 2 ? tiles : num_sms / 2;
    auto launch = [&](auto kern) {
      set_smem_attr(kern, kGemmSmem2);
      kern<<<2 * pairs, NUM_THREADS, kGemmSmem2, stream>>>(tmA, tmB, tmC, p);
    };
    switch (epi) {
      case EPI_BF16: launch(gemm2_tc_kernel<EPI_BF16>); break;
      case EPI_BF16_BIAS: launch(gemm2_tc_kernel<EPI_BF16_BIAS>); break;
      case EPI_RESID_F32: launch(gemm2_tc_kernel<EPI_RESID_F32>); break;
      case EPI_SWIGLU: launch(gemm2_tc_kernel<EPI_SWIGLU>); break;
      case EPI_PART_F32: launch(gemm2_tc_kernel<EPI_PART_F32>); break;
    }
  } else {
    const int tiles = ((p.M + 127) / 128) * n_tiles * ks;
    const int grid = tiles < num_sms ? tiles : num_sms;
    if (grid <= 0) return;
    auto launch = [&](auto kern) {
      set_smem_attr(kern, kGemmSmem1);
      kern<<<grid, NUM_THREADS, kGemmSmem1, stream>>>(tmA, tmB, tmC, p);
    };
    switch (epi) {
      case EPI_BF16: launch(gemm_tc_kernel<EPI_BF16>); break;
      case EPI_BF16_BIAS: launch(gemm_tc_kernel<EPI_BF16_BIAS>); break;
      case EPI_RESID_F32: launch(gemm_tc_kernel<EPI_RESID_F32>); break;
      case EPI_SWIGLU: launch(gemm_tc_kernel<EPI_SWIGLU>); break;
      case EPI_PART_F32: launch(gemm_tc_kernel<EPI_PART_F32>); break;
    }
  }
  count_launch();
}

int gemm_ksplit(int epi, int M, int N, int K, int num_sms, int* mpad) {
  static const bool off = std::getenv("BAT_GEMM_SPLITK") && std::getenv("BAT_GEMM_SPLITK")[0] == '0';
  if (mpad) *mpad = 0;
  if (off || epi == EPI_SWIGLU || M <= 0) return 1;
  const bool pair = M >= 256 && num_sms >= 2;
  const int rows = pair ? 256 : 128;
  const int units = ((M + rows - 1) / rows) * ((N + BN - 1) / BN);  // CTA pairs or CTAs
  const int slots = pair ? num_sms / 2 : num_sms;
  const int num_kb = (K + BK - 1) / BK;
  int ks = slots / units;            // fill the idle SMs...
  ks = ks < num_kb / 4 ? ks : num_kb / 4;  // ...keeping >= 4 k-blocks (256 of K) per slice
  ks = ks < 8 ? ks : 8;
  if (ks < 2) return 1;
  if (mpad) *mpad = ((M + rows - 1) / rows) * rows;
  return ks;
}

__global__ void gemm_reduce_kernel(const float* __restrict__ part, int ksplit, int64_t slab, int M, int N,
                                   void* __restrict__ out, int ldo, const __nv_bfloat16* __restrict__ bias,
                                   int mode) {
  const int64_t n4 = int64_t(M) * (N / 4);
  for (int64_t e = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; e < n4; e += int64_t(gridDim.x) * blockDim.x) {
    const int m = int(e / (N / 4)), c = int(e % (N / 4)) * 4;
    const float4* src = reinterpret_cast<const float4*>(part + int64_t(m) * N + c);
    float4 a = src[0];
    for (int s = 1; s < ksplit; ++s) {  // slice order: deterministic
      const float4 b = src[s * slab / 4];
      a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
    }
    if (mode == 0) {
      float4* h = reinterpret_cast<float4*>(static_cast<float*>(out) + int64_t(m) * ldo + c);
      float4 v = *h;
      v.x += a.x; v.y += a.y; v.z += a.z; v.w += a.w;
      *h = v;
    } else {
      __nv_bfloat16* o = static_cast<__nv_bfloat16*>(out) + int64_t(m) * ldo + c;
      o[0] = __float2bfloat16_rn(a.x + (bias ? __bfloat162float(bias[c]) : 0.0f));
      o[1] = __float2bfloat16_rn(a.y + (bias ? __bfloat162float(bias[c + 1]) : 0.0f));
      o[2] = __float2bfloat16_rn(a.z + (bias ? __bfloat162float(bias[c + 2]) : 0.0f));
      o[3] = __float2bfloat16_rn(a.w + (bias ? __bfloat162float(bias[c + 3]) : 0.0f));
    }
  }
}

void launch_gemm_reduce(const float* part, int ksplit, int mpad, int M, int N, void* out, int ldo,
                        const __nv_bfloat16* bias, int mode, cudaStream_t stream) {
  const int64_t n4 = int64_t(M) * (N / 4);
  const int blocks = int((n4 + 255) / 256 < 1184 ? (n4 + 255) / 256 : 1184);
  gemm_reduce_kernel<<<blocks, 256, 0, stream>>>(part, ksplit, int64_t(mpad) * N, M, N, out, ldo, bias, mode);
  count_launch();
}

}  // namespace bat
