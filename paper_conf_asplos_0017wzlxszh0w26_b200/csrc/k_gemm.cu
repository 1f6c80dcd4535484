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
#include <algorithm>
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
constexpr int GROUP_M_SWIGLU = 32;       // 1-CTA SwiGLU kernel (128-row M-tiles)
constexpr int GROUP_M_SWIGLU_PAIR = 32;  // CTA-pair SwiGLU kernel (256-row M-tiles; profiles/r2_gemm_epilogue.txt (k))
// Epilogue warps per CTA: 4 (one per TMEM lane quarter) or 8 (two per quarter, splitting the
// accumulator's columns).  The SwiGLU GEMM (short K = hidden, MUFU-heavy epilogue) runs 8 and
// gains 5% over 4; the others keep 4 warps and one more ring stage (their K loops are long or
// their epilogues light: 8 warps measured 1-4% slower there, profiles/r2_gemm_epilogue.txt)
#ifndef BAT_GEMM_RESID_EW
#define BAT_GEMM_RESID_EW 4  // epilogue warps of the fp32 residual GEMMs (O, down)
#endif
#ifndef BAT_GEMM_QKV_EW
#define BAT_GEMM_QKV_EW 4  // epilogue warps of the bf16 (+bias) GEMMs (QKV)
#endif
constexpr int epi_warps(int epi) {
  return epi == EPI_SWIGLU ? 8 : (epi == EPI_RESID_F32 || epi == EPI_PART_F32) ? BAT_GEMM_RESID_EW : BAT_GEMM_QKV_EW;
}
// staging buffers per epilogue warp: two (double-buffered TMA stores) unless 8 warps would cost a
// ring stage; SwiGLU keeps two (its 8 warps run with one stage fewer)
constexpr int epi_nbuf(int epi) { return (epi_warps(epi) == 8 && epi != EPI_SWIGLU) ? 1 : 2; }
constexpr int STG_BYTES = 4096;  // per-warp epilogue staging buffer: [32 rows][128 B], 128B-swizzled

constexpr int STAGE1_BYTES = A_BYTES + BN * BK * 2;  // 1-CTA kernel (128 x 256 tiles): 48 KB per stage
constexpr int STAGE2_BYTES = A_BYTES + BROWS * BK * 2;  // CTA pair (256 x 256 tiles, 128 rows of A + B per CTA): 32 KB

struct __align__(8) GemmSmemBars {
  uint64_t full[8], empty[8], tfull[2], tempty[2];
  uint32_t tmem_base;
};
template <int EPI>
struct GemmCfg {
  static constexpr int EW = epi_warps(EPI), NB = epi_nbuf(EPI);
  static constexpr int THREADS = 64 + 32 * EW;
  static constexpr int SPLIT = EW / 4;  // column slices of an accumulator
  static constexpr int STG = EW * NB * STG_BYTES;  // epilogue staging
  static constexpr int BUDGET = 232448 - 1024 /*align slack*/ - 256 /*barriers*/ - STG;
  static constexpr int STAGES1 = BUDGET / STAGE1_BYTES < 4 ? BUDGET / STAGE1_BYTES : 4;
  static constexpr int STG1_OFF = STAGES1 * STAGE1_BYTES;
  static constexpr int STAGES2 = BUDGET / STAGE2_BYTES < 6 ? BUDGET / STAGE2_BYTES : 6;
  static constexpr int STG2_OFF = STAGES2 * STAGE2_BYTES;
  static constexpr size_t SMEM1 = 1024 /*align slack*/ + STG1_OFF + STG + sizeof(GemmSmemBars);
  static constexpr size_t SMEM2 = 1024 /*align slack*/ + STG2_OFF + STG + sizeof(GemmSmemBars);
  static_assert(EW == 4 || EW == 8, "epilogue warps");
  static_assert(SMEM1 <= 232448 && SMEM2 <= 232448, "GEMM shared memory");
  static_assert(STAGES2 <= 8, "barrier array");
};

__device__ __forceinline__ void tile_coords(int t, int num_m, int num_n, int group_m, int& m, int& n) {
  const int per_group = group_m * num_n;
  const int g = t / per_group;
  const int r = t - g * per_group;
  const int rows = min(group_m, num_m - g * group_m);
  m = g * group_m + r % rows;
  n = r / rows;
}

__device__ __forceinline__ float rcp_approx(float x) {
  float y;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float ex2_approx(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// silu(x) = x / (1 + e^-x) with MUFU ex2 and rcp (both ~1 ulp; an IEEE division cost ~10 more
// instructions per output in the epilogue, which paces the short-K SwiGLU GEMM)
__device__ __forceinline__ float silu(float x) { return x * rcp_approx(1.0f + ex2_approx(x * -1.44269504f)); }

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
  uint32_t sbias = 0;  // fused a4: shared-memory copy of the QKV bias (0: read it from global)

  __device__ __forceinline__ void stage_row(uint8_t* buf, int chunk16, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
    ptx::st_shared_v4(buf + lane * 128 + ((chunk16 ^ (lane & 7)) << 4), a, b, c, d);
  }
  __device__ __forceinline__ uint8_t* next_buf() {
    uint8_t* buf = stg + sbuf * STG_BYTES;
    if (lane == 0) {  // the group that last used this buffer is done reading it
      if (GemmCfg<EPI>::NB == 2) ptx::bulk_wait_read<1>();
      else ptx::bulk_wait_read<0>();
    }
    __syncwarp();
    return buf;
  }
  __device__ __forceinline__ void flush(uint8_t* buf, int col, int row) {
    ptx::fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
      if (EPI == EPI_RESID_F32 && p->norm_g) ptx::tma_store_2d(tmC, buf, col, row);  // h_new computed here
      else if (EPI == EPI_RESID_F32) ptx::tma_reduce_add_2d(tmC, buf, col, row);
      else if (EPI == EPI_PART_F32) ptx::tma_store_2d(tmC, buf, col, row);
      else if (p->hints & 2) ptx::tma_store_2d_hint(tmC, buf, col, row, ptx::policy_evict_first());
      else ptx::tma_store_2d(tmC, buf, col, row);
      ptx::bulk_commit();
    }
    sbuf ^= GemmCfg<EPI>::NB - 1;
  }
  // fused RMSNorm, consumer side: this lane's row scale rsqrt(mean(h^2) + eps) (1 without ss_in);
  // the partial sums are loaded together (independent loads), summed in a fixed order
  __device__ __forceinline__ float row_rstd(int row) const {
    if (!p->ss_in || row >= p->M) return 1.0f;
    float v[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) v[j] = j < p->ss_parts ? p->ss_in[int64_t(j) * p->M + row] : 0.0f;
    float ss = 0.0f;
#pragma unroll
    for (int j = 0; j < 32; ++j) ss += v[j];
    return rsqrtf(ss / float(p->norm_h) + p->eps);
  }
  // fused RMSNorm, producer side (EPI_RESID_F32 with norm_g): h_new = h + acc for this lane's row,
  // 32 columns per chunk; h_old is read directly (128 B per lane, one chunk ahead), h_new leaves
  // through the swizzled staging buffer and a TMA store, xg = bf16(h_new * g) with 16-byte stores
  // h_old of this lane's row, PD 32-column chunks ahead (the first PD issued before the
  // accumulator wait: resid_prefetch), so ~PD x 4 KB per warp are in flight against DRAM latency
  static constexpr int PD = 4;
  float4 hpre[PD][8];
  __device__ __forceinline__ void load_h_chunk(int row, int col, float4 (&dst)[8]) {
    const bool ok = row < p->M && col < p->N;
    const float4* src = reinterpret_cast<const float4*>(static_cast<const float*>(p->out) +
                                                        int64_t(ok ? row : 0) * p->ldo + (ok ? col : 0));
#pragma unroll
    for (int i = 0; i < 8; ++i) dst[i] = ok ? __ldcs(src + i) : make_float4(0.f, 0.f, 0.f, 0.f);
  }
  __device__ __forceinline__ void resid_prefetch(int row0, int n, int part) {
    constexpr int NCHK = BN / GemmCfg<EPI>::SPLIT / 32;  // chunks of this warp's column slice
    const int c_lo = part * (BN / GemmCfg<EPI>::SPLIT);
#pragma unroll
    for (int k = 0; k < PD && k < NCHK; ++k) load_h_chunk(row0 + int(lane), n * BN + c_lo + 32 * k, hpre[k]);
  }
  __device__ __forceinline__ void run_resid_norm(uint32_t tbase, int n, int row0, int c_lo, int c_hi, int part) {
    const int row = row0 + int(lane);
    const bool ok = row < p->M;
    const int col_base = n * BN;
    constexpr int NCHK = BN / GemmCfg<EPI>::SPLIT / 32;
    float ss = 0.0f;
#pragma unroll
    for (int k = 0; k < NCHK; ++k) {
      const int c = c_lo + 32 * k;
      float4 (&hv)[8] = hpre[k % PD];
      uint8_t* buf = next_buf();
      uint32_t r[32];
      ptx::tmem_ld32(tbase + c, r);
      ptx::tmem_ld_wait();
      const int col = col_base + c;
      const uint4* g4 = reinterpret_cast<const uint4*>(p->norm_g + (col < p->N ? col : 0));
      uint32_t pk[16];
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const float4 o = hv[j];
        const float v0 = o.x + __uint_as_float(r[4 * j]), v1 = o.y + __uint_as_float(r[4 * j + 1]);
        const float v2 = o.z + __uint_as_float(r[4 * j + 2]), v3 = o.w + __uint_as_float(r[4 * j + 3]);
        ss += v0 * v0 + v1 * v1 + v2 * v2 + v3 * v3;
        stage_row(buf, j, __float_as_uint(v0), __float_as_uint(v1), __float_as_uint(v2), __float_as_uint(v3));
        const uint4 gq = __ldg(g4 + (j >> 1));
        const uint32_t ga = (j & 1) ? gq.z : gq.x, gb = (j & 1) ? gq.w : gq.y;
        const float2 g01 = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&ga));
        const float2 g23 = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&gb));
        pk[2 * j] = ptx::pack_bf16x2(v0 * g01.x, v1 * g01.y);
        pk[2 * j + 1] = ptx::pack_bf16x2(v2 * g23.x, v3 * g23.y);
      }
      if (k + PD < NCHK) load_h_chunk(row, col + 32 * PD, hv);  // refill the slot PD chunks ahead
      if (ok && col < p->N) {
        uint4* xd = reinterpret_cast<uint4*>(p->xg_out + int64_t(row) * p->norm_h + col);
#pragma unroll
        for (int i = 0; i < 4; ++i) xd[i] = make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
      }
      flush(buf, col, row0);
    }
    (void)c_hi;
    if (ok) p->ss_out[int64_t(n * GemmCfg<EPI>::SPLIT + part) * p->M + row] = ss;
  }
  // a4 fused (GemmParams::stage): this lane's row = one suffix token; the N-tile holds 256 / d whole
  // heads (q, then k, then v).  Per head: (x rs) + bias, RoPE of the column pairs (c, c + d/2) at the
  // token's plan position in fp32 (q and k), one bf16 rounding, 16-byte stores into the GQA-packed,
  // 128B-swizzled q-tile row (token x head-in-group) or the suffix page block (K / V) — the layouts
  // stage_kernel writes (k_misc.cu).  The row's plan lookups (request, q-tile, page) are issued
  // before the accumulator wait (StageRow), the (cos, sin) of a column block once for all heads.
  struct StageRow {
    bool ok;
    int t, pos, gq;     // token index in the request's suffix, plan position, global q-tile
    const char* page;   // the suffix page holding the token's K / V
  };
  __device__ __forceinline__ StageRow stage_row(int row_in) const {
    const StageParams& sp = p->stage;
    StageRow r;
    r.ok = row_in < p->M;
    const int row = r.ok ? row_in : p->M - 1;  // lanes past the batch: same loads, no stores
    const int32_t* img = sp.img;
    const int32_t* qi = img + sp.off_qinfo + int64_t(__ldg(img + sp.off_rowreq + row)) * 8;  // the row's request
    r.t = row - __ldg(qi);
    r.pos = min(__ldg(img + sp.off_pos + row), sp.max_pos - 1);
    r.gq = __ldg(qi + 2) + r.t / sp.qt;
    const int target = __ldg(img + sp.off_spages + int64_t(__ldg(qi + 6) + r.t / 16) * 4 + 3);
    r.page = target >= 0 ? sp.pool + int64_t(target) * sp.pool_page_bytes + sp.pool_layer_off
                         : sp.scratch + int64_t(-target - 1) * sp.scratch_page_bytes + sp.scratch_layer_off;
    return r;
  }
  __device__ __forceinline__ void run_stage(uint32_t tbase, int n, const StageRow& sr, float rs, int part) {
    const StageParams& sp = p->stage;
    const int d = sp.head_dim, half = d / 2;
    const int nh = BN / d;  // heads of this N-tile; this warp's: [part, part + 1) * nh / SPLIT
    constexpr int SPLIT = GemmCfg<EPI>::SPLIT;
    const uint32_t chunks = uint32_t(sp.dpad / 64);
    const float4* cs4 = reinterpret_cast<const float4*>(sp.rope + int64_t(sr.pos) * half);
#pragma unroll 1
    for (int c = 0; c < half; c += 32) {  // column pairs (c + i, c + half + i), i < 32, of every head
      float4 rot[16];  // (cos, sin) of pairs c + 2k, c + 2k + 1
#pragma unroll
      for (int k = 0; k < 16; ++k) rot[k] = __ldg(cs4 + (c >> 1) + k);
#pragma unroll 1
      for (int hh = part * nh / SPLIT; hh < (part + 1) * nh / SPLIT; ++hh) {
        const int head = n * nh + hh;  // 0 .. Hq-1: q, then Hkv k heads, then Hkv v heads
        if (head >= sp.q_heads + 2 * sp.kv_heads) break;
        const bool is_q = head < sp.q_heads;
        const int kvi = is_q ? 0 : head - sp.q_heads;  // k: [0, Hkv), v: [Hkv, 2 Hkv)
        const bool rope = sp.rope_enabled && kvi < sp.kv_heads;
        const int rq = (sr.t % sp.qt) * sp.group + head % sp.group;  // q-tile row
        char* dst = is_q ? reinterpret_cast<char*>(sp.qp) +
                               (int64_t(sr.gq) * sp.kv_heads + head / sp.group) * (sp.dpad / 64) * 16384 + int64_t(rq) * 128
                         : const_cast<char*>(sr.page) + (int64_t(kvi / sp.kv_heads) * sp.kv_heads + kvi % sp.kv_heads) * sp.head_bytes;
        uint32_t a[32], b[32];
        ptx::tmem_ld32(tbase + hh * d + c, a);
        ptx::tmem_ld32(tbase + hh * d + half + c, b);
        const int col = n * BN + hh * d + c;
        const uint4* b1 = reinterpret_cast<const uint4*>(p->bias + col);
        const uint4* b2 = reinterpret_cast<const uint4*>(p->bias + col + half);
        uint4 bv1[4], bv2[4];  // the block's bias, in flight with the TMEM loads
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          bv1[j] = sbias ? ptx::ld_shared_v4(sbias + uint32_t(col) * 2 + 16 * j) : __ldg(b1 + j);
          bv2[j] = sbias ? ptx::ld_shared_v4(sbias + uint32_t(col + half) * 2 + 16 * j) : __ldg(b2 + j);
        }
        ptx::tmem_ld_wait();
        uint32_t pa[16], pb[16];
#pragma unroll
        for (int j = 0; j < 4; ++j) {  // 8 columns per bias vector
          const uint4 v1 = bv1[j], v2 = bv2[j];
          const uint32_t w1[4] = {v1.x, v1.y, v1.z, v1.w}, w2[4] = {v2.x, v2.y, v2.z, v2.w};
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const int i = 8 * j + 2 * k;
            const float2 g1 = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&w1[k]));
            const float2 g2 = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&w2[k]));
            float x10 = fmaf(__uint_as_float(a[i]), rs, g1.x), x11 = fmaf(__uint_as_float(a[i + 1]), rs, g1.y);
            float x20 = fmaf(__uint_as_float(b[i]), rs, g2.x), x21 = fmaf(__uint_as_float(b[i + 1]), rs, g2.y);
            if (rope) {
              const float4 t4 = rot[i >> 1];
              const float o10 = x10 * t4.x - x20 * t4.y, o20 = x20 * t4.x + x10 * t4.y;
              const float o11 = x11 * t4.z - x21 * t4.w, o21 = x21 * t4.z + x11 * t4.w;
              x10 = o10; x20 = o20; x11 = o11; x21 = o21;
            }
            pa[i / 2] = ptx::pack_bf16x2(x10, x11);
            pb[i / 2] = ptx::pack_bf16x2(x20, x21);
          }
        }
        if (sr.ok) {
#pragma unroll
          for (int j = 0; j < 4; ++j) {  // 8-column chunks of the two column ranges
            const int c1 = c + 8 * j, c2 = c + half + 8 * j;
            uint32_t o1, o2;
            if (is_q) {
              o1 = (c1 >> 6) * 16384 + ((((c1 & 63) >> 3) ^ (uint32_t(rq) & 7u)) << 4);
              o2 = (c2 >> 6) * 16384 + ((((c2 & 63) >> 3) ^ (uint32_t(rq) & 7u)) << 4);
            } else {
              o1 = ptx::page_blk_off(uint32_t(sr.t % 16), uint32_t(c1), chunks);
              o2 = ptx::page_blk_off(uint32_t(sr.t % 16), uint32_t(c2), chunks);
            }
            *reinterpret_cast<uint4*>(dst + o1) = make_uint4(pa[4 * j], pa[4 * j + 1], pa[4 * j + 2], pa[4 * j + 3]);
            *reinterpret_cast<uint4*>(dst + o2) = make_uint4(pb[4 * j], pb[4 * j + 1], pb[4 * j + 2], pb[4 * j + 3]);
          }
        }
      }
    }
  }
  // tbase: TMEM address of this warp's lanes, column 0 of the accumulator; n: output N-tile;
  // part: this warp's column slice of the accumulator (EPI_SPLIT slices); rs: the row's fused-norm
  // scale (row_rstd, loaded before the accumulator wait)
  __device__ __forceinline__ void run(uint32_t tbase, int n, int row0, int part, float rs) {
    constexpr int W = BN / GemmCfg<EPI>::SPLIT;  // accumulator columns per slice
    const int c_lo = part * W, c_hi = c_lo + W;
    if constexpr (EPI == EPI_RESID_F32) {
      if (p->norm_g) {
        run_resid_norm(tbase, n, row0, c_lo, c_hi, part);
        return;
      }
    }

    if constexpr (EPI == EPI_SWIGLU) {
#pragma unroll 1
      for (int c = c_lo / 2; c < c_hi / 2; c += 64) {  // 64 output columns per staging buffer
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
            float g0 = __uint_as_float(g[2 * i]) * rs, g1 = __uint_as_float(g[2 * i + 1]) * rs;
            float u0 = __uint_as_float(u[2 * i]) * rs, u1 = __uint_as_float(u[2 * i + 1]) * rs;
            pk[i] = ptx::pack_bf16x2(silu(g0) * u0, silu(g1) * u1);
          }
#pragma unroll
          for (int j = 0; j < 4; ++j) stage_row(buf, 4 * h + j, pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
        }
        flush(buf, n * (BN / 2) + c, row0);
      }
    } else if constexpr (EPI == EPI_RESID_F32 || EPI == EPI_PART_F32) {
#pragma unroll 1
      for (int c = c_lo; c < c_hi; c += 32) {  // 32 fp32 columns per staging buffer
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
      for (int c = c_lo; c < c_hi; c += 64) {  // 64 bf16 columns per staging buffer
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
            float v0 = __uint_as_float(r[2 * i]) * rs, v1 = __uint_as_float(r[2 * i + 1]) * rs;
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
__global__ void __launch_bounds__(GemmCfg<EPI>::THREADS, 1)
gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
               const __grid_constant__ CUtensorMap tmC, GemmParams p) {
  extern __shared__ uint8_t smem_raw[];
  // 1 KB-align by offsetting the __shared__ array itself (keeps the shared address space, so
  // the compiler emits LDS/STS rather than generic loads and stores)
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  using C = GemmCfg<EPI>;
  constexpr int STAGES1 = C::STAGES1, STG1_OFF = C::STG1_OFF, EPI_WARPS = C::EW;
  GemmSmemBars* bars = reinterpret_cast<GemmSmemBars*>(smem + STG1_OFF + C::STG);
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
      ptx::mbar_init(&bars->tempty[a], EPI_WARPS);
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
  } else {  // ------------------------------ epilogue warps 2 .. 1 + EPI_WARPS
    const uint32_t sub = warp & 3;  // TMEM sub-partition this warp may access
    const int part = int(warp - 2) / 4;  // column slice
    Epilogue<EPI> epi{&tmC, &p, smem + STG1_OFF + (warp - 2) * C::NB * STG_BYTES, lane};
    if constexpr (EPI == EPI_BF16_BIAS) {
      // fused a4: the bias lives in the staging region (the a4 path stores directly, not via TMA)
      if (p.stage_on && p.N * 2 <= C::STG) {
        const int t = int(threadIdx.x) - 64;  // epilogue threads 0 .. 32 * EPI_WARPS - 1
        uint32_t* dst = reinterpret_cast<uint32_t*>(smem + STG1_OFF);
        const uint32_t* src = reinterpret_cast<const uint32_t*>(p.bias);
        for (int i = t; i < p.N / 2; i += 32 * EPI_WARPS) dst[i] = __ldg(src + i);
        ptx::bar_sync(1, 32 * EPI_WARPS);
        epi.sbias = ptx::smem_u32(smem + STG1_OFF);
      }
    }
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int t = blockIdx.x; t < num_work; t += gridDim.x) {
      int m, n;
      tile_coords(t % num_tiles, num_m, num_n, p.group_m, m, n);
      const int slab = EPI == EPI_PART_F32 ? (t / num_tiles) * p.mpad : 0;
      const int row0 = slab + m * 128 + int(sub) * 32;
      const float rs = (EPI == EPI_SWIGLU || EPI == EPI_BF16_BIAS) ? epi.row_rstd(row0 + int(lane)) : 1.0f;
      if constexpr (EPI == EPI_RESID_F32) {
        if (p.norm_g) epi.resid_prefetch(row0, n, part);  // h_old in flight during the accumulator wait
      }
      bool staged = false;
      if constexpr (EPI == EPI_BF16_BIAS) {
        if (p.stage_on) {  // a4 fused: the row's plan lookups overlap the accumulator wait
          const auto sr = epi.stage_row(row0 + int(lane));
          ptx::mbar_wait(&bars->tfull[acc], acc_phase);
          ptx::tc_fence_after();
          epi.run_stage(tmem + ((sub * 32) << 16) + acc * BN, n, sr, rs, part);
          staged = true;
        }
      }
      if (!staged) {
        ptx::mbar_wait(&bars->tfull[acc], acc_phase);
        ptx::tc_fence_after();
        epi.run(tmem + ((sub * 32) << 16) + acc * BN, n, row0, part, rs);
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive_relaxed(&bars->tempty[acc]);  // orders the TMEM reads only
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
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(GemmCfg<EPI>::THREADS, 1)
gemm2_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                const __grid_constant__ CUtensorMap tmC, GemmParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  using C = GemmCfg<EPI>;
  constexpr int STAGES2 = C::STAGES2, STG2_OFF = C::STG2_OFF, EPI_WARPS = C::EW;
  GemmSmemBars* bars = reinterpret_cast<GemmSmemBars*>(smem + STG2_OFF + C::STG);
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
      ptx::mbar_init(&bars->tempty[a], 2 * EPI_WARPS);  // leader: the epilogue warps of both CTAs
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
      const uint64_t pol_b = ptx::policy_evict_last();
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
          if (p.hints & 1)
            ptx::tma_load_2d_pair_hint(sb, &tmB, kb * BK, b_row<EPI>(p, n, int(rank)), full_leader, pol_b);
          else
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
  } else {  // ------------------------------ epilogue warps (both CTAs): my 128 rows
    const uint32_t sub = warp & 3;
    const int part = int(warp - 2) / 4;  // column slice
    Epilogue<EPI> epi{&tmC, &p, smem + STG2_OFF + (warp - 2) * C::NB * STG_BYTES, lane};
    if constexpr (EPI == EPI_BF16_BIAS) {
      // fused a4: the bias lives in the staging region (the a4 path stores directly, not via TMA)
      if (p.stage_on && p.N * 2 <= C::STG) {
        const int t = int(threadIdx.x) - 64;  // epilogue threads 0 .. 32 * EPI_WARPS - 1
        uint32_t* dst = reinterpret_cast<uint32_t*>(smem + STG2_OFF);
        const uint32_t* src = reinterpret_cast<const uint32_t*>(p.bias);
        for (int i = t; i < p.N / 2; i += 32 * EPI_WARPS) dst[i] = __ldg(src + i);
        ptx::bar_sync(1, 32 * EPI_WARPS);
        epi.sbias = ptx::smem_u32(smem + STG2_OFF);
      }
    }
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int t = pair; t < num_work; t += n_pairs) {
      int m, n;
      tile_coords(t % num_tiles, num_m, num_n, p.group_m, m, n);
      const int slab = EPI == EPI_PART_F32 ? (t / num_tiles) * p.mpad : 0;
      const int row0 = slab + m * 256 + int(rank) * 128 + int(sub) * 32;
      const float rs = (EPI == EPI_SWIGLU || EPI == EPI_BF16_BIAS) ? epi.row_rstd(row0 + int(lane)) : 1.0f;
      if constexpr (EPI == EPI_RESID_F32) {
        if (p.norm_g) epi.resid_prefetch(row0, n, part);  // h_old in flight during the accumulator wait
      }
      bool staged = false;
      if constexpr (EPI == EPI_BF16_BIAS) {
        if (p.stage_on) {  // a4 fused: the row's plan lookups overlap the accumulator wait
          const auto sr = epi.stage_row(row0 + int(lane));
          ptx::mbar_wait(&bars->tfull[acc], acc_phase);
          ptx::tc_fence_after();
          epi.run_stage(tmem + ((sub * 32) << 16) + acc * BN, n, sr, rs, part);
          staged = true;
        }
      }
      if (!staged) {
        ptx::mbar_wait(&bars->tfull[acc], acc_phase);
        ptx::tc_fence_after();
        epi.run(tmem + ((sub * 32) << 16) + acc * BN, n, row0, part, rs);
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive_cluster_relaxed(ptx::mapa(ptx::smem_u32(&bars->tempty[acc]), 0));
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

bool gemm_qkv_stage_fusable(int head_dim) {
  // whole heads per epilogue warp, 32-column blocks of each half head
  return head_dim % 64 == 0 && (BN / head_dim) % GemmCfg<EPI_BF16_BIAS>::SPLIT == 0;
}

int gemm_epi_col_splits() { return GemmCfg<EPI_RESID_F32>::SPLIT; }

size_t gemm_smem_bytes() {
  size_t m = 0;
  for (size_t v : {GemmCfg<EPI_BF16>::SMEM1, GemmCfg<EPI_BF16>::SMEM2, GemmCfg<EPI_BF16_BIAS>::SMEM1,
                   GemmCfg<EPI_BF16_BIAS>::SMEM2, GemmCfg<EPI_RESID_F32>::SMEM1, GemmCfg<EPI_RESID_F32>::SMEM2,
                   GemmCfg<EPI_SWIGLU>::SMEM1, GemmCfg<EPI_SWIGLU>::SMEM2, GemmCfg<EPI_PART_F32>::SMEM1,
                   GemmCfg<EPI_PART_F32>::SMEM2})
    m = std::max(m, v);
  return m;
}

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
  // SwiGLU on CTA pairs by default (BAT_GEMM_SWIGLU_PAIR=0: 1-CTA 128-row tiles): 8 epilogue warps
  // and MUFU ex2 / rcp silu, 1,202 -> 1,375-1,389 TFLOP/s in the configs[2] step against the 1-CTA
  // kernel with the same epilogue (profiles/r2_gemm_epilogue.txt); rasterisation groups of 32 pair
  // M-tiles (8,192 rows) or 32 1-CTA M-tiles, evict_last weight loads (the 55 MB of gate/up
  // weights are re-streamed once per group; profiles/r1_gemm_raster.txt)
  static const char* sp_env = std::getenv("BAT_GEMM_SWIGLU_PAIR");
  static const bool swiglu_pair = !(sp_env && sp_env[0] == '0');
  const bool pair = p.M >= 256 && num_sms >= 2 && (epi != EPI_SWIGLU || swiglu_pair);
  if (p.group_m <= 0)
    p.group_m = epi == EPI_SWIGLU ? (g_swiglu ? g_swiglu : (pair ? GROUP_M_SWIGLU_PAIR : GROUP_M_SWIGLU))
                                  : (g_all ? g_all : GROUP_M);
  if (epi == EPI_SWIGLU && !std::getenv("BAT_GEMM_HINTS")) p.hints |= 1;
  const int out_bn = (epi == EPI_SWIGLU) ? BN / 2 : BN;
  const int n_tiles = (p.N + out_bn - 1) / out_bn;
  const int ks = epi == EPI_PART_F32 ? p.ksplit : 1;
  if (pair) {
    const int tiles = ((p.M + 255) / 256) * n_tiles * ks;
    const int pairs = tiles < num_sms / 2 ? tiles : num_sms / 2;
    auto launch = [&](auto kern, auto cfg) {
      using C = decltype(cfg);
      set_smem_attr(kern, C::SMEM2);
      kern<<<2 * pairs, C::THREADS, C::SMEM2, stream>>>(tmA, tmB, tmC, p);
    };
    switch (epi) {
      case EPI_BF16: launch(gemm2_tc_kernel<EPI_BF16>, GemmCfg<EPI_BF16>{}); break;
      case EPI_BF16_BIAS: launch(gemm2_tc_kernel<EPI_BF16_BIAS>, GemmCfg<EPI_BF16_BIAS>{}); break;
      case EPI_RESID_F32: launch(gemm2_tc_kernel<EPI_RESID_F32>, GemmCfg<EPI_RESID_F32>{}); break;
      case EPI_SWIGLU: launch(gemm2_tc_kernel<EPI_SWIGLU>, GemmCfg<EPI_SWIGLU>{}); break;
      case EPI_PART_F32: launch(gemm2_tc_kernel<EPI_PART_F32>, GemmCfg<EPI_PART_F32>{}); break;
    }
  } else {
    const int tiles = ((p.M + 127) / 128) * n_tiles * ks;
    const int grid = tiles < num_sms ? tiles : num_sms;
    if (grid <= 0) return;
    auto launch = [&](auto kern, auto cfg) {
      using C = decltype(cfg);
      set_smem_attr(kern, C::SMEM1);
      kern<<<grid, C::THREADS, C::SMEM1, stream>>>(tmA, tmB, tmC, p);
    };
    switch (epi) {
      case EPI_BF16: launch(gemm_tc_kernel<EPI_BF16>, GemmCfg<EPI_BF16>{}); break;
      case EPI_BF16_BIAS: launch(gemm_tc_kernel<EPI_BF16_BIAS>, GemmCfg<EPI_BF16_BIAS>{}); break;
      case EPI_RESID_F32: launch(gemm_tc_kernel<EPI_RESID_F32>, GemmCfg<EPI_RESID_F32>{}); break;
      case EPI_SWIGLU: launch(gemm_tc_kernel<EPI_SWIGLU>, GemmCfg<EPI_SWIGLU>{}); break;
      case EPI_PART_F32: launch(gemm_tc_kernel<EPI_PART_F32>, GemmCfg<EPI_PART_F32>{}); break;
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
