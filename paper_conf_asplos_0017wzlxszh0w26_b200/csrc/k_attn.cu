// Bipartite attention over paged prefix KV + the suffix's own KV (
// PAPER.md P:207).
//
// One work item = (request b, KV head, packed q-tile): 128 rows = qt suffix tokens x the g
// query heads sharing that KV head (GQA packing), against the item's list of live 128-key
// k-tiles from the plan (block-skip: dead tiles never reach the kernel; "full" tiles skip
// the element mask; "partial" tiles apply  kord <= rord && (kseg == rseg || (kseg|rseg) < 0)).
//
// Warp roles (192 threads, one CTA per SM, persistent over work items):
//   warp 0   loader: one bulk copy for the q-tile (pre-packed and pre-swizzled by the stage
//            kernel) and, per k-tile, 2 KB bulk copies of each page's K and V blocks — the
//            pool stores pages in the tensor-core operand layout, so no TMA descriptor or
//            reshuffle is needed — plus the k-tile's key metadata (1 KB).
//   warp 1   MMA issuer (one thread): S = Q K^T (tcgen05.mma SS, M=128 N=128 K=16) into one
//            of two TMEM S buffers; O += P V (tcgen05.mma TS: P read from TMEM, V MN-major
//            from smem) into a TMEM O accumulator.  Issue order S0 S1 PV0 S2 PV1 ... keeps the
//            tensor pipe busy while the softmax warps work on the other S buffer.
//   warps 2-5 softmax (thread = row): tcgen05.ld of the S row, mask, online softmax in the
//            log2 domain with a lazy running max (O is rescaled only when the max grows by
//            more than 2^8, FA4-style), P = exp2(.) packed to bf16 and written back into the S
//            buffer's TMEM columns with tcgen05.st; finally O / l is stored as bf16.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace bat {
namespace {

constexpr int NUM_THREADS = 192;
constexpr float kRescaleThreshold = 8.0f;  // log2 units: P <= 2^8 between rescales

template <int DP>
struct AttnSmem {
  static constexpr int CHUNKS = DP / 64;
  static constexpr int TILE_BYTES = CHUNKS * 128 * 128;  // [CHUNKS][128 rows][64] bf16
  static constexpr int Q_OFF = 0;                        // 2 q buffers
  static constexpr int K_OFF = Q_OFF + 2 * TILE_BYTES;   // 2 stages
  static constexpr int V_OFF = K_OFF + 2 * TILE_BYTES;   // 2 stages
  static constexpr int META_OFF = V_OFF + 2 * TILE_BYTES;  // 2 x 128 x int2
  static constexpr int BAR_OFF = META_OFF + 2 * 1024;
  static constexpr int TOTAL = BAR_OFF + 256;
};

struct __align__(8) AttnBars {
  uint64_t q_full[2], q_empty[2];
  uint64_t k_full[2], v_full[2], kv_empty[2];
  uint64_t s_full[2], p_full[2], pv_done[2];
  uint64_t o_full, o_empty;
  uint32_t tmem_base;
};

__device__ __forceinline__ const char* resolve_page(const AttnParams& p, int32_t page) {
  if (page == kZeroPage) return p.zero_page;
  if (page >= 0) return p.pool + int64_t(page) * p.pool_page_bytes + p.pool_layer_off;
  return p.scratch + int64_t(-page - 1) * p.scratch_page_bytes + p.scratch_layer_off;
}

template <int DP>
__global__ void __launch_bounds__(NUM_THREADS, 1) attn_tc_kernel(const __grid_constant__ AttnParams p) {
  using L = AttnSmem<DP>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  AttnBars* bars = reinterpret_cast<AttnBars*>(smem + L::BAR_OFF);
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();
  constexpr uint32_t S_COLS = 128;
  constexpr uint32_t O_COL = 256;
  constexpr uint32_t IDESC_S = ptx::idesc_bf16(128, 128, 0, 0);
  constexpr uint32_t IDESC_PV = ptx::idesc_bf16(128, DP, 0, 1);

  if (warp == 0 && lane == 0) {
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&bars->q_full[i], 1);
      ptx::mbar_init(&bars->q_empty[i], 1);
      ptx::mbar_init(&bars->k_full[i], 1);
      ptx::mbar_init(&bars->v_full[i], 1);
      ptx::mbar_init(&bars->kv_empty[i], 1);
      ptx::mbar_init(&bars->s_full[i], 1);
      ptx::mbar_init(&bars->p_full[i], 4);
      ptx::mbar_init(&bars->pv_done[i], 1);
    }
    ptx::mbar_init(&bars->o_full, 1);
    ptx::mbar_init(&bars->o_empty, 4);
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc(&bars->tmem_base, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = bars->tmem_base;

  const int32_t* img = p.img;
  const int32_t* work = img + p.off_work;

  if (warp == 0) {
    if (lane == 0) {  // ------------------------------------------------------ loader
      uint32_t qc = 0, kc = 0;
      for (int w = blockIdx.x; w < p.n_work; w += gridDim.x, ++qc) {
        const int4 wi = *reinterpret_cast<const int4*>(work + int64_t(w) * 4);
        const int b = wi.x, kvh = wi.y >> 16, qi = wi.y & 0xFFFF, kt_off = wi.z, kt_n = wi.w;
        const int32_t* q_info = img + p.off_qinfo + int64_t(b) * 8;
        const int qtile0 = q_info[2], page_off = q_info[4];
        const int qb = qc & 1;
        ptx::mbar_wait(&bars->q_empty[qb], ((qc >> 1) & 1) ^ 1);
        ptx::mbar_expect_tx(&bars->q_full[qb], L::TILE_BYTES);
        const char* qsrc = reinterpret_cast<const char*>(p.qp) +
                           (int64_t(qtile0 + qi) * p.kv_heads + kvh) * L::TILE_BYTES;
        ptx::bulk_g2s(smem + L::Q_OFF + qb * L::TILE_BYTES, qsrc, L::TILE_BYTES, &bars->q_full[qb]);
        for (int x = 0; x < kt_n; ++x, ++kc) {
          const int j = img[kt_off + x] & 0xFFFFFF;
          const int s = kc & 1;
          ptx::mbar_wait(&bars->kv_empty[s], ((kc >> 1) & 1) ^ 1);
          uint8_t* sk = smem + L::K_OFF + s * L::TILE_BYTES;
          uint8_t* sv = smem + L::V_OFF + s * L::TILE_BYTES;
          const int32_t* pages = img + p.off_pages + page_off + j * kKtilePages;
          ptx::mbar_expect_tx(&bars->k_full[s], L::TILE_BYTES + 1024);
          for (int pg = 0; pg < kKtilePages; ++pg) {
            const char* base = resolve_page(p, pages[pg]) + int64_t(kvh) * p.head_bytes;
#pragma unroll
            for (int c = 0; c < L::CHUNKS; ++c)
              ptx::bulk_g2s(sk + c * 16384 + pg * 2048, base + c * 2048, 2048, &bars->k_full[s]);
          }
          ptx::bulk_g2s(smem + L::META_OFF + s * 1024,
                        img + p.off_kmeta + (int64_t(page_off) + int64_t(j) * kKtilePages) * kPageTokens * 2,
                        1024, &bars->k_full[s]);
          ptx::mbar_expect_tx(&bars->v_full[s], L::TILE_BYTES);
          for (int pg = 0; pg < kKtilePages; ++pg) {
            const char* base = resolve_page(p, pages[pg]) + int64_t(p.kv_heads + kvh) * p.head_bytes;
#pragma unroll
            for (int c = 0; c < L::CHUNKS; ++c)
              ptx::bulk_g2s(sv + c * 16384 + pg * 2048, base + c * 2048, 2048, &bars->v_full[s]);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ---------------------------------------------------- MMA issuer
      uint32_t qc = 0, kc = 0;
      for (int w = blockIdx.x; w < p.n_work; w += gridDim.x, ++qc) {
        const int4 wi = *reinterpret_cast<const int4*>(work + int64_t(w) * 4);
        const int kt_n = wi.w;
        const int qb = qc & 1;
        ptx::mbar_wait(&bars->q_full[qb], (qc >> 1) & 1);
        ptx::tc_fence_after();
        const uint32_t sq = ptx::smem_u32(smem + L::Q_OFF + qb * L::TILE_BYTES);
        auto issue_pv = [&](int y) {
          const uint32_t g = kc + y;
          const int s = g & 1;
          const uint32_t ph = (g >> 1) & 1;
          if (y == 0) ptx::mbar_wait(&bars->o_empty, (qc & 1) ^ 1);
          ptx::mbar_wait(&bars->p_full[s], ph);
          ptx::mbar_wait(&bars->v_full[s], ph);
          ptx::tc_fence_after();
          const uint32_t sv = ptx::smem_u32(smem + L::V_OFF + s * L::TILE_BYTES);
#pragma unroll
          for (int kk = 0; kk < 8; ++kk) {
            uint64_t db = ptx::desc_sw128(sv + kk * 2048, 16384, 1024);
            ptx::mma_ts(tmem + O_COL, tmem + s * S_COLS + kk * 8, db, IDESC_PV, (y | kk) ? 1u : 0u);
          }
          ptx::mma_commit(&bars->kv_empty[s]);
          ptx::mma_commit(&bars->pv_done[s]);
        };
        for (int x = 0; x < kt_n; ++x) {
          const uint32_t g = kc + x;
          const int s = g & 1;
          ptx::mbar_wait(&bars->k_full[s], (g >> 1) & 1);
          ptx::tc_fence_after();
          const uint32_t sk = ptx::smem_u32(smem + L::K_OFF + s * L::TILE_BYTES);
#pragma unroll
          for (int kk = 0; kk < DP / 16; ++kk) {
            const uint32_t off = (kk >> 2) * 16384 + (kk & 3) * 32;
            uint64_t da = ptx::desc_sw128(sq + off, 16, 1024);
            uint64_t db = ptx::desc_sw128(sk + off, 16, 1024);
            ptx::mma_ss(tmem + s * S_COLS, da, db, IDESC_S, kk ? 1u : 0u);
          }
          ptx::mma_commit(&bars->s_full[s]);
          if (x == kt_n - 1) ptx::mma_commit(&bars->q_empty[qb]);
          if (x >= 1) issue_pv(x - 1);
        }
        if (kt_n > 0) issue_pv(kt_n - 1);
        ptx::mma_commit(&bars->o_full);
        kc += kt_n;
      }
    }
  } else {  // ------------------------------------------------------------ softmax warps
    const uint32_t sub = warp & 3;
    const int row = sub * 32 + lane;
    const uint32_t lane_base = (sub * 32) << 16;
    uint32_t qc = 0, kc = 0;
    for (int w = blockIdx.x; w < p.n_work; w += gridDim.x, ++qc) {
      const int4 wi = *reinterpret_cast<const int4*>(work + int64_t(w) * 4);
      const int b = wi.x, kvh = wi.y >> 16, qi = wi.y & 0xFFFF, kt_off = wi.z, kt_n = wi.w;
      const int32_t* q_info = img + p.off_qinfo + int64_t(b) * 8;
      const int tok_off = q_info[0], S = q_info[1];
      const int tok_local = qi * p.qt + row / p.group;
      const bool valid_row = row < p.qt * p.group && tok_local < S;
      const int32_t rseg = valid_row ? img[p.off_rseg + tok_off + tok_local] : -1;
      const int32_t rord = valid_row ? tok_local + 1 : kInvalidOrd - 1;
      float m_ref = -INFINITY, l_sum = 0.0f;
      for (int x = 0; x < kt_n; ++x) {
        const uint32_t g = kc + x;
        const int s = g & 1;
        const uint32_t ph = (g >> 1) & 1;
        const int state = img[kt_off + x] >> 24;
        ptx::mbar_wait(&bars->s_full[s], ph);
        ptx::tc_fence_after();
        float v[128];
        {
          uint32_t r[32];
#pragma unroll
          for (int c = 0; c < 4; ++c) {
            ptx::tmem_ld32(tmem + lane_base + s * S_COLS + c * 32, r);
            ptx::tmem_ld_wait();
#pragma unroll
            for (int i = 0; i < 32; ++i) v[c * 32 + i] = __uint_as_float(r[i]) * p.scale_log2;
          }
        }
        if (state == 2) {
          ptx::mbar_wait(&bars->k_full[s], ph);  // key metadata landed (already complete)
          const int2* meta = reinterpret_cast<const int2*>(smem + L::META_OFF + s * 1024);
#pragma unroll
          for (int c = 0; c < 128; ++c) {
            const int2 km = meta[c];  // (kseg, kord), same address across the warp: broadcast
            const bool vis = (km.y <= rord) && ((km.x == rseg) || ((km.x | rseg) < 0));
            v[c] = vis ? v[c] : -INFINITY;
          }
        }
        float mt = v[0];
#pragma unroll
        for (int c = 1; c < 128; ++c) mt = fmaxf(mt, v[c]);
        const float m_old = m_ref;
        const float m_new = fmaxf(m_ref, mt);
        const bool grow = m_new > m_ref + kRescaleThreshold;
        float alpha = 1.0f;
        if (grow) {
          alpha = exp2f(m_ref - m_new);  // 0 when m_ref = -inf
          l_sum *= alpha;
          m_ref = m_new;
        }
        // rescale the O accumulator rows of this warp when any lane's reference max moved
        const bool need_o = grow && (m_old != -INFINITY) && (x > 0);
        if (__any_sync(0xffffffffu, need_o)) {
          const uint32_t gp = g - 1;
          ptx::mbar_wait(&bars->pv_done[gp & 1], (gp >> 1) & 1);
          ptx::tc_fence_after();
          const float a = need_o ? alpha : 1.0f;
#pragma unroll
          for (int c = 0; c < DP / 32; ++c) {
            uint32_t r[32];
            ptx::tmem_ld32(tmem + lane_base + O_COL + c * 32, r);
            ptx::tmem_ld_wait();
#pragma unroll
            for (int i = 0; i < 32; ++i) r[i] = __float_as_uint(__uint_as_float(r[i]) * a);
            ptx::tmem_st32(tmem + lane_base + O_COL + c * 32, r);
          }
          ptx::tmem_st_wait();
        }
        const float mref = (m_ref == -INFINITY) ? 0.0f : m_ref;
        float lsum = 0.0f;
#pragma unroll
        for (int c = 0; c < 2; ++c) {
          uint32_t pk[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const float p0 = exp2f(v[c * 64 + 2 * i] - mref);
            const float p1 = exp2f(v[c * 64 + 2 * i + 1] - mref);
            lsum += p0 + p1;
            pk[i] = ptx::pack_bf16x2(p0, p1);
          }
          ptx::tmem_st32(tmem + lane_base + s * S_COLS + c * 32, pk);
        }
        l_sum += lsum;
        ptx::tmem_st_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&bars->p_full[s]);
      }
      // ---- epilogue: O / l -> bf16
      ptx::mbar_wait(&bars->o_full, qc & 1);
      ptx::tc_fence_after();
      const float inv = (l_sum > 0.0f) ? 1.0f / l_sum : 0.0f;
      const int head = kvh * p.group + row % p.group;
      __nv_bfloat16* dst = p.out + int64_t(tok_off + tok_local) * p.ldo + int64_t(head) * p.head_dim;
#pragma unroll
      for (int c = 0; c < DP / 32; ++c) {
        uint32_t r[32];
        ptx::tmem_ld32(tmem + lane_base + O_COL + c * 32, r);
        ptx::tmem_ld_wait();
        if (valid_row && kt_n > 0 && c * 32 < p.head_dim) {
          uint32_t pk[16];
#pragma unroll
          for (int i = 0; i < 16; ++i)
            pk[i] = ptx::pack_bf16x2(__uint_as_float(r[2 * i]) * inv, __uint_as_float(r[2 * i + 1]) * inv);
          const int n16 = min(4, (p.head_dim - c * 32) / 8);  // 16-byte stores of real columns
          uint4* d4 = reinterpret_cast<uint4*>(dst + c * 32);
          for (int i = 0; i < n16; ++i) d4[i] = make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
        }
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&bars->o_empty);
      kc += kt_n;
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) ptx::tmem_dealloc(tmem, 512);
}

}  // namespace

size_t attn_smem_bytes(int dpad) {
  return 1024 + (dpad == 128 ? AttnSmem<128>::TOTAL : AttnSmem<64>::TOTAL);
}

void launch_attention(int dpad, const AttnParams& p, int num_sms, cudaStream_t stream) {
  const int grid = p.n_work < num_sms ? p.n_work : num_sms;
  if (grid <= 0) return;
  const size_t smem = attn_smem_bytes(dpad);
  if (dpad == 128) {
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(attn_tc_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
      attr = true;
    }
    attn_tc_kernel<128><<<grid, NUM_THREADS, smem, stream>>>(p);
  } else {
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(attn_tc_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
      attr = true;
    }
    attn_tc_kernel<64><<<grid, NUM_THREADS, smem, stream>>>(p);
  }
  count_launch();
}

}  // namespace bat
