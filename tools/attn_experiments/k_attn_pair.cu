// Bipartite attention over paged prefix KV + the suffix's own KV, CTA-pair version (SURVEY
// §8(a) a5) — opt-in (BAT_ATTN=pair), head_dim 128.
//
// A cluster of two CTAs (one per SM) runs one work item = (request, KV head, q-tile pair): CTA
// rank r owns q-tile r (rows = tokens x GQA heads, as in k_attn.cu) and the pair leader issues
// tcgen05 cta_group::2 MMAs with M = 256:
//   S = Q K^T   (M=256 N=128 K=16 x 8): A = each CTA's own q-tile, B = the 128-key K tile split
//               along N — rank r stages keys [64 r, 64 r + 64) (page blocks 4r..4r+3);
//   O += P V    (M=256 N=128 K=16 x 8): A = P from each CTA's TMEM, B = the V tile split along
//               N = head_dim — rank r supplies columns [64 r, 64 r + 64) of all 128 keys.
// Per SM this halves the MMA instructions and the K/V shared-memory traffic against the 1-CTA
// kernel, and frees TMEM for DOUBLE-BUFFERED S and P: TMEM = O [0,128) S0 [128,256) S1 [256,384)
// P0 [384,448) P1 [448,512).  S_{t+2} is issued as soon as the softmax of tile t holds S_t in
// registers, P.V_t reads P from its own buffer, so the S -> softmax -> P.V chain of a tile no
// longer gates the next S (tools/attn_timeline*.py measured it on the critical path).
//
// Softmax: four warpgroups (tile parity, key half): warpgroup (w, h) handles the tiles t with
// t % 2 == w (S buffer w), 64 key columns [64 h, 64 h + 64) per row in registers; the two halves
// agree on the row max through shared memory.  The running reference max is a per-row chain
// across tiles: the tile-t warpgroup takes tile t-1's reference from shared memory (named
// barrier per warp pair), decides its own reference from its row max BEFORE computing any
// exponential (m_t = m_{t-1} unless the row max exceeds it by 2^8: lazy rescaling), publishes
// it, and only then runs the exponentials — so the two warpgroups overlap on consecutive tiles.
// A moved reference rescales O in TMEM (after the previous P.V completed); each warpgroup keeps
// its row sum relative to its own last reference and the two are combined at the item's end.
// Masks: the planner's block-skip tile states (dead / full / partial) and per-plan partial-tile
// visibility masks, exactly as in k_attn.cu.
//
// Loads: 2-D TMA (cta_group::2) of 128-byte rows — the pool / scratch pages are stored in the
// tensor-core operand layout, so a page block is copied verbatim; the peer CTA's loads signal
// the leader's full barriers, the leader's commits multicast to both CTAs' empty barriers.
// Warps: 0 Q + K loader, 1 MMA issuer (leader; converged warp, elected lane), 2 V loader,
// 3-18 softmax warpgroups (parity 0 half 0, parity 0 half 1, parity 1 half 0, parity 1 half 1).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "attn_math.cuh"
#include "common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace bat {
namespace {

constexpr int PT = 608;  // 19 warps: the register file allows 104 registers per thread
constexpr int NST = 3;            // K / V ring stages (one 128-key tile each)
constexpr int Q_BYTES = 32768;    // q-tile [2 chunks][128 rows][64] bf16, 128B-swizzled
constexpr int KH_BYTES = 16384;   // my half of a K tile: 4 page blocks (64 keys x 128)
// V: every CTA loads the whole V tile (8 page blocks, 4 KB copies: far fewer TMA requests than
// 1 KB atoms of its own column half), rank 1 shifted down by 1 KB so that ITS column chunk
// lands at the addresses where rank 0 has chunk 0 — the pair MMA reads both CTAs' B halves at
// one shared-memory address.  Stages are 33 KB apart (the shift's slack).
constexpr int V_BYTES = 32768;
constexpr int V_STRIDE = V_BYTES + 1024;
constexpr int Q_OFF = 0;          // two q-tile buffers (items alternate)
constexpr int K_OFF = Q_OFF + 2 * Q_BYTES;
constexpr int V_OFF = K_OFF + NST * KH_BYTES + 1024;
constexpr int X_OFF = V_OFF + NST * V_STRIDE;
constexpr int BAR_OFF = X_OFF + 12288;
constexpr int SMEM_TOTAL = BAR_OFF + 256;
constexpr float kThr = 8.0f;      // lazy rescale threshold (log2 units): P <= 2^8
#ifndef BAT_PAIR_POLY
#define BAT_PAIR_POLY 0           // of every 16 column pairs, exp2 on the FMA pipe (rest: MUFU; swept 0/2/4/8)
#endif

// debug timeline (bat_debug_attention_layer + BAT_ATTN_TIMELINE): event ev of global tile i, CTA 0
#define PDBG(ev, i)                                                                    \
  do {                                                                                 \
    if (p.dbg && blockIdx.x == 0 && (i) < 64) p.dbg[(ev) * 64 + (i)] = clock64();      \
  } while (0)

struct PairX {
  float mref[128];                     // reference max of the latest decided tile, per row
  float hmax[2][2][128];               // [parity][half][row]: raw row max of my key half
  float xl[2][4][128], xm[2][4][128];  // [item parity][warpgroup][row]: row sum and its reference
};
static_assert(sizeof(PairX) <= 12288, "exchange area");

struct __align__(8) PairBars {
  uint64_t q_full[2], q_empty[2];
  uint64_t k_full[NST], k_empty[NST], v_full[NST], v_empty[NST];
  uint64_t s_full[2], s_free[2], p_full[2], pv_done[2];
  uint64_t o_full, o_empty;
  uint32_t tmem_base;
};
static_assert(sizeof(PairBars) <= 256, "barrier area");

// 128-byte-row coordinate of head kvh's K (kv = 0) or V (kv = 1) block of `page` at the layer
__device__ __forceinline__ int32_t page_row(const AttnPairParams& P, int32_t page, int kv, int kvh, bool& scr) {
  const AttnParams& p = P.a;
  const int64_t blk = (int64_t(kv) * p.kv_heads + kvh) * p.head_bytes;
  scr = false;
  if (page == kZeroPage) return int32_t(P.zero_row);
  if (page >= 0) return int32_t((int64_t(page) * p.pool_page_bytes + p.pool_layer_off + blk) >> 7);
  scr = true;
  return int32_t((int64_t(-page - 1) * p.scratch_page_bytes + p.scratch_layer_off + blk) >> 7);
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(PT, 1)
    attn_pair_kernel(const __grid_constant__ AttnPairParams P) {
  const AttnParams& p = P.a;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  PairBars* bars = reinterpret_cast<PairBars*>(smem + BAR_OFF);
  PairX* X = reinterpret_cast<PairX*>(smem + X_OFF);
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();
  const uint32_t rank = ptx::cluster_ctarank();
  const int pair = blockIdx.x >> 1, n_pairs = gridDim.x >> 1;
  constexpr uint32_t IDESC_S = ptx::idesc_bf16(256, 128, 0, 0);
  constexpr uint32_t IDESC_PV = ptx::idesc_bf16(256, 128, 0, 1);

  if (warp == 0 && lane == 0) {
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&bars->q_full[i], 1);
      ptx::mbar_init(&bars->q_empty[i], 1);
      ptx::mbar_init(&bars->s_full[i], 1);
      ptx::mbar_init(&bars->p_full[i], 16);  // 8 softmax warps (both key halves) of each CTA
      ptx::mbar_init(&bars->s_free[i], 16);  // the same warps, once they hold S in registers
      ptx::mbar_init(&bars->pv_done[i], 1);  // pair commit: P.V of the P buffer done
    }
    for (int i = 0; i < NST; ++i) {
      ptx::mbar_init(&bars->k_full[i], 1);
      ptx::mbar_init(&bars->k_empty[i], 1);
      ptx::mbar_init(&bars->v_full[i], 1);
      ptx::mbar_init(&bars->v_empty[i], 1);
    }
    ptx::mbar_init(&bars->o_full, 1);
    ptx::mbar_init(&bars->o_empty, 32);  // 16 softmax warps of each CTA
    ptx::fence_mbar_init();
    ptx::prefetch_tmap(&P.tm_pool_k);
    ptx::prefetch_tmap(&P.tm_pool_v);
    ptx::prefetch_tmap(&P.tm_scr_k);
    ptx::prefetch_tmap(&P.tm_scr_v);
    ptx::prefetch_tmap(&P.tm_q);
  }
  if (warp == 1) ptx::tmem_alloc2(&bars->tmem_base, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem = bars->tmem_base;
  const int32_t* img = p.img;
  const int32_t* work = img + p.off_work;
  auto next_item = [&](int w) {
    for (w += n_pairs; w < p.n_work; w += n_pairs)
      if (work[int64_t(w) * 8 + 5] > 0) break;
    return w;
  };
  auto first_item = [&]() {
    int w = pair;
    if (w < p.n_work && work[int64_t(w) * 8 + 5] == 0) w = next_item(w);
    return w;
  };

  if (warp == 0 || warp == 2) {  // ---------------------------------------------- loaders
    const bool kq = warp == 0;
    const uint32_t leader = 0;
    uint32_t it = 0, t = 0;
    for (int w = first_item(); w < p.n_work; w = next_item(w), ++it) {
      const WorkItem wi = load_work(work, w);
      if (kq && lane == 0) {  // my q-tile (rank 1 of a single-q-tile item reloads q-tile 0)
        const uint32_t qb = it & 1;
        ptx::mbar_wait(&bars->q_empty[qb], ((it >> 1) & 1) ^ 1);
        if (rank == 0) ptx::mbar_expect_tx(&bars->q_full[qb], 2 * Q_BYTES);
        const int qi = (rank == 1 && wi.q1 >= 0) ? wi.q1 : wi.q0;
        const int qtile0 = img[p.off_qinfo + int64_t(wi.b) * 8 + 2];
        const int32_t row = int32_t((int64_t(qtile0 + qi) * p.kv_heads + wi.kvh) * (Q_BYTES / 128));
        ptx::tma_load_2d_pair(smem + Q_OFF + qb * Q_BYTES, &P.tm_q, 0, row,
                              ptx::mapa(ptx::smem_u32(&bars->q_full[qb]), leader));
      }
      int32_t pid = lane < kKtilePages ? img[wi.tp_off + lane] : 0;
      for (int x = 0; x < wi.kt_n; ++x, ++t) {
        const int32_t pid_next = (lane < kKtilePages && x + 1 < wi.kt_n) ? img[wi.tp_off + (x + 1) * kKtilePages + lane] : 0;
        const uint32_t st = t % NST, ph = (t / NST) & 1;
        if (kq) {
          int32_t rows[4];
          bool scr[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) rows[i] = page_row(P, __shfl_sync(0xffffffffu, pid, 4 * rank + i), 0, wi.kvh, scr[i]);
          if (lane == 0) {
            ptx::mbar_wait(&bars->k_empty[st], ph ^ 1);
            PDBG(10, t);
            if (rank == 0) ptx::mbar_expect_tx(&bars->k_full[st], 2 * KH_BYTES);
            const uint32_t bar = ptx::mapa(ptx::smem_u32(&bars->k_full[st]), leader);
            uint8_t* dst = smem + K_OFF + st * KH_BYTES;
#pragma unroll
            for (int i = 0; i < 4; ++i)
              ptx::tma_load_2d_pair(dst + i * 4096, scr[i] ? &P.tm_scr_k : &P.tm_pool_k, 0, rows[i], bar);
          }
        } else {
          int32_t rows[8];
          bool scr[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) rows[i] = page_row(P, __shfl_sync(0xffffffffu, pid, i), 1, wi.kvh, scr[i]);
          if (lane == 0) {
            ptx::mbar_wait(&bars->v_empty[st], ph ^ 1);
            PDBG(11, t);
            if (rank == 0) ptx::mbar_expect_tx(&bars->v_full[st], 2 * V_BYTES);
            const uint32_t bar = ptx::mapa(ptx::smem_u32(&bars->v_full[st]), leader);
            // page block [2 slot groups][2 column chunks][8][64]; my chunk `rank` of slot group g
            // of page i must land at stage + 4096 i + 2048 g
            uint8_t* dst = smem + V_OFF + st * V_STRIDE - int(rank) * 1024;
#pragma unroll
            for (int i = 0; i < 8; ++i)
              ptx::tma_load_2d_pair(dst + i * 4096, scr[i] ? &P.tm_scr_v : &P.tm_pool_v, 0, rows[i], bar);
          }
        }
        __syncwarp();
        pid = pid_next;
      }
    }
  } else if (warp == 1) {  // ------------------------------------- pair MMA issuer (leader)
    if (rank == 0) {
      const uint32_t sq0 = ptx::smem_u32(smem + Q_OFF);
      const uint32_t tO = tmem;
      // Event loop over two cursors walking the pair's tiles: S(g) is issued as soon as the
      // softmax of tile g-2 released S buffer g & 1 (s_free), its item's q-tile and K tile are
      // resident and P.V(g-4) has been issued (so when tile g's softmax runs, P.V(g-4) is
      // complete: every pv_done wait below is unambiguous); P.V(g) as soon as P(g) and V(g) are
      // ready.  Neither stream blocks the other.
      struct Cur {
        int w;
        WorkItem wi;
        uint32_t it, g;
        int x;
      };
      auto start = [&](Cur& c) {
        c.w = first_item();
        c.wi = c.w < p.n_work ? load_work(work, c.w) : WorkItem{0, 0, -1, -1, 0, 0, 0, 0};
        c.it = 0;
        c.g = 0;
        c.x = 0;
      };
      auto advance = [&](Cur& c) {  // returns true when it moved to the next item
        ++c.g;
        if (++c.x < c.wi.kt_n) return false;
        c.w = next_item(c.w);
        c.wi = c.w < p.n_work ? load_work(work, c.w) : WorkItem{0, 0, -1, -1, 0, 0, 0, 0};
        ++c.it;
        c.x = 0;
        return true;
      };
      auto ready = [&](uint64_t* bar, uint32_t parity) {
        return __shfl_sync(0xffffffffu, int(ptx::mbar_test(bar, parity)), 0) != 0;
      };
      uint32_t total = 0;
      for (int w = first_item(); w < p.n_work; w = next_item(w)) total += uint32_t(work[int64_t(w) * 8 + 5]);
      Cur sc, pc;
      start(sc);
      start(pc);
      bool sq_ok = false;
      while (pc.g < total) {
        bool prog = false;
        if (sc.g < total) {
          const uint32_t g = sc.g, st = g % NST, qb = sc.it & 1;
          bool ok = g < 2 || ready(&bars->s_free[g & 1], ((g - 2) >> 1) & 1);
          if (ok && g >= 4) ok = pc.g > g - 4;
          if (ok && !sq_ok) ok = sq_ok = ready(&bars->q_full[qb], (sc.it >> 1) & 1);
          if (ok) ok = ready(&bars->k_full[st], (g / NST) & 1);
          if (ok) {
            PDBG(12, g);
            ptx::tc_fence_after();
            const uint32_t sq = sq0 + qb * Q_BYTES;
            const uint32_t sk = ptx::smem_u32(smem + K_OFF + st * KH_BYTES);
            const uint32_t tS = tmem + 128 + (g & 1) * 128;
#pragma unroll
            for (int kk = 0; kk < 8; ++kk)
              ptx::mma2_ss_elect(tS, ptx::desc_sw128(sq + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024),
                                 ptx::desc_sw128(sk + (kk >> 2) * 1024 + (kk & 3) * 32, 16, 2048), IDESC_S, kk ? 1u : 0u);
            ptx::mma2_commit_elect(&bars->s_full[g & 1], 3);
            PDBG(0, g);
            ptx::mma2_commit_elect(&bars->k_empty[st], 3);
            if (sc.x == sc.wi.kt_n - 1) ptx::mma2_commit_elect(&bars->q_empty[qb], 3);
            if (advance(sc)) sq_ok = false;
            prog = true;
          }
        }
        if (pc.g < sc.g) {
          const uint32_t g = pc.g, st = g % NST, b = g & 1;
          bool ok = ready(&bars->p_full[b], (g >> 1) & 1);
          if (ok && pc.x == 0) ok = ready(&bars->o_empty, (pc.it & 1) ^ 1);
          if (ok) ok = ready(&bars->v_full[st], (g / NST) & 1);
          if (ok) {
            PDBG(2, g);
            ptx::tc_fence_after();
            const uint32_t sv = ptx::smem_u32(smem + V_OFF + st * V_STRIDE);
            const uint32_t tP = tmem + 384 + b * 64;
#pragma unroll
            for (int i = 0; i < 8; ++i)
              ptx::mma2_ts_elect(tO, tP + (i >> 2) * 32 + (i & 3) * 8, ptx::desc_sw128(sv + i * 4096, 1024, 2048),
                                 IDESC_PV, (pc.x > 0 || i > 0) ? 1u : 0u);
            ptx::mma2_commit_elect(&bars->pv_done[b], 3);
            PDBG(4, g);
            ptx::mma2_commit_elect(&bars->v_empty[st], 3);
            if (pc.x == pc.wi.kt_n - 1) ptx::mma2_commit_elect(&bars->o_full, 3);
            advance(pc);
            prog = true;
          }
        }
        if (!prog) __nanosleep(20);
      }
    }
  } else if (warp >= 3) {  // -------------------------------------------- softmax warpgroups
    // warpgroup (par, h): tiles t with t % 2 == par (S buffer par), key half h (S columns
    // [64 h, 64 h + 64)); thread = one row of my CTA's q-tile
    const int wgi = (warp - 3) >> 2;  // warps 3-18: any 4 consecutive warps cover the 4 TMEM lane quadrants
    const int par = wgi >> 1, h = wgi & 1;
    const uint32_t sub = warp & 3;
    const int row = sub * 32 + lane;
    const uint32_t lane_base = (sub * 32) << 16;
    const uint32_t tS = tmem + 128 + par * 128 + h * 64 + lane_base;  // my S half
    const uint32_t tO = tmem + lane_base;
    // named barriers: 1-4 / 5-8 the reference chain into parity 0 / 1 (per sub; 128 threads:
    // both key halves of both parities — it also publishes the halves' row maxima to each
    // other), 9 the item-end rendezvous, 10-13 the halves' max exchange of tile 0 (no chain yet)
    const uint32_t id_in = 1 + par * 4 + sub, id_out = 1 + (par ^ 1) * 4 + sub;
    const uint32_t p_full_leader = ptx::mapa(ptx::smem_u32(&bars->p_full[par]), 0);
    const uint32_t s_free_leader = ptx::mapa(ptx::smem_u32(&bars->s_free[par]), 0);
    const uint32_t tP = tmem + 384 + par * 64 + h * 32 + lane_base;  // my P half (bf16 pairs)
    const uint32_t o_empty_leader = ptx::mapa(ptx::smem_u32(&bars->o_empty), 0);
    const uint64_t sc2 = pk2(p.scale_log2, p.scale_log2);
    uint32_t total = 0;  // tiles of this pair (the last one publishes no reference)
    for (int w = first_item(); w < p.n_work; w = next_item(w)) total += uint32_t(work[int64_t(w) * 8 + 5]);
    uint32_t t = 0, it = 0;
    for (int w = first_item(); w < p.n_work; w = next_item(w), ++it) {
      const WorkItem wi = load_work(work, w);
      const int qi = rank == 0 ? wi.q0 : wi.q1;
      const bool active = qi >= 0;
      const int32_t* q_info = img + p.off_qinfo + int64_t(wi.b) * 8;
      const int tok_off = q_info[0], S = q_info[1];
      const int tok_local = (active ? qi : 0) * p.qt + row / p.group;
      const bool valid_row = active && row < p.qt * p.group && tok_local < S;
      const int mrow = valid_row ? row / p.group : p.qt;
      const int32_t* ktl = img + wi.kt_off;
      float l_own = 0.0f, m_own = -INFINITY;
      auto mask_of = [&](int mid) {  // my half's 64 visibility bits of a partial tile
        return __ldg(reinterpret_cast<const uint2*>(img + p.off_masks + (int64_t(mid) * (p.qt + 1) + mrow) * 4) + h);
      };
      const int x0 = int((t & 1) != uint32_t(par));  // my first tile of this item
      int n_state = 0, n_mid = 0;
      uint2 n_mv = make_uint2(~0u, ~0u);
      if (x0 < wi.kt_n && active) {
        n_state = (ktl[x0] >> (24 + 2 * int(rank))) & 3;
        n_mid = img[wi.km_off + 2 * x0 + int(rank)];
        if (n_state == 2) n_mv = mask_of(n_mid);
      }
      for (int x = 0; x < wi.kt_n; ++x, ++t) {
        if (int(t & 1) != par) continue;
        const int state = n_state;
        const uint2 mv = n_mv;
        if (x + 2 < wi.kt_n && active) {  // the next own tile's state / mask id, issued now
          n_state = (ktl[x + 2] >> (24 + 2 * int(rank))) & 3;
          n_mid = img[wi.km_off + 2 * (x + 2) + int(rank)];
        } else {
          n_state = 0;
        }
        const bool dl = h == 0 && sub == 0 && lane == 0;
        if (dl) PDBG(5, t);
        ptx::mbar_wait(&bars->s_full[par], (t >> 1) & 1);
        if (dl) PDBG(6, t);
        ptx::tc_fence_after();
        // pass 1: my half's row max (S is read again for the exponentials: keeping 64 scores
        // live across the reference chain would not fit the register budget of 20 warps)
        float mt = -INFINITY;
        if (state != 0) {
          uint32_t r[32], q[32];
          ptx::tmem_ld32(tS, r);
          ptx::tmem_ld32(tS + 32, q);
          ptx::tmem_ld_wait();
          if (state == 2) {
#pragma unroll
            for (int i = 0; i < 32; ++i) {
              r[i] = ((mv.x >> i) & 1u) ? r[i] : 0xff800000u;
              q[i] = ((mv.y >> i) & 1u) ? q[i] : 0xff800000u;
            }
          }
          float m0 = -INFINITY, m1 = -INFINITY, m2 = -INFINITY, m3 = -INFINITY;
#pragma unroll
          for (int i = 0; i < 32; i += 4) {
            m0 = fmax3(m0, __uint_as_float(r[i]), __uint_as_float(r[i + 1]));
            m1 = fmax3(m1, __uint_as_float(r[i + 2]), __uint_as_float(r[i + 3]));
            m2 = fmax3(m2, __uint_as_float(q[i]), __uint_as_float(q[i + 1]));
            m3 = fmax3(m3, __uint_as_float(q[i + 2]), __uint_as_float(q[i + 3]));
          }
          mt = fmaxf(fmax3(m0, m1, m2), m3);
        }
        // ---- row max over both halves, then the reference chain (tile t-1 -> t), both decided
        // before any exponential
        X->hmax[par][h][row] = mt;
        if (dl) PDBG(7, t);
        float m_prev = -INFINITY;
        if (t > 0) {
          ptx::bar_sync(id_in, 128);
          if (x > 0) m_prev = X->mref[row];
        } else {
          ptx::bar_sync(10 + sub, 64);
        }
        mt = fmaxf(mt, X->hmax[par][h ^ 1][row]);
        if (dl) PDBG(8, t);
        const float mts = mt * p.scale_log2;
        const float m_new = (mts > m_prev + kThr) ? mts : m_prev;
        if (h == 0) X->mref[row] = m_new;  // both halves decide the same value
        if (t + 1 < total) ptx::bar_arrive(id_out, 128);
        // O holds this item's earlier tiles relative to m_prev: rescale my 64 O columns
        const bool need_o = x > 0 && m_prev != -INFINITY && m_new != m_prev;
        if (__any_sync(0xffffffffu, need_o)) {
          // P.V of tile t-1 (and all before) done.  Its P buffer's barrier completes for t-3 and
          // then t-1; P.V(t-4), hence t-5, is complete (S_t was issued after P.V(t-4)), so waiting
          // for t-3 and then t-1 is unambiguous.
          if (t >= 3) ptx::mbar_wait(&bars->pv_done[(t - 1) & 1], ((t - 3) >> 1) & 1);
          ptx::mbar_wait(&bars->pv_done[(t - 1) & 1], ((t - 1) >> 1) & 1);
          ptx::tc_fence_after();
          const float a = need_o ? ex2(m_prev - m_new) : 1.0f;
#pragma unroll 1
          for (int c = 0; c < 2; ++c) {
            uint32_t o[32];
            ptx::tmem_ld32(tO + h * 64 + c * 32, o);
            ptx::tmem_ld_wait();
#pragma unroll
            for (int i = 0; i < 32; ++i) o[i] = __float_as_uint(__uint_as_float(o[i]) * a);
            ptx::tmem_st32(tO + h * 64 + c * 32, o);
          }
        }
        // ---- P = 2^(s * scale - m_new) as bf16 into my half of P buffer par.  S_t is read into
        // registers first and released (s_free) so the next S can overwrite it while the
        // exponentials run; P buffer par is free once P.V of tile t-2 completed.
        float lsum = 0.0f;
        uint32_t pk[2][16];
        if (state != 0) {
          const float mu = (m_new == -INFINITY) ? 0.0f : m_new;
          const uint64_t nm2 = pk2(-mu, -mu);
          uint64_t acc0 = pk2(0.0f, 0.0f), acc1 = acc0;
#pragma unroll
          for (int c = 0; c < 2; ++c) {
            uint32_t r[32];
            ptx::tmem_ld32(tS + c * 32, r);
            ptx::tmem_ld_wait();
            if (c == 1) {  // all of S_t is in registers: release the buffer
              ptx::tc_fence_before();
              __syncwarp();
              if (lane == 0) ptx::mbar_arrive_remote(s_free_leader);
            }
            if (state == 2) {
              const uint32_t vw = c ? mv.y : mv.x;
#pragma unroll
              for (int i = 0; i < 32; ++i) r[i] = ((vw >> i) & 1u) ? r[i] : 0xff800000u;
            }
#pragma unroll
            for (int i = 0; i < 16; ++i) {
              const uint32_t ra = r[2 * i], rb = r[2 * i + 1];
              const uint64_t xv = ffma2(pk2(__uint_as_float(ra), __uint_as_float(rb)), sc2, nm2);
              uint64_t e;
              if (i < BAT_PAIR_POLY) {
                e = exp2_poly2(xv);
                if (state == 2) {  // the polynomial clamps at -127: re-zero masked lanes
                  float p0, p1;
                  up2(e, p0, p1);
                  e = pk2(ra == 0xff800000u ? 0.0f : p0, rb == 0xff800000u ? 0.0f : p1);
                }
              } else {
                float x0f, x1f;
                up2(xv, x0f, x1f);
                e = pk2(ex2(x0f), ex2(x1f));
              }
              if (i & 1) acc1 = fadd2(acc1, e);
              else acc0 = fadd2(acc0, e);
              float p0, p1;
              up2(e, p0, p1);
              pk[c][i] = ptx::pack_bf16x2(p0, p1);
            }
          }
          float a0, a1, b0, b1;
          up2(acc0, a0, a1);
          up2(acc1, b0, b1);
          lsum = (a0 + a1) + (b0 + b1);
        } else {
          ptx::tc_fence_before();
          __syncwarp();
          if (lane == 0) ptx::mbar_arrive_remote(s_free_leader);
#pragma unroll
          for (int i = 0; i < 16; ++i) pk[0][i] = pk[1][i] = 0u;
        }
        if (t >= 2) ptx::mbar_wait(&bars->pv_done[par], ((t >> 1) + 1) & 1);  // P.V of tile t-2 read P buffer par
        ptx::tc_fence_after();
#pragma unroll
        for (int c = 0; c < 2; ++c)
          asm volatile(
              "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
              "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(tP + c * 16),
              "r"(pk[c][0]), "r"(pk[c][1]), "r"(pk[c][2]), "r"(pk[c][3]), "r"(pk[c][4]), "r"(pk[c][5]), "r"(pk[c][6]),
              "r"(pk[c][7]), "r"(pk[c][8]), "r"(pk[c][9]), "r"(pk[c][10]), "r"(pk[c][11]), "r"(pk[c][12]),
              "r"(pk[c][13]), "r"(pk[c][14]), "r"(pk[c][15]));
        if (l_own > 0.0f && m_own != m_new) l_own *= ex2(m_own - m_new);
        l_own += lsum;
        m_own = m_new;
        ptx::tmem_st_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (dl) PDBG(9, t);
        if (lane == 0) ptx::mbar_arrive_remote(p_full_leader);
        if (dl) PDBG(13, t);
        n_mv = make_uint2(~0u, ~0u);
        if (n_state == 2) n_mv = mask_of(n_mid);
      }
      // ---- item end: combine the four partial row sums; O / l -> bf16, 32 columns per warpgroup
      const uint32_t ib = it & 1;
      X->xl[ib][wgi][row] = l_own;
      X->xm[ib][wgi][row] = m_own;
      ptx::bar_sync(9, 512);
      float mf = -INFINITY;
#pragma unroll
      for (int g = 0; g < 4; ++g) mf = fmaxf(mf, X->xm[ib][g][row]);
      float lt = 0.0f;
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        const float lg = X->xl[ib][g][row];
        lt += lg > 0.0f ? lg * ex2(X->xm[ib][g][row] - mf) : 0.0f;
      }
      const float inv = lt > 0.0f ? 1.0f / lt : 0.0f;
      ptx::mbar_wait(&bars->o_full, it & 1);
      ptx::tc_fence_after();
      const int head = wi.kvh * p.group + row % p.group;
      const int col0 = wgi * 32;
      __nv_bfloat16* dst = p.out + int64_t(tok_off + tok_local) * p.ldo + int64_t(head) * p.head_dim + col0;
      uint32_t o[32];
      ptx::tmem_ld32(tO + col0, o);
      ptx::tmem_ld_wait();
      if (valid_row) {
        uint32_t pk[16];
#pragma unroll
        for (int i = 0; i < 16; ++i)
          pk[i] = ptx::pack_bf16x2(__uint_as_float(o[2 * i]) * inv, __uint_as_float(o[2 * i + 1]) * inv);
        uint4* d4 = reinterpret_cast<uint4*>(dst);
#pragma unroll
        for (int i = 0; i < 4; ++i) d4[i] = make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive_remote(o_empty_leader);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::cluster_sync();  // no CTA leaves while its peer's MMAs / signals may still target it
  if (warp == 1) ptx::tmem_dealloc2(tmem, 512);
}

}  // namespace

// Opt-in (BAT_ATTN=pair): measured on the configs[1] bench step it reaches 534 TFLOP/s against
// 613 for the 1-CTA kernel — its per-parity S -> softmax -> P.V chain is still exposed (the two
// S buffers give one tile of slack; the 128-key softmax of a tile takes ~2.4k clk), see
// DESIGN.md §5.1 and profiles/r1_attn_kernels.txt.
bool attn_pair_supported(int dpad) {
  static const bool on = [] {
    const char* e = getenv("BAT_ATTN");
    return e && e[0] == 'p';
  }();
  return dpad == 128 && on;
}

int attn_grid_slots(int dpad, int num_sms) { return attn_pair_supported(dpad) ? num_sms / 2 : num_sms; }

void launch_attention_pair(const AttnPairParams& P, int num_sms, cudaStream_t stream) {
  const int max_pairs = num_sms / 2;
  const int pairs = P.a.n_work < max_pairs ? P.a.n_work : max_pairs;
  if (pairs <= 0) return;
  const size_t smem = 1024 + SMEM_TOTAL;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_pair_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    attr = true;
  }
  attn_pair_kernel<<<2 * pairs, PT, smem, stream>>>(P);
  count_launch();
}

}  // namespace bat
