// Bipartite attention over paged prefix KV + the suffix's own KV (
// PAPER.md P:207).
//
// One work item = (request b, KV head, a pair of packed q-tiles).  A q-tile is 128 rows =
// qt suffix tokens x the g query heads sharing the KV head (GQA packing).  Both q-tiles of
// the pair share every 128-key K/V tile the loader brings in (halving K/V traffic per FLOP).
// The plan lists the pair's live k-tiles (block-skip: dead tiles never reach the kernel)
// with a state per q-tile: 0 dead (P = 0), 1 full (no element mask), 2 partial: the element
// mask  kord <= rord && (kseg == rseg || (kseg|rseg) < 0)  precomputed once per plan by
// launch_masks (shared by all KV heads and layers); a row reads its 64 bits per tile.
//
// Warp roles (640 threads, one CTA per SM, persistent over work items, FA4-style):
//   warps 0,2,3 loaders, three independent streams: warp 0 Q and K (a 3-tile ring), warps 2 / 3
//               the first / second V half of every tile (a 3-slot ring of 64-key halves; the
//               tile's key metadata rides with the first half).  One bulk copy per page block:
//               pages are stored in the tensor-core operand layout (128-byte swizzle,
//               ptx::page_blk_off), so a block drops into shared memory ready for tcgen05.mma
//               (8-row-group stride Dp/64 KB).  Page ids are read three tiles ahead and the
//               blocks of the tile two ahead are prefetched into L2.
//   warp 1      MMA issuer (one thread): S0 = Q0 K^T, S1 = Q1 K^T (SS, M=128 N=128 K=16) and
//               O0 += P0 V, O1 += P1 V (TS: P read from TMEM, V MN-major from smem), issued as
//               S0_0 S1_0 | PV0_j S0_{j+1} PV1_j S1_{j+1} | ... so the softmax of one q-tile
//               runs while the tensor core serves the other.
//   warps 4-19  four softmax warpgroups: q-tile q = wg & 1, key half h = wg >> 1.  Thread
//               (q, h, row) owns the 64 S columns [64h, 64h+64) of one row: exp2 of its half
//               against the row's reference max, P as bf16 into TMEM columns [64h, 64h+32) of
//               the S buffer, and the O columns [DP/2 h, DP/2 (h+1)) for rescaling and the
//               epilogue.  The two halves of a row agree on the reference max through shared
//               memory and a 64-thread named barrier per warp pair; the reference max only
//               moves when a row's exponent would exceed 2^8 (lazy rescaling).
// TMEM (512 columns): S0 [0,128) S1 [128,256) O0 [256,384) O1 [384,512).
#include <cstdlib>
#include <string>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "common.h"
#include "kernels.h"
#include "ptx.cuh"
#include "attn_math.cuh"

namespace bat {
namespace {

constexpr int NUM_THREADS = 640;
constexpr int NCH = 2;  // 32-column S chunks per softmax thread (half of a 128-key row)
constexpr float kRescaleThreshold = 8.0f;  // log2 units: P <= 2^8 between rescales
#ifndef BAT_ATTN_L2PF
#define BAT_ATTN_L2PF 0  // 1: prefetch the K/V blocks of the tile two ahead into L2 (measured slower)
#endif
#ifndef BAT_ATTN_NOMASK
#define BAT_ATTN_NOMASK 0  // timing experiment: partial tiles take the unmasked path (wrong results)
#endif
#ifndef BAT_ATTN_NOLOAD
#define BAT_ATTN_NOLOAD 0  // timing experiment: skip the K / V copies (wrong results)
#endif
#ifndef BAT_SUMCHECK
#define BAT_SUMCHECK 0  // 1: fast-path bound from the row-half sum instead of a per-element max (measured equal: 598.7 vs 601.0 TFLOP/s)
#endif
#ifndef BAT_LOADER_SLEEP
#define BAT_LOADER_SLEEP 0  // 1: loader warps wait on their ring barriers with a suspend hint
#endif
#if BAT_LOADER_SLEEP
#define BAT_LWAIT(b, ph) ptx::mbar_wait_sleep(b, ph)
#else
#define BAT_LWAIT(b, ph) ptx::mbar_wait(b, ph)
#endif
#ifndef BAT_SOFT_SLEEP
#define BAT_SOFT_SLEEP 0  // 1: softmax warps wait for S / O with a suspend hint instead of re-polling
#endif
#if BAT_SOFT_SLEEP
#define BAT_SWAIT(b, ph) ptx::mbar_wait_sleep(b, ph)
#else
#define BAT_SWAIT(b, ph) ptx::mbar_wait(b, ph)
#endif
#ifndef BAT_ATTN_DBE
#define BAT_ATTN_DBE 1  // 1: decide-before-exp softmax (row max -> halves exchange -> P per chunk); 0: single pass + vote
#endif
#ifndef BAT_POLY_PAIRS
#define BAT_POLY_PAIRS 2  // of every 16 column pairs, exp2 on the FMA pipe (rest: MUFU); swept 0/2/4/8: 600/613/604/542 TFLOP/s
#endif

template <int DP>
struct AttnSmem {
  static constexpr int CHUNKS = DP / 64;
  static constexpr int TILE_BYTES = CHUNKS * 128 * 128;  // Q: [CHUNKS][128 rows][64] bf16
  // K / V tiles: 8 page blocks [2 slot groups][CHUNKS][8][64] (ptx::page_blk_off), i.e. 16
  // 8-row groups at stride GROUP_BYTES, chunk c of a group at +c * 1024
  static constexpr int PAGE_BYTES = CHUNKS * 2048;
  static constexpr int GROUP_BYTES = CHUNKS * 1024;
  static constexpr int HALF_BYTES = TILE_BYTES / 2;        // 4 pages = 64 keys
  static constexpr int KST = 3;                            // K ring: whole tiles (S needs N = 128 contiguous keys)
  static constexpr int VST = 3;                            // V ring: half tiles (P.V runs 16 keys per MMA)
  static constexpr int Q_OFF = 0;                          // Q0, Q1
  static constexpr int K_OFF = Q_OFF + 2 * TILE_BYTES;
  static constexpr int V_OFF = K_OFF + KST * TILE_BYTES;
  static constexpr int XCH_OFF = V_OFF + VST * HALF_BYTES;  // row-half exchange (see XchSmem)
  static constexpr int BAR_OFF = XCH_OFF + 8192;
  static constexpr int TOTAL = BAR_OFF + 256;
};
static_assert(AttnSmem<128>::TOTAL + 1024 <= 232448, "attention shared memory");

// exchange between the two key halves of a row ([parity][q][h]...)
struct XchSmem {
  float rmax[2][2][2][128];  // partial raw row maxima (slow path)
  int ok[2][2][2][4];        // per-warp "all exponents <= threshold" votes (fast path)
  float lsum[2][2][128];     // partial row sums (epilogue)
};
static_assert(sizeof(XchSmem) <= 8192, "exchange area");

struct __align__(8) AttnBars {
  uint64_t q_full, q_empty;
  uint64_t k_full[3], k_empty[3], v_full[3], v_empty[3];
  uint64_t s_full[2], p_full[2], o_full[2], o_empty[2];
  uint64_t seq[2];  // softmax turn token: seq[q] completes when it is q-tile team q's turn
  uint32_t tmem_base;
};
static_assert(sizeof(AttnBars) <= 256, "barrier area");
#ifndef BAT_ATTN_SEQ
#define BAT_ATTN_SEQ 0  // 1: the two q-tile softmax teams take turns (FA4-style); measured 543 vs 600 TFLOP/s
                        // 2: only their exp phases (DBE: after the reference decision, until P is stored) take turns
#endif

// ring positions: K tile g -> slot g % 3; V half h (= 2 g + {0,1}) -> slot h % 3
__device__ __forceinline__ uint32_t ring_slot(uint32_t i) { return i % 3u; }
__device__ __forceinline__ uint32_t ring_phase(uint32_t i) { return (i / 3u) & 1u; }

__device__ __forceinline__ const char* resolve_page(const AttnParams& p, int32_t page) {
  if (page == kZeroPage) return p.zero_page;
  if (page >= 0) return p.pool + int64_t(page) * p.pool_page_bytes + p.pool_layer_off;
  return p.scratch + int64_t(-page - 1) * p.scratch_page_bytes + p.scratch_layer_off;
}

#define DBG(ev, x)                                                                       \
  do {                                                                                   \
    if (p.dbg && blockIdx.x == 0 && (x) < 64 && dbg_first) p.dbg[(ev) * 64 + (x)] = clock64(); \
  } while (0)

// ---- softmax passes over one 128-column S row held in TMEM (one row per thread) ----------
// Row max of the raw scores; MASKED applies the visibility bits.
template <bool MASKED, int NC>
__device__ __forceinline__ float row_max(uint32_t tS, const uint32_t (&vis)[NC]) {
  float mt = -INFINITY;
#pragma unroll
  for (int c = 0; c < NC; c += 2) {
    uint32_t r[32], q[32];
    ptx::tmem_ld32(tS + c * 32, r);
    ptx::tmem_ld32(tS + (c + 1) * 32, q);
    ptx::tmem_ld_wait();
    if (MASKED) {
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        r[i] = ((vis[c] >> i) & 1u) ? r[i] : 0xff800000u;  // -inf
        q[i] = ((vis[c + 1] >> i) & 1u) ? q[i] : 0xff800000u;
      }
    }
    float m0 = mt, m1 = -INFINITY, m2 = -INFINITY, m3 = -INFINITY;
#pragma unroll
    for (int i = 0; i < 32; i += 4) {
      m0 = fmax3(m0, __uint_as_float(r[i]), __uint_as_float(r[i + 1]));
      m1 = fmax3(m1, __uint_as_float(r[i + 2]), __uint_as_float(r[i + 3]));
      m2 = fmax3(m2, __uint_as_float(q[i]), __uint_as_float(q[i + 1]));
      m3 = fmax3(m3, __uint_as_float(q[i + 2]), __uint_as_float(q[i + 3]));
    }
    mt = fmaxf(fmax3(m0, m1, m2), m3);
  }
  return mt;
}

// P = exp2(s * scale - mref) written as bf16 pairs into the row's first 64 TMEM columns
// (columns [16c, 16c+16) after S columns [32c, 32c+32) were read); returns the row sum.
template <bool MASKED, int NC>
__device__ __forceinline__ float row_exp(uint32_t tS, const uint32_t (&vis)[NC], uint64_t sc2, uint64_t nm2) {
  uint64_t acc0 = pk2(0.0f, 0.0f), acc1 = acc0;
  uint32_t ra[32], rb[32];
  ptx::tmem_ld32(tS, ra);
  ptx::tmem_ld_wait();
#pragma unroll
  for (int c = 0; c < NC; ++c) {
    uint32_t (&r)[32] = (c & 1) ? rb : ra;
    uint32_t (&rn)[32] = (c & 1) ? ra : rb;
    if (c + 1 < NC) ptx::tmem_ld32(tS + (c + 1) * 32, rn);  // in flight while chunk c computes
    uint32_t pk[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      const uint64_t xv = ffma2(pk2(__uint_as_float(r[2 * i]), __uint_as_float(r[2 * i + 1])), sc2, nm2);
      uint64_t e;
      if (i < BAT_POLY_PAIRS) {
        e = exp2_poly2(xv);
      } else {
        float x0, x1;
        up2(xv, x0, x1);
        e = pk2(ex2(x0), ex2(x1));
      }
      float p0, p1;
      up2(e, p0, p1);
      if (MASKED) {
        p0 = ((vis[c] >> (2 * i)) & 1u) ? p0 : 0.0f;
        p1 = ((vis[c] >> (2 * i + 1)) & 1u) ? p1 : 0.0f;
        e = pk2(p0, p1);
      }
      if (i & 1) acc1 = fadd2(acc1, e);
      else acc0 = fadd2(acc0, e);
      pk[i] = ptx::pack_bf16x2(p0, p1);
    }
    // P columns [16c, 16c+16): S columns already consumed (chunk c+1 reads [32c+32, 32c+64))
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
        "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(tS + c * 16),
        "r"(pk[0]), "r"(pk[1]), "r"(pk[2]), "r"(pk[3]), "r"(pk[4]), "r"(pk[5]), "r"(pk[6]), "r"(pk[7]),
        "r"(pk[8]), "r"(pk[9]), "r"(pk[10]), "r"(pk[11]), "r"(pk[12]), "r"(pk[13]), "r"(pk[14]),
        "r"(pk[15]));
    if (c + 1 < NC) ptx::tmem_ld_wait();
  }
  float a0, a1, b0, b1;
  up2(acc0, a0, a1);
  up2(acc1, b0, b1);
  return (a0 + a1) + (b0 + b1);
}

// Single-pass variant against the current reference max: computes all of P in registers and
// tracks the row's largest exponent; P is written to TMEM only if no visible exponent exceeds
// `limit` (the lazy-rescale threshold) — the common case once the running max has settled.
// Returns false (nothing written, S intact) when the caller must take the two-pass path.
template <bool MASKED, int NC, class Agree>
__device__ __forceinline__ bool row_exp_opt(uint32_t tS, const uint32_t (&vis)[NC], uint64_t sc2, uint64_t nm2,
                                            float limit, float& lsum, Agree&& agree) {
  uint64_t acc0 = pk2(0.0f, 0.0f), acc1 = acc0;
  uint32_t pk[NC * 16];
  float xm0 = -INFINITY, xm1 = -INFINITY;
#pragma unroll
  for (int c = 0; c < NC; ++c) {
    uint32_t r[32];
    ptx::tmem_ld32(tS + c * 32, r);
    ptx::tmem_ld_wait();
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      uint64_t xv = ffma2(pk2(__uint_as_float(r[2 * i]), __uint_as_float(r[2 * i + 1])), sc2, nm2);
      float x0, x1;
      up2(xv, x0, x1);
      if (MASKED) {
        x0 = ((vis[c] >> (2 * i)) & 1u) ? x0 : -INFINITY;
        x1 = ((vis[c] >> (2 * i + 1)) & 1u) ? x1 : -INFINITY;
        xv = pk2(x0, x1);
      }
      if (!BAT_SUMCHECK) {
        if (i & 1) xm1 = fmax3(xm1, x0, x1);
        else xm0 = fmax3(xm0, x0, x1);
      }
      uint64_t e;
      if (i < BAT_POLY_PAIRS) {
        e = exp2_poly2(xv);
        if (MASKED) {  // the polynomial clamps at -126: re-zero masked lanes
          float p0, p1;
          up2(e, p0, p1);
          e = pk2(x0 == -INFINITY ? 0.0f : p0, x1 == -INFINITY ? 0.0f : p1);
        }
      } else {
        e = pk2(ex2(x0), ex2(x1));  // ex2(-inf) = 0
      }
      float p0, p1;
      up2(e, p0, p1);
      if (i & 1) acc1 = fadd2(acc1, e);
      else acc0 = fadd2(acc0, e);
      pk[c * 16 + i] = ptx::pack_bf16x2(p0, p1);
    }
  }
  float a0, a1, b0, b1;
  up2(acc0, a0, a1);
  up2(acc1, b0, b1);
  // fast-path condition "every P <= 2^limit": with BAT_SUMCHECK the row-half sum bounds every
  // (non-negative) P, sparing the per-element max tracking (one FMNMX3 per pair); a sum above
  // the bound (rare once the reference max settled, and never missing an overflow) takes the
  // two-pass path
  const bool ok = BAT_SUMCHECK ? ((a0 + a1) + (b0 + b1) <= exp2f(limit)) : (fmaxf(xm0, xm1) <= limit);
  if (!agree(__all_sync(0xffffffffu, ok))) return false;
#pragma unroll
  for (int c = 0; c < NC; ++c)
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
        "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(tS + c * 16),
        "r"(pk[c * 16 + 0]), "r"(pk[c * 16 + 1]), "r"(pk[c * 16 + 2]), "r"(pk[c * 16 + 3]), "r"(pk[c * 16 + 4]),
        "r"(pk[c * 16 + 5]), "r"(pk[c * 16 + 6]), "r"(pk[c * 16 + 7]), "r"(pk[c * 16 + 8]), "r"(pk[c * 16 + 9]),
        "r"(pk[c * 16 + 10]), "r"(pk[c * 16 + 11]), "r"(pk[c * 16 + 12]), "r"(pk[c * 16 + 13]),
        "r"(pk[c * 16 + 14]), "r"(pk[c * 16 + 15]));
  lsum = (a0 + a1) + (b0 + b1);
  return true;
}

// Decide-before-exp (BAT_ATTN_DBE): the row half's 64 S values are loaded once (two tcgen05.ld,
// one wait) and kept in registers; their raw max goes to `decide`, which exchanges it with the
// other half, moves the reference when the row max grew by > 2^8 (rescaling O) and returns the
// reference every P of this tile is taken against (0 while the row has seen no visible key);
// P = exp2(s * scale - ref) is then written per 32-column chunk as soon as it is packed, so the
// first chunk's tcgen05.st overlaps the second chunk's math.  Returns the row-half sum.
template <bool MASKED, class Decide>
__device__ __forceinline__ float row_softmax_dbe(uint32_t tS, const uint32_t (&vis)[2], float scale,
                                                 Decide&& decide) {
  uint32_t r[2][32];
  ptx::tmem_ld32(tS, r[0]);
  ptx::tmem_ld32(tS + 32, r[1]);
  ptx::tmem_ld_wait();
  if (MASKED) {
#pragma unroll
    for (int c = 0; c < 2; ++c)
#pragma unroll
      for (int i = 0; i < 32; ++i) r[c][i] = ((vis[c] >> i) & 1u) ? r[c][i] : 0xff800000u;  // -inf
  }
  float m0 = -INFINITY, m1 = -INFINITY;
#pragma unroll
  for (int c = 0; c < 2; ++c)
#pragma unroll
    for (int i = 0; i < 32; i += 4) {
      m0 = fmax3(m0, __uint_as_float(r[c][i]), __uint_as_float(r[c][i + 1]));
      m1 = fmax3(m1, __uint_as_float(r[c][i + 2]), __uint_as_float(r[c][i + 3]));
    }
  const float ref = decide(fmaxf(m0, m1));
  const uint64_t sc2 = pk2(scale, scale), nm2 = pk2(-ref, -ref);
  uint64_t acc0 = pk2(0.0f, 0.0f), acc1 = acc0;
#pragma unroll
  for (int c = 0; c < 2; ++c) {
    uint32_t pk[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      const uint64_t xv = ffma2(pk2(__uint_as_float(r[c][2 * i]), __uint_as_float(r[c][2 * i + 1])), sc2, nm2);
      float x0, x1;
      up2(xv, x0, x1);
      uint64_t e;
      if (i < BAT_POLY_PAIRS) {
        e = exp2_poly2(xv);
        if (MASKED) {  // the polynomial clamps at -126: re-zero masked lanes
          float p0, p1;
          up2(e, p0, p1);
          e = pk2(x0 == -INFINITY ? 0.0f : p0, x1 == -INFINITY ? 0.0f : p1);
        }
      } else {
        e = pk2(ex2(x0), ex2(x1));  // ex2(-inf) = 0
      }
      float p0, p1;
      up2(e, p0, p1);
      if (i & 1) acc1 = fadd2(acc1, e);
      else acc0 = fadd2(acc0, e);
      pk[i] = ptx::pack_bf16x2(p0, p1);
    }
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
        "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(tS + c * 16),
        "r"(pk[0]), "r"(pk[1]), "r"(pk[2]), "r"(pk[3]), "r"(pk[4]), "r"(pk[5]), "r"(pk[6]), "r"(pk[7]),
        "r"(pk[8]), "r"(pk[9]), "r"(pk[10]), "r"(pk[11]), "r"(pk[12]), "r"(pk[13]), "r"(pk[14]),
        "r"(pk[15]));
  }
  float a0, a1, b0, b1;
  up2(acc0, a0, a1);
  up2(acc1, b0, b1);
  return (a0 + a1) + (b0 + b1);
}

template <int NC>
__device__ __forceinline__ void row_zero_p(uint32_t tS) {
#pragma unroll
  for (int c = 0; c < NC; ++c)
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
        "{%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1};" ::"r"(tS + c * 16), "r"(0u));
}

// ---- roles shared by the attention kernels -------------------------------------------------
// Loaders (warps 0, 2, 3 of the CTA): see the file comment.
template <int DP>
__device__ __forceinline__ void attn_loaders(const AttnParams& p, uint8_t* smem, AttnBars* bars, uint32_t warp,
                                             uint32_t lane) {
  using L = AttnSmem<DP>;
  const int32_t* img = p.img;
  const int32_t* work = img + p.off_work;
  {
    // Three independent streams so each runs as far ahead as its ring allows: warp 0 loads Q and
    // the K tiles (one bulk copy per page: the page block is the operand layout), warp 2 the first
    // V half of every tile (pages 0-3, plus the tile's key metadata), warp 3 the second half.
    // Page ids come from the work item's tile-page records (8 per listed tile, lanes 0-7) at
    // addresses known in advance, loaded three tiles ahead; the blocks of the tile two ahead are
    // prefetched into L2 by the stream that will load them.
    const int role = warp == 0 ? 0 : int(warp) - 1;  // 0: Q + K, 1: V half a, 2: V half b
    uint32_t qc = 0, kc = 0;
    const bool pl = lane < kKtilePages;
    constexpr int32_t kNone = kZeroPage + 1;  // "no tile": nothing to prefetch
    auto ids = [&](const WorkItem& a, const WorkItem& n, int t) -> int32_t {
      if (!pl) return kNone;
      if (t < a.kt_n) return img[a.tp_off + t * kKtilePages + lane];
      t -= a.kt_n;
      if (t < n.kt_n) return img[n.tp_off + t * kKtilePages + lane];
      return kNone;
    };
    const bool mine = pl && (role == 0 || (lane >> 2) == role - 1);  // lanes whose page this stream prefetches
    const int64_t kv_off = role == 0 ? 0 : int64_t(p.kv_heads) * p.head_bytes;  // K or V block of a page
    const WorkItem none{0, 0, -1, -1, 0, 0, 0, 0};
    for (int w = blockIdx.x; w < p.n_work; w += gridDim.x) {
      const WorkItem wi = load_work(work, w);
      if (wi.kt_n == 0) continue;  // padding of the planner's LPT rounds
      const WorkItem nx = (w + int(gridDim.x) < p.n_work) ? load_work(work, w + gridDim.x) : none;
      const int32_t* q_info = img + p.off_qinfo + int64_t(wi.b) * 8;
      const int qtile0 = q_info[2];
      int32_t pa = ids(wi, nx, 0), pb = ids(wi, nx, 1), pc = ids(wi, nx, 2);
      if (role == 0 && lane == 0) {
        BAT_LWAIT(&bars->q_empty, (qc & 1) ^ 1);
        const int nq = wi.q1 >= 0 ? 2 : 1;
        ptx::mbar_expect_tx(&bars->q_full, nq * L::TILE_BYTES);
        const char* qbase = reinterpret_cast<const char*>(p.qp);
        ptx::bulk_g2s(smem + L::Q_OFF, qbase + (int64_t(qtile0 + wi.q0) * p.kv_heads + wi.kvh) * L::TILE_BYTES,
                      L::TILE_BYTES, &bars->q_full);
        if (wi.q1 >= 0)
          ptx::bulk_g2s(smem + L::Q_OFF + L::TILE_BYTES,
                        qbase + (int64_t(qtile0 + wi.q1) * p.kv_heads + wi.kvh) * L::TILE_BYTES, L::TILE_BYTES,
                        &bars->q_full);
      }
      for (int x = 0; x < wi.kt_n; ++x, ++kc) {
        const int32_t pd = ids(wi, nx, x + 3);
        if (BAT_ATTN_L2PF && mine && pc != kNone && pc != kZeroPage) {  // L2 prefetch of tile x + 2 (maybe the next item's)
          const int kvh = (x + 2 < wi.kt_n) ? wi.kvh : nx.kvh;
          ptx::bulk_prefetch_l2(resolve_page(p, pc) + kv_off + int64_t(kvh) * p.head_bytes, L::PAGE_BYTES);
        }
        const bool dbg_first = (qc == 0) && role <= 1;
        if (role == 0) {
          const char* src[kKtilePages];
#pragma unroll
          for (int i = 0; i < kKtilePages; ++i) src[i] = resolve_page(p, __shfl_sync(0xffffffffu, pa, i));
          if (lane == 0) {
            const uint32_t ks = ring_slot(kc);
            uint8_t* sk = smem + L::K_OFF + ks * L::TILE_BYTES;
            DBG(0, x);
            BAT_LWAIT(&bars->k_empty[ks], ring_phase(kc) ^ 1);
            DBG(1, x);
            if (BAT_ATTN_NOLOAD) {  // timing experiment only: K never loaded (results are garbage)
              ptx::mbar_arrive(&bars->k_full[ks]);
            } else {
            ptx::mbar_expect_tx(&bars->k_full[ks], kKtilePages * L::PAGE_BYTES);
#pragma unroll
            for (int i = 0; i < kKtilePages; ++i)
              ptx::bulk_g2s(sk + i * L::PAGE_BYTES, src[i] + int64_t(wi.kvh) * p.head_bytes, L::PAGE_BYTES,
                            &bars->k_full[ks]);
            }
            DBG(2, x);
          }
        } else {
          const int hf = role - 1;
          const char* src[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) src[i] = resolve_page(p, __shfl_sync(0xffffffffu, pa, 4 * hf + i));
          if (lane == 0) {
            const uint32_t vi = 2 * kc + hf, vs = ring_slot(vi);
            uint8_t* sv = smem + L::V_OFF + vs * L::HALF_BYTES;
            if (hf == 0) DBG(3, x);
            BAT_LWAIT(&bars->v_empty[vs], ring_phase(vi) ^ 1);
            if (hf == 0) DBG(4, x);
            if (BAT_ATTN_NOLOAD) {
              ptx::mbar_arrive(&bars->v_full[vs]);
            } else {
            ptx::mbar_expect_tx(&bars->v_full[vs], 4 * L::PAGE_BYTES);
#pragma unroll
            for (int i = 0; i < 4; ++i)
              ptx::bulk_g2s(sv + i * L::PAGE_BYTES, src[i] + kv_off + int64_t(wi.kvh) * p.head_bytes, L::PAGE_BYTES,
                            &bars->v_full[vs]);
            }
          }
        }
        __syncwarp();
        pa = pb;
        pb = pc;
        pc = pd;
      }
      ++qc;
    }
  }
}

// MMA issuer (warp 1).  P_HALF_COLS: TMEM column offset of the P of key half 1 within an S
// buffer (P of half h at [64h, 64h+32)).
template <int DP, int P_HALF_COLS>
__device__ __forceinline__ void attn_mma(const AttnParams& p, uint8_t* smem, AttnBars* bars, uint32_t tmem,
                                         uint32_t lane) {
  using L = AttnSmem<DP>;
  constexpr uint32_t IDESC_S = ptx::idesc_bf16(128, 128, 0, 0);
  constexpr uint32_t IDESC_PV = ptx::idesc_bf16(128, DP, 0, 1);
  const int32_t* work = p.img + p.off_work;
  const bool dbg_first = false;
  (void)dbg_first;
    // the whole warp runs the issuer (converged: uniform-register descriptor math); every
    // tcgen05.mma / commit is issued by one elected lane
    {
      uint32_t qc = 0, kc = 0, pc0 = 0, pc1 = 0, oc0 = 0, oc1 = 0;
      const uint32_t sq0 = ptx::smem_u32(smem + L::Q_OFF);
      const uint32_t sq1 = sq0 + L::TILE_BYTES;
      const uint32_t tS0 = tmem, tS1 = tmem + 128, tO0 = tmem + 256, tO1 = tmem + 384;
      auto sk_of = [&](uint32_t g) { return ptx::smem_u32(smem + L::K_OFF + ring_slot(g) * L::TILE_BYTES); };
      auto sv_of = [&](uint32_t vi) { return ptx::smem_u32(smem + L::V_OFF + ring_slot(vi) * L::HALF_BYTES); };
      auto wait_k = [&](uint32_t g) {
        ptx::mbar_wait(&bars->k_full[ring_slot(g)], ring_phase(g));
        ptx::tc_fence_after();
      };
      auto issue_s = [&](uint32_t sq, uint32_t tS, uint32_t sk) {
#pragma unroll
        for (int kk = 0; kk < DP / 16; ++kk) {
          const uint32_t qoff = (kk >> 2) * 16384 + (kk & 3) * 32;  // Q: chunk-major, 8-row groups 1 KB apart
          const uint32_t koff = (kk >> 2) * 1024 + (kk & 3) * 32;   // K: page blocks, groups GROUP_BYTES apart
          ptx::mma_ss_elect(tS, ptx::desc_sw128(sq + qoff, 16, 1024), ptx::desc_sw128(sk + koff, 16, L::GROUP_BYTES),
                      IDESC_S, kk ? 1u : 0u);
        }
      };
      // O += P V for one V half (keys [64 hf, 64 hf + 64) = pages 4 hf .. 4 hf + 3): the P of key half
      // hf (bf16 pairs) sits at S columns [64 hf, 64 hf + 32), so keys [16 i, 16 i + 16) of the half
      // are at column 64 hf + 8 i; V page i of the half at sv + i * PAGE_BYTES
      auto issue_pv = [&](uint32_t tS, uint32_t tO, uint32_t sv, int hf, bool acc) {
#pragma unroll
        for (int i = 0; i < 4; ++i)
          ptx::mma_ts_elect(tO, tS + hf * P_HALF_COLS + i * 8, ptx::desc_sw128(sv + i * L::PAGE_BYTES, 1024, L::GROUP_BYTES),
                      IDESC_PV, (acc || hf || i) ? 1u : 0u);
      };
      // Items are software-pipelined: the next item's S0_0 is issued right after the current
      // item's last P0.V (S0 holds P0 until then) and its S1_0 right after the last P1.V, so the
      // softmax teams find their next S ready when they finish an epilogue.
      auto next_item = [&](int w) {
        for (w += gridDim.x; w < p.n_work; w += gridDim.x)
          if (work[int64_t(w) * 8 + 5] > 0) break;  // skip the planner's LPT padding
        return w;
      };
      auto first_s0 = [&](const WorkItem& wi, int w, uint32_t g0) {  // Q of wi + its K tile 0 -> S0_0
        ptx::mbar_wait(&bars->q_full, qc & 1);
        if (p.dbg_items) p.dbg_items[int64_t(w) * 6 + 0] = clock64();
        wait_k(g0);
        issue_s(sq0, tS0, sk_of(g0));
        ptx::mma_commit_elect(&bars->s_full[0]);
      };
      auto first_s1 = [&](const WorkItem& wi, int w, uint32_t g0) {  // -> S1_0, release K tile 0 / Q
        if (wi.q1 >= 0) {
          issue_s(sq1, tS1, sk_of(g0));
          ptx::mma_commit_elect(&bars->s_full[1]);
        }
        ptx::mma_commit_elect(&bars->k_empty[ring_slot(g0)]);
        if (wi.kt_n == 1) ptx::mma_commit_elect(&bars->q_empty);
        ++qc;
        if (p.dbg_items) p.dbg_items[int64_t(w) * 6 + 1] = clock64();
      };
      int w = blockIdx.x;
      if (w < p.n_work && work[int64_t(w) * 8 + 5] == 0) w = next_item(w);
      if (w < p.n_work) {
        const WorkItem wi = load_work(work, w);
        first_s0(wi, w, kc);
        first_s1(wi, w, kc);
      }
      while (w < p.n_work) {
        const WorkItem wi = load_work(work, w);
        const bool has1 = wi.q1 >= 0;
        const int n = wi.kt_n;
        const int wn = next_item(w);
        const WorkItem wni = wn < p.n_work ? load_work(work, wn) : WorkItem{0, 0, -1, -1, 0, 0, 0, 0};
        const bool dbg_first = (qc == 1);
        for (int x = 0; x < n; ++x) {
          const uint32_t g = kc + x;
          const uint32_t va = 2 * g, vb = 2 * g + 1;
          const uint32_t sva = sv_of(va), svb = sv_of(vb);
          DBG(5, x);
          const bool more = x + 1 < n;
          const uint32_t gn = g + 1;  // K tile of S_{x+1}, or tile 0 of the next item
          // ---- q-tile 0: PV0_x, then S0_{x+1} (or the next item's S0_0)
          ptx::mbar_wait(&bars->p_full[0], pc0 & 1);
          DBG(6, x);
          ++pc0;
          if (x == 0) ptx::mbar_wait(&bars->o_empty[0], (oc0 & 1) ^ 1);
          ptx::mbar_wait(&bars->v_full[ring_slot(va)], ring_phase(va));
          DBG(7, x);
          ptx::tc_fence_after();
          issue_pv(tS0, tO0, sva, 0, x > 0);
          ptx::mbar_wait(&bars->v_full[ring_slot(vb)], ring_phase(vb));
          ptx::tc_fence_after();
          issue_pv(tS0, tO0, svb, 1, true);
          if (more) {
            wait_k(gn);
            DBG(8, x);
            issue_s(sq0, tS0, sk_of(gn));
            ptx::mma_commit_elect(&bars->s_full[0]);
          } else {
            ptx::mma_commit_elect(&bars->o_full[0]);
            ++oc0;
            if (wn < p.n_work) first_s0(wni, wn, gn);
          }
          // ---- q-tile 1: PV1_x, then S1_{x+1} (or the next item's S1_0)
          if (has1) {
            ptx::mbar_wait(&bars->p_full[1], pc1 & 1);
            DBG(9, x);
            ++pc1;
            if (x == 0) ptx::mbar_wait(&bars->o_empty[1], (oc1 & 1) ^ 1);
            ptx::tc_fence_after();
            issue_pv(tS1, tO1, sva, 0, x > 0);
          }
          ptx::mma_commit_elect(&bars->v_empty[ring_slot(va)]);
          if (has1) issue_pv(tS1, tO1, svb, 1, true);
          ptx::mma_commit_elect(&bars->v_empty[ring_slot(vb)]);
          if (more) {
            if (has1) {
              issue_s(sq1, tS1, sk_of(gn));
              ptx::mma_commit_elect(&bars->s_full[1]);
            }
            ptx::mma_commit_elect(&bars->k_empty[ring_slot(gn)]);
            if (x + 1 == n - 1) ptx::mma_commit_elect(&bars->q_empty);
          } else {
            if (has1) {
              ptx::mma_commit_elect(&bars->o_full[1]);
              ++oc1;
            }
            if (p.dbg_items) {
              p.dbg_items[int64_t(w) * 6 + 2] = clock64();
              p.dbg_items[int64_t(w) * 6 + 4] = n;
              p.dbg_items[int64_t(w) * 6 + 5] = blockIdx.x;
            }
            if (wn < p.n_work) first_s1(wni, wn, gn);
          }
          DBG(10, x);
        }
        kc += n;
        w = wn;
      }
    }
}

template <int DP>
__global__ void __launch_bounds__(NUM_THREADS, 1) attn_tc_kernel(const __grid_constant__ AttnParams p) {
  using L = AttnSmem<DP>;
  extern __shared__ uint8_t smem_raw[];
  // 1 KB-align by offsetting the __shared__ array itself (keeps the shared address space, so
  // the compiler emits LDS/STS rather than generic loads and stores)
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  AttnBars* bars = reinterpret_cast<AttnBars*>(smem + L::BAR_OFF);
  const uint32_t warp = ptx::warp_id(), lane = ptx::lane_id();

  if (warp == 0 && lane == 0) {
    ptx::mbar_init(&bars->q_full, 1);
    ptx::mbar_init(&bars->q_empty, 1);
    for (int i = 0; i < 3; ++i) {
      ptx::mbar_init(&bars->k_full[i], 1);
      ptx::mbar_init(&bars->k_empty[i], 1);
      ptx::mbar_init(&bars->v_full[i], 1);
      ptx::mbar_init(&bars->v_empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&bars->s_full[i], 1);
      ptx::mbar_init(&bars->p_full[i], 8);
      ptx::mbar_init(&bars->o_full[i], 1);
      ptx::mbar_init(&bars->o_empty[i], 8);
      ptx::mbar_init(&bars->seq[i], 8);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc(&bars->tmem_base, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = bars->tmem_base;

  const int32_t* img = p.img;
  const int32_t* work = img + p.off_work;

  if (warp == 0 || warp == 2 || warp == 3) {  // ------------------------------------ loaders
    attn_loaders<DP>(p, smem, bars, warp, lane);
  } else if (warp == 1) {  // ---------------------------------------------- MMA issuer
    attn_mma<DP, 64>(p, smem, bars, tmem, lane);
  } else if (warp >= 4) {  // ------------------------------------------ softmax warpgroups
    const int wgi = (warp - 4) >> 2;
    const int wg = wgi & 1, h = wgi >> 1;  // q-tile, key half
    const uint32_t sub = warp & 3;
    const int row = sub * 32 + lane;
    const uint32_t lane_base = (sub * 32) << 16;
    const uint32_t tS = tmem + wg * 128 + h * 64 + lane_base;       // my S half; P at its first 32 columns
    constexpr int OCH = DP / 64;                                     // 32-column O chunks per half
    const uint32_t tO = tmem + 256 + wg * 128 + h * (DP / 2) + lane_base;
    const uint32_t pair_bar = 1 + wg * 4 + sub;                      // named barrier of the warp pair
    XchSmem* xch = reinterpret_cast<XchSmem*>(smem + L::XCH_OFF);
    uint32_t kc = 0, sc = 0, oc = 0;
    // Turn-taking (FA4-style softmax sequencing): team 0 runs the softmax of its tile x, then
    // team 1 of its tile x, then team 0 of tile x + 1, ... — each softmax runs alone on the
    // MUFU/FMA pipes while the tensor pipe serves the other q-tile's P.V and next S, instead of
    // both overlapping at half speed with both q-tiles' MMAs bunched together.  A team without a
    // q-tile in an item passes the token through for each of its tiles.
    uint32_t turn = 0;
    auto seq_wait = [&]() {
      if (!BAT_ATTN_SEQ) return;
      if (wg == 0) {
        if (turn > 0) ptx::mbar_wait(&bars->seq[0], (turn - 1) & 1);
      } else {
        ptx::mbar_wait(&bars->seq[1], turn & 1);
      }
    };
    auto seq_pass = [&]() {
      if (!BAT_ATTN_SEQ) return;
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&bars->seq[wg ^ 1]);
      ++turn;
    };
    for (int w = blockIdx.x; w < p.n_work; w += gridDim.x) {
      const WorkItem wi = load_work(work, w);
      const int qi = wg == 0 ? wi.q0 : wi.q1;
      if (qi < 0 || wi.kt_n == 0) {
        for (int x = 0; x < wi.kt_n; ++x) {
          seq_wait();
          seq_pass();
        }
        kc += wi.kt_n;
        continue;
      }
      const int32_t* q_info = img + p.off_qinfo + int64_t(wi.b) * 8;
      const int tok_off = q_info[0], S = q_info[1];
      const int tok_local = qi * p.qt + row / p.group;
      const bool valid_row = row < p.qt * p.group && tok_local < S;
      const int mrow = valid_row ? row / p.group : p.qt;  // row of this thread in the masks
      const int32_t* ktl = img + wi.kt_off;
      float m_ref = -INFINITY, l_sum = 0.0f;
      // tile state and partial-tile visibility bits, loaded ONE TILE AHEAD: the state / mask-id
      // loads (independent, plan image in L2) are issued at the top of the previous tile and
      // the mask bits once they land, so none of the ~1k clk L2 round trips sits between S
      // landing and the softmax (tools/chain_rate.cu: the bare chain runs at 2.75k clk per
      // k-tile pair, the kernel at ~3.9k before this)
      auto mask_of = [&](int mid) {
        return __ldg(reinterpret_cast<const uint2*>(img + p.off_masks + (int64_t(mid) * (p.qt + 1) + mrow) * 4) + h);
      };
      int n_state = (ktl[0] >> (24 + 2 * wg)) & 3;
      int n_mid = img[wi.km_off + wg];
      uint2 n_mv = make_uint2(0xffffffffu, 0xffffffffu);
      if (n_state == 2) n_mv = mask_of(n_mid);
      for (int x = 0; x < wi.kt_n; ++x) {
        const uint32_t g = kc + x;
        const int s = g & 1;
        const int state = (BAT_ATTN_NOMASK && n_state == 2) ? 1 : n_state;  // NOMASK: timing experiment only
        const uint2 mv = n_mv;
        if (x + 1 < wi.kt_n) {
          n_state = (ktl[x + 1] >> (24 + 2 * wg)) & 3;
          n_mid = img[wi.km_off + 2 * (x + 1) + wg];
        } else {
          n_state = 0;
        }
        const bool dbg_first = (kc == 0) && row == 0 && h == 0;
        BAT_SWAIT(&bars->s_full[wg], sc & 1);
        DBG(11 + 3 * wg, x);
        ++sc;
        if (BAT_ATTN_SEQ == 1) seq_wait();
        ptx::tc_fence_after();
        const uint32_t vis[NCH] = {mv.x, mv.y};
        float lsum = 0.0f;
#if BAT_ATTN_DBE
        if (state == 0) {
          row_zero_p<NCH>(tS);
          if (BAT_ATTN_SEQ == 2) {
            seq_wait();
            seq_pass();
          }
        } else {
          // the row's reference for this tile: both halves' raw maxima through smem, then the
          // same lazy-rescale decision in both (so they agree without a vote)
          bool need_o = false;
          float alpha = 1.0f;
          auto decide = [&](float mt) {
            if (wg == 0) DBG(18, x);
            xch->rmax[s][wg][h][row] = mt;
            ptx::bar_sync(pair_bar, 64);
            if (wg == 0) DBG(19, x);
            mt = fmaxf(mt, xch->rmax[s][wg][h ^ 1][row]);
            const float m_new = fmaxf(m_ref, mt * p.scale_log2);
            if (m_new > m_ref + kRescaleThreshold) {
              alpha = ex2(m_ref - m_new);  // 0 when m_ref = -inf
              l_sum *= alpha;
              need_o = (m_ref != -INFINITY) && (x > 0);
              m_ref = m_new;
            }
            if (BAT_ATTN_SEQ == 2) seq_wait();  // the exp phases of the two teams take turns
            return (m_ref == -INFINITY) ? 0.0f : m_ref;
          };
          lsum = (state == 1) ? row_softmax_dbe<false>(tS, vis, p.scale_log2, decide)
                              : row_softmax_dbe<true>(tS, vis, p.scale_log2, decide);
          if (BAT_ATTN_SEQ == 2) seq_pass();
          // O rows of this warp rescaled (my half of the columns) before P is handed over: the
          // previous P.V of this q-tile is complete (issued before this S, in-order tensor pipe)
          // and this tile's P.V waits for the hand-off
          if (__any_sync(0xffffffffu, need_o)) {
            const float a = need_o ? alpha : 1.0f;
#pragma unroll 1
            for (int c = 0; c < OCH; ++c) {
              uint32_t r[32];
              ptx::tmem_ld32(tO + c * 32, r);
              ptx::tmem_ld_wait();
#pragma unroll
              for (int i = 0; i < 32; ++i) r[i] = __float_as_uint(__uint_as_float(r[i]) * a);
              ptx::tmem_st32(tO + c * 32, r);
            }
          }
        }
        if (wg == 0) DBG(12, x);
#else
        // fast path: one pass against the settled reference max; both halves must agree
        bool done = false;
        if (state == 0) {
          row_zero_p<NCH>(tS);
          done = true;
        } else if (__all_sync(0xffffffffu, m_ref != -INFINITY)) {  // same in both halves of the pair
          const uint64_t sc2 = pk2(p.scale_log2, p.scale_log2), nm2 = pk2(-m_ref, -m_ref);
          auto agree = [&](bool ok) {
            if (wg == 0) DBG(18, x);
            if (lane == 0) xch->ok[s][wg][h][sub] = ok;
            ptx::bar_sync(pair_bar, 64);
            if (wg == 0) DBG(19, x);
            return ok && xch->ok[s][wg][h ^ 1][sub] != 0;
          };
          done = (state == 1) ? row_exp_opt<false>(tS, vis, sc2, nm2, kRescaleThreshold, lsum, agree)
                              : row_exp_opt<true>(tS, vis, sc2, nm2, kRescaleThreshold, lsum, agree);
        }
        if (wg == 0) DBG(12, x);
        if (!done) {
          // slow path, pass 1: row max of the raw scores over both halves
          float mt = (state == 1) ? row_max<false>(tS, vis) : row_max<true>(tS, vis);
          xch->rmax[s][wg][h][row] = mt;
          ptx::bar_sync(pair_bar, 64);
          mt = fmaxf(mt, xch->rmax[s][wg][h ^ 1][row]);
          const float m_old = m_ref;
          const float m_new = fmaxf(m_ref, mt * p.scale_log2);
          const bool grow = m_new > m_ref + kRescaleThreshold;
          float alpha = 1.0f;
          if (grow) {
            alpha = ex2(m_ref - m_new);  // 0 when m_ref = -inf
            l_sum *= alpha;
            m_ref = m_new;
          }
          // O rows of this warp are rescaled (my half of the columns) when a lane's reference
          // max moved.  The previous P.V of this q-tile is complete: it was issued before this
          // S (in-order tensor pipe).
          const bool need_o = grow && (m_old != -INFINITY) && (x > 0);
          if (__any_sync(0xffffffffu, need_o)) {
            const float a = need_o ? alpha : 1.0f;
#pragma unroll 1
            for (int c = 0; c < OCH; ++c) {
              uint32_t r[32];
              ptx::tmem_ld32(tO + c * 32, r);
              ptx::tmem_ld_wait();
#pragma unroll
              for (int i = 0; i < 32; ++i) r[i] = __float_as_uint(__uint_as_float(r[i]) * a);
              ptx::tmem_st32(tO + c * 32, r);
            }
            ptx::tmem_st_wait();
          }
          // pass 2: P = exp2(s * scale - m_ref) -> bf16 into my half's first 32 columns
          const float mref = (m_ref == -INFINITY) ? 0.0f : m_ref;
          const uint64_t sc2 = pk2(p.scale_log2, p.scale_log2), nm2 = pk2(-mref, -mref);
          lsum = (state == 1) ? row_exp<false>(tS, vis, sc2, nm2) : row_exp<true>(tS, vis, sc2, nm2);
        }
#endif
        l_sum += lsum;
        ptx::tmem_st_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&bars->p_full[wg]);
        if (BAT_ATTN_SEQ == 1) seq_pass();
        DBG(13 + 2 * wg, x);
        n_mv = make_uint2(0xffffffffu, 0xffffffffu);
        if (n_state == 2) n_mv = mask_of(n_mid);
      }
      kc += wi.kt_n;
      // ---- epilogue: O / l -> bf16, my half of the head's columns
      xch->lsum[wg][h][row] = l_sum;
      BAT_SWAIT(&bars->o_full[wg], oc & 1);
      ++oc;
      ptx::tc_fence_after();
      ptx::bar_sync(pair_bar, 64);
      const float l_tot = l_sum + xch->lsum[wg][h ^ 1][row];
      const float inv = (l_tot > 0.0f) ? 1.0f / l_tot : 0.0f;
      const int head = wi.kvh * p.group + row % p.group;
      __nv_bfloat16* dst = p.out + int64_t(tok_off + tok_local) * p.ldo + int64_t(head) * p.head_dim;
      // split-KV chunk: O / l in fp32 and the row's (m, l) go to the item's partial slot instead
      const int slot = p.part_o ? img[p.off_wslot + w] : -1;
      if (slot >= 0) {
        const int64_t pr = (int64_t(slot) * 2 + wg) * 128 + row;
        if (h == 0) reinterpret_cast<float2*>(p.part_ml)[pr] = make_float2(m_ref, l_tot);
        float* po = p.part_o + pr * DP + h * (DP / 2);
#pragma unroll 1
        for (int c = 0; c < OCH; ++c) {
          uint32_t r[32];
          ptx::tmem_ld32(tO + c * 32, r);
          ptx::tmem_ld_wait();
          if (valid_row) {
            float4* d4 = reinterpret_cast<float4*>(po + c * 32);
#pragma unroll
            for (int i = 0; i < 8; ++i)
              d4[i] = make_float4(__uint_as_float(r[4 * i]) * inv, __uint_as_float(r[4 * i + 1]) * inv,
                                  __uint_as_float(r[4 * i + 2]) * inv, __uint_as_float(r[4 * i + 3]) * inv);
          }
        }
      }
#pragma unroll 1
      for (int c = 0; c < (slot >= 0 ? 0 : OCH); ++c) {
        const int col0 = h * (DP / 2) + c * 32;
        uint32_t r[32];
        ptx::tmem_ld32(tO + c * 32, r);
        ptx::tmem_ld_wait();
        if (valid_row && col0 < p.head_dim) {
          uint32_t pk[16];
#pragma unroll
          for (int i = 0; i < 16; ++i)
            pk[i] = ptx::pack_bf16x2(__uint_as_float(r[2 * i]) * inv, __uint_as_float(r[2 * i + 1]) * inv);
          const int n16 = min(4, (p.head_dim - col0) / 8);  // 16-byte stores of real columns
          uint4* d4 = reinterpret_cast<uint4*>(dst + col0);
          for (int i = 0; i < n16; ++i) d4[i] = make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
        }
      }
      ptx::tc_fence_before();
      __syncwarp();
      // relaxed: orders this warp's TMEM reads of O (waited above), not its global O stores
      if (lane == 0) ptx::mbar_arrive_relaxed(&bars->o_empty[wg]);
      if (p.dbg_items && wg == 0 && h == 0 && sub == 0 && lane == 0) p.dbg_items[int64_t(w) * 6 + 3] = clock64();
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) ptx::tmem_dealloc(tmem, 512);
}


// ==========================================================================================
// Round-2 kernel (default): ONE softmax thread per S row, all 128 columns in registers.
// Warps: 0 Q+K loader, 1 MMA issuer, 2 / 3 V-half loaders (attn_loaders / attn_mma as above),
// 4-7 the softmax team of q-tile 0, 8-11 of q-tile 1 (warp w owns TMEM lanes 32 (w % 4)..).
// Per tile a thread loads its row's 128 S values (4 tcgen05.ld), applies the partial-tile mask,
// takes the row max FIRST (thread-local: no cross-thread agreement, no retry path), moves the
// reference max only when the row max exceeds it by > 2^8 (then O is rescaled in TMEM — O is
// stable: this S was issued after the previous P.V), and writes P = exp2(s * scale - m) as bf16
// pairs into the S buffer's first 64 columns (key k at column k / 2) as each 32-key chunk is
// ready; V2_POLY of the 64 pairs of a full tile take exp2 on the FMA pipe.  The two teams
// alternate naturally: team 0's softmax runs while the tensor pipe does q-tile 1's P.V and next
// S, and vice versa (tools/fa4_chain.cu measures the bare chain).
// Split-KV combine: one warp per (split group, q-tile of the pair, row); O = sum_p w_p O_p /
// sum_p w_p with w_p = l_p 2^(m_p - max m) over the group's parts (O_p already divided by l_p).
template <int DP>
__global__ void attn_combine_kernel(const AttnParams p, int64_t off_sgrp) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int rid = blockIdx.x * (blockDim.x >> 5) + warp;  // (group, q-tile, row)
  const int g = rid / 256, qsel = (rid >> 7) & 1, row = rid & 127;
  const int32_t* gr = p.img + off_sgrp + int64_t(g) * 6;
  const int b = gr[0], kvh = gr[1], qi = qsel ? gr[3] : gr[2], slot0 = gr[4], parts = gr[5];
  if (qi < 0) return;
  const int32_t* q_info = p.img + p.off_qinfo + int64_t(b) * 8;
  const int tok_off = q_info[0], S = q_info[1];
  const int tok_local = qi * p.qt + row / p.group;
  if (row >= p.qt * p.group || tok_local >= S) return;
  const float2* ml = reinterpret_cast<const float2*>(p.part_ml);
  float m = -INFINITY;
  for (int k = 0; k < parts; ++k) {
    const float2 v = ml[(int64_t(slot0 + k) * 2 + qsel) * 128 + row];
    if (v.y > 0.0f) m = fmaxf(m, v.x);
  }
  constexpr int PER = DP / 32;
  float acc[PER];
#pragma unroll
  for (int i = 0; i < PER; ++i) acc[i] = 0.0f;
  float wsum = 0.0f;
  for (int k = 0; k < parts; ++k) {
    const int64_t pr = (int64_t(slot0 + k) * 2 + qsel) * 128 + row;
    const float2 v = ml[pr];
    if (!(v.y > 0.0f)) continue;
    const float wgt = v.y * ex2(v.x - m);
    wsum += wgt;
    const float* po = p.part_o + pr * DP;
#pragma unroll
    for (int i = 0; i < PER; ++i) acc[i] = fmaf(wgt, po[lane + 32 * i], acc[i]);
  }
  const float inv = wsum > 0.0f ? 1.0f / wsum : 0.0f;
  const int head = kvh * p.group + row % p.group;
  __nv_bfloat16* dst = p.out + int64_t(tok_off + tok_local) * p.ldo + int64_t(head) * p.head_dim;
#pragma unroll
  for (int i = 0; i < PER; ++i)
    if (lane + 32 * i < p.head_dim) dst[lane + 32 * i] = __float2bfloat16_rn(acc[i] * inv);
}

}  // namespace

int attn_grid_slots(int, int num_sms) { return num_sms; }

int attn_qtiles_per_item() { return 2; }

size_t attn_smem_bytes(int dpad) {
  return 1024 + (dpad == 128 ? AttnSmem<128>::TOTAL : AttnSmem<64>::TOTAL);
}

void launch_attention_combine(int dpad, const AttnParams& p, int64_t off_sgrp, int n_sgrp, cudaStream_t stream) {
  if (n_sgrp <= 0) return;
  const int blocks = n_sgrp * 256 / 8;  // 8 warps (rows) per block
  if (dpad == 128) attn_combine_kernel<128><<<blocks, 256, 0, stream>>>(p, off_sgrp);
  else attn_combine_kernel<64><<<blocks, 256, 0, stream>>>(p, off_sgrp);
  count_launch();
}

void launch_attention(int dpad, const AttnParams& p, int num_sms, cudaStream_t stream) {
  const int grid = p.n_work < num_sms ? p.n_work : num_sms;
  if (grid <= 0) return;
  const size_t smem = attn_smem_bytes(dpad);
  if (dpad == 128) {
    set_smem_attr(attn_tc_kernel<128>, smem);
    attn_tc_kernel<128><<<grid, NUM_THREADS, smem, stream>>>(p);
  } else {
    set_smem_attr(attn_tc_kernel<64>, smem);
    attn_tc_kernel<64><<<grid, NUM_THREADS, smem, stream>>>(p);
  }
  count_launch();
}

}  // namespace bat
