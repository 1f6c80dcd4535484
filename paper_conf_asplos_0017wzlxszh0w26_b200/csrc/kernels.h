// Launchers of libbat's device kernels (all sm_100a).  Every launcher bumps the launch
// counter reported by bat_kernel_launch_count().
#pragma once

#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cstdint>

namespace bat {

void count_launch(int n = 1);
int64_t launch_count();

// Opt a kernel into `bytes` of dynamic shared memory on the CURRENT device (the attribute is
// per device context); cached per (kernel, device), thread-safe, fails with BAT_E_CUDA.
void set_smem_attr_raw(const void* func, int bytes);
template <class K>
inline void set_smem_attr(K* kern, size_t bytes) {
  set_smem_attr_raw(reinterpret_cast<const void*>(kern), static_cast<int>(bytes));
}

// a4 staging parameters (RoPE + q-tile / suffix-page layout), shared by stage_kernel and the
// QKV GEMM epilogue that fuses it (GemmParams::stage)
struct StageParams {
  const __nv_bfloat16* qkv;  // [M][(Hq+2Hkv)*d]
  const int32_t* img;
  int64_t off_pos, off_qinfo, off_qtiles, off_spages;
  int32_t n_qtiles, n_spages;
  const float2* rope;        // [max_pos][d/2] (cos, sin)
  int32_t rope_enabled, max_pos;
  int32_t q_heads, kv_heads, head_dim, dpad, group, qt;
  __nv_bfloat16* qp;         // q-tiles out
  char* pool;                // target pages: pool page p (>= 0) or scratch page s (-(s+1))
  int64_t pool_page_bytes, pool_layer_off;
  char* scratch;
  int64_t scratch_page_bytes, scratch_layer_off;
  int64_t head_bytes;
  int32_t n_req;             // requests of the plan (q_info rows)
  int64_t off_rowreq;        // [M] request of every suffix row (the fused QKV epilogue's lookup)
};

// ------------------------------------------------------------------------ tcgen05 GEMM
enum GemmEpi { EPI_BF16 = 0, EPI_BF16_BIAS = 1, EPI_RESID_F32 = 2, EPI_SWIGLU = 3, EPI_PART_F32 = 4 };
struct GemmParams {
  int M, N, K;        // N = output columns (SWIGLU: the ffn width F)
  void* out;          // bf16 [M][ldo] or fp32 residual [M][ldo]
  int ldo;
  const __nv_bfloat16* bias;  // EPI_BF16_BIAS
  int up_row0;        // EPI_SWIGLU: first "up" row of B (= F)
  int group_m = 0;    // M-tiles per rasterisation group (0: launch_gemm's default)
  int hints = 0;      // 1-CTA kernel L2 hints: bit 0 B loads evict_last, bit 1 bf16 C stores evict_first
  int ksplit = 1;     // EPI_PART_F32: K split in ksplit slices; slice s stores its fp32 partial at
  int mpad = 0;       // rows [s * mpad, s * mpad + M) of the partial buffer (tmC)
  // RMSNorm fused across the residual update (a3 / a7, P:169 layer structure): the producer
  // (EPI_RESID_F32 with norm_g set) writes h_new = h + acc by TMA store instead of reduce-add,
  // xg = bf16(h_new * g) for the next projection's A operand and, per N-tile j, the partial sum of
  // squares ss_out[j * M + row] of its columns; the consumer (EPI_BF16_BIAS / EPI_SWIGLU with ss_in
  // set) scales each accumulator row by rsqrt(sum_j ss_in[j * M + row] / norm_h + eps) before its
  // bias / SwiGLU — RMSNorm(h) W^T = rstd * ((h * g) W^T) with no separate norm pass.
  const __nv_bfloat16* norm_g = nullptr;
  __nv_bfloat16* xg_out = nullptr;
  float* ss_out = nullptr;
  const float* ss_in = nullptr;
  int ss_parts = 0;
  int norm_h = 0;
  float eps = 0.0f;
  // a4 fused into the QKV epilogue (EPI_BF16_BIAS, stage_on): each row's q / k / v heads are
  // rotated (RoPE at the plan position) in fp32 and written straight into the q-tiles and suffix
  // pages; the qkv activation is never stored
  int stage_on = 0;
  StageParams stage{};
};
// Split-K for grids that would leave SMs idle (small M: batch-1 requests, the last layer's
// discriminant rows): slices per tile (1 = no split) for a GEMM of this shape and the row pitch of
// its partial slabs.  Deterministic: the partials are summed in slice order by launch_gemm_reduce.
int gemm_ksplit(int epi, int M, int N, int K, int num_sms, int* mpad);
// out = sum_s part[s] (+ bias), mode 0: fp32 residual h += ..., mode 1: bf16 out = .. + bias
void launch_gemm_reduce(const float* part, int ksplit, int mpad, int M, int N, void* out, int ldo,
                        const __nv_bfloat16* bias, int mode, cudaStream_t stream);
size_t gemm_smem_bytes();
// column slices per accumulator in the epilogue (fused-norm partial sums per N-tile)
int gemm_epi_col_splits();
// the QKV epilogue can run a4 (one warp per TMEM lane quarter holds whole rows of a head)
bool gemm_qkv_stage_fusable(int head_dim);
// tmC: output tensor map — bf16 [M][ldo] with box {64, 32} (EPI_BF16*, EPI_SWIGLU) or fp32
// [M][ldo] with box {32, 32} (EPI_RESID_F32, TMA reduce-add), 128-byte swizzle
void launch_gemm(int epi, const CUtensorMap& tmA, const CUtensorMap& tmB, const CUtensorMap& tmC,
                 const GemmParams& p, int num_sms, cudaStream_t stream);

// ------------------------------------------------------------------ bipartite attention
struct AttnParams {
  const int32_t* img;       // plan image (device)
  int64_t off_qinfo, off_pages, off_kmeta, off_rseg, off_work;
  int32_t n_work;
  const char* pool;         // arena; page p, layer l at pool + p*pool_page_bytes + pool_layer_off
  int64_t pool_page_bytes, pool_layer_off;
  const char* scratch;      // suffix pages; page s at scratch + s*scratch_page_bytes + scratch_layer_off
  int64_t scratch_page_bytes, scratch_layer_off;
  const char* zero_page;    // all-zero K/V block source for page-list padding
  int64_t head_bytes;       // bytes of one head's K (or V) in a page-layer block
  int32_t kv_heads, group, qt, head_dim, ldo;
  const __nv_bfloat16* qp;  // packed, swizzled q-tiles
  __nv_bfloat16* out;       // O [M][q_heads*head_dim]
  float scale_log2;         // log2(e) / sqrt(head_dim)
  long long* dbg;           // optional timeline (clock64) of CTA 0's first work item
  long long* dbg_items;     // optional per-work-item record [n_work][6] (see k_attn.cu)
  int64_t off_masks;        // visibility masks of the partial tiles (launch_masks)
  int64_t off_wslot;        // split-KV: per work item its partial slot (-1: direct output)
  float* part_o;            // split-KV partials [slot][2][128][Dp] (O / l, fp32); nullptr: no split
  float* part_ml;           // [slot][2][128] (m, l)
};
size_t attn_smem_bytes(int dpad);

// number of persistent work slots the planner balances the attention work list over
int attn_grid_slots(int dpad, int num_sms);
// q-tiles per attention work item of the kernel launch_attention runs (2: pairs, 1: singles)
int attn_qtiles_per_item();

// Visibility masks of the plan's partial (q-tile, k-tile) pairs (PlanImage::off_mdesc): one block
// per mask, bit (32 c + i) of row r's word c = key slot 32 c + i of the k-tile visible to token
// r of the q-tile, by kord <= rord && (kseg == rseg || (kseg | rseg) < 0); row qt (and rows past
// the request's suffix) = the padding rows' mask (every valid key).
void launch_masks(int32_t* img, int64_t off_mdesc, int64_t off_qinfo, int64_t off_kmeta, int64_t off_rseg,
                  int64_t off_masks, int32_t n_masks, int32_t qt, cudaStream_t s);
void launch_attention(int dpad, const AttnParams& p, int num_sms, cudaStream_t stream);
// merge the split-KV partials of n_sgrp groups (PlanImage::off_sgrp) into p.out
void launch_attention_combine(int dpad, const AttnParams& p, int64_t off_sgrp, int n_sgrp, cudaStream_t stream);

// --------------------------------------------------------------------- small kernels
// fused-norm form: also xg = bf16(h0 * g) and ss[m] = sum h0^2 (the first layer's RMSNorm inputs)
void launch_embed_norm(const __nv_bfloat16* E, const int32_t* tok, float* h, const __nv_bfloat16* g,
                       __nv_bfloat16* xg, float* ss, int M, int H, cudaStream_t s);
void launch_embed(const __nv_bfloat16* E, const int32_t* tok, float* h, int M, int H,
                  cudaStream_t s);
// y = x * rsqrt(mean(x^2) + eps) * g  (rows given by idx when idx != nullptr)
void launch_rmsnorm_bf16(const float* x, const __nv_bfloat16* g, __nv_bfloat16* y, int M, int H,
                         float eps, cudaStream_t s);
void launch_rmsnorm_f32out(const float* x, const __nv_bfloat16* g, float* y, int M, int H,
                           float eps, cudaStream_t s);
void launch_rope_table(float2* tab, int max_pos, int d, double theta, cudaStream_t s);

void launch_stage(const StageParams& p, cudaStream_t s);

void launch_gather_rows_bf16(const __nv_bfloat16* src, const int32_t* idx, __nv_bfloat16* dst,
                             int n, int cols, cudaStream_t s);
void launch_gather_rows_f32(const float* src, const int32_t* idx, float* dst, int n, int cols,
                            cudaStream_t s);
void launch_score(const float* hidden, const __nv_bfloat16* w_out, const int32_t* labels,
                  const int32_t* n_items, int B, int n_max, int H, float* scores, int k,
                  int32_t* topk, float* logits, cudaStream_t s);

// KV pool page scatter / gather in the swizzled page layout (bf16)
struct PageIO {
  char* arena;
  int64_t page_bytes, layer_bytes, head_bytes;
  int32_t layers, kv_heads, head_dim;
};
void launch_kv_scatter(const PageIO& io, const __nv_bfloat16* k, const __nv_bfloat16* v,
                       const int32_t* pages_dev, int n_tokens, int slot0, int n_total,
                       cudaStream_t s);
void launch_kv_gather(const PageIO& io, __nv_bfloat16* k, __nv_bfloat16* v,
                      const int32_t* pages_dev, int n_tokens, cudaStream_t s);
// copy whole pages: dst_arena page dst[i] <- src_ptrs[i] (peer-mapped)
void launch_page_copy(const uint64_t* src_ptrs, const int32_t* dst_pages, char* dst_arena,
                      int64_t page_bytes, int n, cudaStream_t s);

// ------------------------------------------------- FP32 SIMT correctness mode (k_f32.cu)
struct StageF32Params {
  const float* qkv;  // [M][(Hq+2Hkv)*d]
  const int32_t* img;
  int64_t off_pos, off_qinfo, off_spages;
  int32_t M, n_spages;
  const float2* rope;
  int32_t rope_enabled, max_pos;
  int32_t q_heads, kv_heads, head_dim;
  float* qf;  // [M][Hq][d]
  char* pool;
  int64_t pool_page_bytes, pool_layer_off;
  char* scratch;
  int64_t scratch_page_bytes;
};
struct AttnF32Params {
  const int32_t* img;
  int64_t off_qinfo, off_pages, off_kmeta, off_rseg;
  const char* pool;
  int64_t pool_page_bytes, pool_layer_off;
  const char* scratch;
  int64_t scratch_page_bytes;
  int32_t q_heads, kv_heads, group, head_dim;
  const float* qf;
  float* out;  // [M][Hq*d]
  float scale;
};
void launch_embed_f32(const float* E, const int32_t* tok, float* h, int M, int H, cudaStream_t s);
void launch_rmsnorm_f32(const float* x, const float* g, float* y, const int32_t* idx, int M, int H, float eps,
                        cudaStream_t s);
// epi: 0 out = A W^T + bias, 1 out += A W^T, 2 out = silu(A Wg^T) * (A Wu^T) (Wu = rows from up_row0)
void launch_gemm_f32(int epi, const float* A, const float* W, const float* bias, float* out, int M, int N, int K,
                     int up_row0, cudaStream_t s);
void launch_stage_f32(const StageF32Params& p, cudaStream_t s);
void launch_attention_f32(const AttnF32Params& p, int B, int max_S, cudaStream_t s);
void launch_kv_scatter_f32(const PageIO& io, const float* k, const float* v, const int32_t* pages_dev, int n_tokens,
                           int slot0, int n_total, cudaStream_t s);
void launch_kv_gather_f32(const PageIO& io, float* k, float* v, const int32_t* pages_dev, int n_tokens,
                          cudaStream_t s);
// one discriminant hidden row per item: hidden [B][n_max][H] (exactly one of w_bf16 / w_f32)
void launch_score_multi(const float* hidden, const __nv_bfloat16* w_bf16, const float* w_f32, const int32_t* labels,
                        const int32_t* n_items, int B, int n_max, int H, float* scores, int k, int32_t* topk,
                        float* logits, cudaStream_t s);
void launch_score_f32w(const float* hidden, const float* w_out, const int32_t* labels, const int32_t* n_items, int B,
                       int n_max, int H, float* scores, int k, int32_t* topk, float* logits, cudaStream_t s);

}  // namespace bat
