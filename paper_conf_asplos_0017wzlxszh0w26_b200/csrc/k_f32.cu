// FP32 SIMT correctness mode (bat_dtype BAT_FP32; north_star: "1e-5 for an fp32
// mode").  The same path as the bf16 product kernels — embedding (a2), RMSNorm + QKV (a3), RoPE
// at the bipartite positions + suffix K/V staging into pages (a4), bipartite attention over the
// paged prefix + suffix keys under the plan's key metadata (a5, P:251/P:255/P:257), O / MLP
// GEMMs with residual (a6/a7), final norm (a9) — in plain fp32 CUDA-core arithmetic, so that
// the planner's positions, segments, page tables and masks are checked against the fp64 oracle
// at a tolerance (1e-5) where any single wrong key or position is visible.  Not a fast path:
// tiled SIMT GEMM, one warp per (row, head) attention with an online softmax.
//
// Page layout (fp32 pools): page = [layers][2 (K,V)][kv_heads][16 slots][head_dim] fp32.
#include <cuda_runtime.h>

#include "common.h"
#include "kernels.h"

namespace bat {
namespace {

__device__ __forceinline__ float warp_sum32(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__global__ void embed_f32_kernel(const float* __restrict__ E, const int32_t* __restrict__ tok,
                                 float* __restrict__ h, int H) {
  const int m = blockIdx.x;
  const float* src = E + int64_t(tok[m]) * H;
  for (int c = threadIdx.x; c < H; c += blockDim.x) h[int64_t(m) * H + c] = src[c];
}

// y[r] = x[idx ? idx[r] : r] / sqrt(mean(x^2) + eps) * g, one warp per row
__global__ void rmsnorm_f32_kernel(const float* __restrict__ x, const float* __restrict__ g,
                                   float* __restrict__ y, const int32_t* __restrict__ idx, int M, int H,
                                   float eps) {
  const int r = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (r >= M) return;
  const float* xr = x + int64_t(idx ? idx[r] : r) * H;
  float ss = 0.0f;
  for (int c = lane; c < H; c += 32) ss += xr[c] * xr[c];
  ss = warp_sum32(ss);
  const float inv = rsqrtf(ss / float(H) + eps);
  for (int c = lane; c < H; c += 32) y[int64_t(r) * H + c] = xr[c] * inv * g[c];
}

// C = A W^T: A [M][K], W [N][K] (rows = output features).  64 x 64 tiles, 16-deep K slabs,
// 256 threads x (4 x 4) outputs.  EPI: 0 out = C + bias, 1 out += C, 2 out = silu(A Wg^T) * (A Wu^T)
// with Wg = W rows [0, N), Wu = W rows [up_row0, up_row0 + N).
constexpr int GT = 64, GK = 16;
template <int EPI>
__global__ void __launch_bounds__(256) gemm_f32_kernel(const float* __restrict__ A, const float* __restrict__ W,
                                                       const float* __restrict__ bias, float* __restrict__ out,
                                                       int M, int N, int K, int up_row0) {
  __shared__ float As[GK][GT + 4];
  __shared__ float Ws[GK][GT + 4];
  __shared__ float Us[EPI == 2 ? GK : 1][GT + 4];
  const int m0 = blockIdx.y * GT, n0 = blockIdx.x * GT;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  float acc[4][4] = {}, accu[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += GK) {
    for (int e = threadIdx.x; e < GT * GK; e += 256) {
      const int r = e / GK, kk = e % GK;
      const int gm = m0 + r, gn = n0 + r, gk = k0 + kk;
      As[kk][r] = (gm < M && gk < K) ? A[int64_t(gm) * K + gk] : 0.0f;
      Ws[kk][r] = (gn < N && gk < K) ? W[int64_t(gn) * K + gk] : 0.0f;
      if (EPI == 2) Us[kk][r] = (gn < N && gk < K) ? W[int64_t(up_row0 + gn) * K + gk] : 0.0f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < GK; ++kk) {
      float a[4], w[4], u[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        a[i] = As[kk][ty * 4 + i];
        w[i] = Ws[kk][tx * 4 + i];
        if (EPI == 2) u[i] = Us[kk][tx * 4 + i];
      }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          acc[i][j] = fmaf(a[i], w[j], acc[i][j]);
          if (EPI == 2) accu[i][j] = fmaf(a[i], u[j], accu[i][j]);
        }
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int gm = m0 + ty * 4 + i, gn = n0 + tx * 4 + j;
      if (gm >= M || gn >= N) continue;
      float* o = out + int64_t(gm) * N + gn;
      if (EPI == 0) *o = acc[i][j] + (bias ? bias[gn] : 0.0f);
      else if (EPI == 1) *o += acc[i][j];
      else {
        const float gt = acc[i][j];
        *o = gt / (1.0f + expf(-gt)) * accu[i][j];
      }
    }
}

// rotate-half RoPE of one head vector (fp32): element c < d/2 pairs with c + d/2
__device__ __forceinline__ float rope_at(const float* x, int c, int d, const float2* cs, bool on) {
  if (!on) return x[c];
  const int h = d / 2;
  const float2 t = cs[c % h];
  return c < h ? x[c] * t.x - x[c + h] * t.y : x[c] * t.x + x[c - h] * t.y;
}

// a4 (fp32): blocks [0, M): q of row m -> qf [M][Hq][d]; blocks [M, M + n_spages): the suffix
// page's K (rotated) and V rows -> the page target (pool page >= 0, scratch page -(s+1)).
__global__ void stage_f32_kernel(const StageF32Params p) {
  const int d = p.head_dim;
  const int nqkv = (p.q_heads + 2 * p.kv_heads) * d;
  const int32_t* img = p.img;
  if (int(blockIdx.x) < p.M) {
    const int m = blockIdx.x;
    const int pos = min(img[p.off_pos + m], p.max_pos - 1);
    const float2* cs = p.rope + int64_t(pos) * (d / 2);
    for (int e = threadIdx.x; e < p.q_heads * d; e += blockDim.x) {
      const int h = e / d, c = e % d;
      p.qf[int64_t(m) * p.q_heads * d + e] = rope_at(p.qkv + int64_t(m) * nqkv + h * d, c, d, cs, p.rope_enabled);
    }
    return;
  }
  const int sp = blockIdx.x - p.M;
  const int4 si = *reinterpret_cast<const int4*>(img + p.off_spages + int64_t(sp) * 4);
  const int b = si.x, t0 = si.y, ntok = si.z, target = si.w;
  const int tok_off = img[p.off_qinfo + int64_t(b) * 8];
  float* page = reinterpret_cast<float*>(target >= 0 ? p.pool + int64_t(target) * p.pool_page_bytes + p.pool_layer_off
                                                     : p.scratch + int64_t(-target - 1) * p.scratch_page_bytes);
  for (int e = threadIdx.x; e < 2 * ntok * p.kv_heads * d; e += blockDim.x) {
    const int kv = e / (ntok * p.kv_heads * d);
    const int rem = e % (ntok * p.kv_heads * d);
    const int j = rem / (p.kv_heads * d), h = (rem / d) % p.kv_heads, c = rem % d;
    const int m = tok_off + t0 + j;
    const int pos = min(img[p.off_pos + m], p.max_pos - 1);
    const float* src = p.qkv + int64_t(m) * nqkv + (p.q_heads + kv * p.kv_heads + h) * d;
    page[((int64_t(kv) * p.kv_heads + h) * kPageTokens + j) * d + c] =
        rope_at(src, c, d, p.rope + int64_t(pos) * (d / 2), kv == 0 && p.rope_enabled);
  }
}

// a5 (fp32): one warp per (suffix row t of request b, q head j); keys = the request's page list
// (prefix pages, then its suffix pages) in virtual-key order; key slot s visible to row t iff
// kord[s] <= t + 1 and (kseg[s] == seg[t] or either < 0) (plan.cpp header).
__global__ void attn_f32_kernel(const AttnF32Params p) {
  const int b = blockIdx.y;
  const int32_t* img = p.img;
  const int32_t* qi = img + p.off_qinfo + int64_t(b) * 8;
  const int tok_off = qi[0], S = qi[1], page_off = qi[4], n_ktiles = qi[5];
  const int wid = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  const int t = wid / p.q_heads, head = wid % p.q_heads;
  if (t >= S) return;
  const int d = p.head_dim, kvh = head / p.group;
  const int m = tok_off + t;
  const int32_t rseg = img[p.off_rseg + m], rord = t + 1;
  constexpr int DMAX = 4;  // head_dim <= 128
  float q[DMAX], acc[DMAX];
#pragma unroll
  for (int i = 0; i < DMAX; ++i) {
    const int c = lane + 32 * i;
    q[i] = c < d ? p.qf[(int64_t(m) * p.q_heads + head) * d + c] : 0.0f;
    acc[i] = 0.0f;
  }
  float mx = -INFINITY, l = 0.0f;
  const int n_slots = n_ktiles * kKtilePages * kPageTokens;
  const int2* km = reinterpret_cast<const int2*>(img + p.off_kmeta) + int64_t(page_off) * kPageTokens;
  for (int s = 0; s < n_slots; ++s) {
    const int2 k = km[s];
    if (!(k.y <= rord && (k.x == rseg || (k.x | rseg) < 0))) continue;
    const int32_t pg = img[p.off_pages + page_off + s / kPageTokens];
    const char* base = pg >= 0 ? p.pool + int64_t(pg) * p.pool_page_bytes + p.pool_layer_off
                               : p.scratch + int64_t(-pg - 1) * p.scratch_page_bytes;
    const float* kr = reinterpret_cast<const float*>(base) + (int64_t(kvh) * kPageTokens + s % kPageTokens) * d;
    const float* vr = reinterpret_cast<const float*>(base) + (int64_t(p.kv_heads + kvh) * kPageTokens + s % kPageTokens) * d;
    float dot = 0.0f;
#pragma unroll
    for (int i = 0; i < DMAX; ++i) {
      const int c = lane + 32 * i;
      if (c < d) dot = fmaf(q[i], kr[c], dot);
    }
    const float sc = warp_sum32(dot) * p.scale;
    const float mn = fmaxf(mx, sc);
    const float alpha = expf(mx - mn);  // 0 on the first visible key (mx = -inf)
    const float pe = expf(sc - mn);
    l = l * alpha + pe;
#pragma unroll
    for (int i = 0; i < DMAX; ++i) {
      const int c = lane + 32 * i;
      acc[i] = acc[i] * alpha + (c < d ? pe * vr[c] : 0.0f);
    }
    mx = mn;
  }
  const float inv = l > 0.0f ? 1.0f / l : 0.0f;
#pragma unroll
  for (int i = 0; i < DMAX; ++i) {
    const int c = lane + 32 * i;
    if (c < d) p.out[int64_t(m) * p.q_heads * d + head * d + c] = acc[i] * inv;
  }
}

// K/V [layers][n][kv_heads][d] fp32 (plain) <-> fp32 pages; one block per (token, layer)
template <bool TO_PAGES>
__global__ void kv_pages_f32_kernel(PageIO io, float* k, float* v, const int32_t* __restrict__ pages,
                                    int n_tokens, int slot0, int n_total) {
  const int t = blockIdx.x, l = blockIdx.y;
  const int d = io.head_dim;
  const int slot = slot0 + t;
  float* page = reinterpret_cast<float*>(io.arena + int64_t(pages[slot / kPageTokens]) * io.page_bytes +
                                         int64_t(l) * io.layer_bytes);
  const int j = slot % kPageTokens;
  for (int e = threadIdx.x; e < 2 * io.kv_heads * d; e += blockDim.x) {
    const int kv = e / (io.kv_heads * d), h = (e / d) % io.kv_heads, c = e % d;
    float* plain = (kv == 0 ? k : v) + ((int64_t(l) * n_total + t) * io.kv_heads + h) * d + c;
    float* pg = page + ((int64_t(kv) * io.kv_heads + h) * kPageTokens + j) * d + c;
    if (TO_PAGES) *pg = *plain;
    else *plain = *pg;
  }
}

}  // namespace

void launch_embed_f32(const float* E, const int32_t* tok, float* h, int M, int H, cudaStream_t s) {
  if (M <= 0) return;
  embed_f32_kernel<<<M, 128, 0, s>>>(E, tok, h, H);
  count_launch();
}
void launch_rmsnorm_f32(const float* x, const float* g, float* y, const int32_t* idx, int M, int H, float eps,
                        cudaStream_t s) {
  if (M <= 0) return;
  rmsnorm_f32_kernel<<<(M + 7) / 8, 256, 0, s>>>(x, g, y, idx, M, H, eps);
  count_launch();
}
void launch_gemm_f32(int epi, const float* A, const float* W, const float* bias, float* out, int M, int N, int K,
                     int up_row0, cudaStream_t s) {
  if (M <= 0) return;
  const dim3 grid((N + GT - 1) / GT, (M + GT - 1) / GT);
  if (epi == 0) gemm_f32_kernel<0><<<grid, 256, 0, s>>>(A, W, bias, out, M, N, K, up_row0);
  else if (epi == 1) gemm_f32_kernel<1><<<grid, 256, 0, s>>>(A, W, bias, out, M, N, K, up_row0);
  else gemm_f32_kernel<2><<<grid, 256, 0, s>>>(A, W, bias, out, M, N, K, up_row0);
  count_launch();
}
void launch_stage_f32(const StageF32Params& p, cudaStream_t s) {
  const int grid = p.M + p.n_spages;
  if (grid <= 0) return;
  stage_f32_kernel<<<grid, 256, 0, s>>>(p);
  count_launch();
}
void launch_attention_f32(const AttnF32Params& p, int B, int max_S, cudaStream_t s) {
  if (B <= 0 || max_S <= 0) return;
  const int warps = 8;
  const dim3 grid((max_S * p.q_heads + warps - 1) / warps, B);
  attn_f32_kernel<<<grid, warps * 32, 0, s>>>(p);
  count_launch();
}
void launch_kv_scatter_f32(const PageIO& io, const float* k, const float* v, const int32_t* pages_dev, int n_tokens,
                           int slot0, int n_total, cudaStream_t s) {
  if (n_tokens <= 0) return;
  kv_pages_f32_kernel<true><<<dim3(n_tokens, io.layers), 128, 0, s>>>(io, const_cast<float*>(k), const_cast<float*>(v),
                                                                    pages_dev, n_tokens, slot0, n_total);
  count_launch();
}
void launch_kv_gather_f32(const PageIO& io, float* k, float* v, const int32_t* pages_dev, int n_tokens,
                          cudaStream_t s) {
  if (n_tokens <= 0) return;
  kv_pages_f32_kernel<false><<<dim3(n_tokens, io.layers), 128, 0, s>>>(io, k, v, pages_dev, n_tokens, 0, n_tokens);
  count_launch();
}

}  // namespace bat
