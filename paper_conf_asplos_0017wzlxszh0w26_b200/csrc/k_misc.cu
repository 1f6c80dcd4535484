// Memory-bound kernels of the path: embedding gather (a2), RMSNorm (a3/a7/a9), RoPE at the
// bipartite positions + staging of the GQA-packed q-tiles and the suffix K/V pages (a4),
// row gathers for the last-layer trim (a8), the discriminant score (a9), and the KV-page
// scatter/gather/copy kernels behind bat_kv_append / bat_kv_read / bat_kv_fetch.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <atomic>
#include <map>
#include <mutex>
#include <string>

#include "common.h"
#include "kernels.h"
#include "ptx.cuh"

namespace bat {

static std::atomic<int64_t> g_launches{0};
void count_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }
int64_t launch_count() { return g_launches.load(std::memory_order_relaxed); }

void set_smem_attr_raw(const void* func, int bytes) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, int> done;  // (kernel, device) -> bytes set
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) fail(BAT_E_CUDA, "cudaGetDevice failed");
  std::lock_guard<std::mutex> lk(mu);
  auto key = std::make_pair(func, dev);
  auto it = done.find(key);
  if (it != done.end() && it->second >= bytes) return;
  const cudaError_t e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e != cudaSuccess)
    fail(BAT_E_CUDA, std::string("cudaFuncSetAttribute(MaxDynamicSharedMemorySize): ") + cudaGetErrorString(e));
  done[key] = bytes;
}

namespace {

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// h0[m] = E[x_m], bf16 table -> fp32 residual stream
__global__ void embed_kernel(const __nv_bfloat16* __restrict__ E, const int32_t* __restrict__ tok,
                             float* __restrict__ h, int M, int H) {
  const int m = blockIdx.x;
  const int64_t src = int64_t(tok[m]) * H;
  for (int c = threadIdx.x * 8; c < H; c += blockDim.x * 8) {
    uint4 raw = *reinterpret_cast<const uint4*>(E + src + c);
    const __nv_bfloat162* b2 = reinterpret_cast<const __nv_bfloat162*>(&raw);
    float4 o0, o1;
    float2 f;
    f = __bfloat1622float2(b2[0]); o0.x = f.x; o0.y = f.y;
    f = __bfloat1622float2(b2[1]); o0.z = f.x; o0.w = f.y;
    f = __bfloat1622float2(b2[2]); o1.x = f.x; o1.y = f.y;
    f = __bfloat1622float2(b2[3]); o1.z = f.x; o1.w = f.y;
    float4* d = reinterpret_cast<float4*>(h + int64_t(m) * H + c);
    d[0] = o0;
    d[1] = o1;
  }
}

// fused-norm embedding: one warp per row; h0 = E[x_m] (fp32), xg = bf16(h0 * g), ss[m] = sum h0^2
// (the first layer's RMSNorm is finished in the QKV GEMM epilogue, GemmParams::ss_in)
__global__ void embed_norm_kernel(const __nv_bfloat16* __restrict__ E, const int32_t* __restrict__ tok,
                                  float* __restrict__ h, const __nv_bfloat16* __restrict__ g,
                                  __nv_bfloat16* __restrict__ xg, float* __restrict__ ss_out, int M, int H) {
  const int m = blockIdx.x * 8 + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (m >= M) return;
  const int64_t src = int64_t(tok[m]) * H;
  float ss = 0.0f;
  for (int c = lane * 8; c < H; c += 256) {
    const uint4 raw = *reinterpret_cast<const uint4*>(E + src + c);
    const uint4 graw = *reinterpret_cast<const uint4*>(g + c);
    const __nv_bfloat162* b2 = reinterpret_cast<const __nv_bfloat162*>(&raw);
    const __nv_bfloat162* g2 = reinterpret_cast<const __nv_bfloat162*>(&graw);
    float v[8];
    uint32_t pk[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 f = __bfloat1622float2(b2[i]), gg = __bfloat1622float2(g2[i]);
      v[2 * i] = f.x;
      v[2 * i + 1] = f.y;
      ss += f.x * f.x + f.y * f.y;
      pk[i] = ptx::pack_bf16x2(f.x * gg.x, f.y * gg.y);
    }
    float4* d = reinterpret_cast<float4*>(h + int64_t(m) * H + c);
    d[0] = make_float4(v[0], v[1], v[2], v[3]);
    d[1] = make_float4(v[4], v[5], v[6], v[7]);
    *reinterpret_cast<uint4*>(xg + int64_t(m) * H + c) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
  }
  ss = warp_sum(ss);
  if (lane == 0) ss_out[m] = ss;
}

// one warp per row: y = x / sqrt(mean(x^2) + eps) * g
template <bool F32OUT>
__global__ void rmsnorm_kernel(const float* __restrict__ x, const __nv_bfloat16* __restrict__ g,
                               void* __restrict__ y, int M, int H, float eps) {
  const int row = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= M) return;
  const float* xr = x + int64_t(row) * H;
  float ss = 0.0f;
  for (int c = lane * 4; c < H; c += 128) {
    float4 v = *reinterpret_cast<const float4*>(xr + c);
    ss += v.x * v.x + v.y * v.y + v.z * v.z + v.w * v.w;
  }
  ss = warp_sum(ss);
  const float r = rsqrtf(ss / float(H) + eps);
  for (int c = lane * 4; c < H; c += 128) {
    float4 v = *reinterpret_cast<const float4*>(xr + c);
    const __nv_bfloat162* g2 = reinterpret_cast<const __nv_bfloat162*>(g + c);
    float2 ga = __bfloat1622float2(g2[0]), gb = __bfloat1622float2(g2[1]);
    float o0 = v.x * r * ga.x, o1 = v.y * r * ga.y, o2 = v.z * r * gb.x, o3 = v.w * r * gb.y;
    if (F32OUT) {
      *reinterpret_cast<float4*>(static_cast<float*>(y) + int64_t(row) * H + c) = make_float4(o0, o1, o2, o3);
    } else {
      uint2 pk = make_uint2(ptx::pack_bf16x2(o0, o1), ptx::pack_bf16x2(o2, o3));
      *reinterpret_cast<uint2*>(static_cast<__nv_bfloat16*>(y) + int64_t(row) * H + c) = pk;
    }
  }
}

// Register-resident variant for H = 128 NV: the row is read from HBM once (NV float4 per lane
// kept in registers across the reduction), normalised and written as bf16.
template <int NV>
__global__ void __launch_bounds__(256) rmsnorm_reg_kernel(const float* __restrict__ x, const __nv_bfloat16* __restrict__ g,
                                                          __nv_bfloat16* __restrict__ y, int M, float eps) {
  constexpr int H = NV * 128;
  const int row = blockIdx.x * 8 + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= M) return;
  const float4* xr = reinterpret_cast<const float4*>(x + int64_t(row) * H);
  float4 v[NV];
#pragma unroll
  for (int i = 0; i < NV; ++i) v[i] = __ldcs(xr + lane + 32 * i);  // streamed: read once
  float ss = 0.0f;
#pragma unroll
  for (int i = 0; i < NV; ++i) ss += v[i].x * v[i].x + v[i].y * v[i].y + v[i].z * v[i].z + v[i].w * v[i].w;
  ss = warp_sum(ss);
  const float r = rsqrtf(ss / float(H) + eps);
  uint2* yr = reinterpret_cast<uint2*>(y + int64_t(row) * H);
  const uint2* g2 = reinterpret_cast<const uint2*>(g);
#pragma unroll
  for (int i = 0; i < NV; ++i) {
    const uint2 gg = g2[lane + 32 * i];
    const float2 ga = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&gg.x));
    const float2 gb = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&gg.y));
    yr[lane + 32 * i] = make_uint2(ptx::pack_bf16x2(v[i].x * r * ga.x, v[i].y * r * ga.y),
                                   ptx::pack_bf16x2(v[i].z * r * gb.x, v[i].w * r * gb.y));
  }
}

// cos/sin table in double precision, rounded once to fp32: tab[pos][i] = (cos, sin)(pos * theta^(-2i/d))
__global__ void rope_table_kernel(float2* tab, int max_pos, int d, double theta) {
  const int half = d / 2;
  const int64_t n = int64_t(max_pos) * half;
  for (int64_t e = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; e < n; e += int64_t(gridDim.x) * blockDim.x) {
    const int pos = int(e / half), i = int(e % half);
    const double inv = pow(theta, -2.0 * double(i) / double(d));
    double sn, cs;
    sincos(double(pos) * inv, &sn, &cs);
    tab[e] = make_float2(float(cs), float(sn));
  }
}

// rotate-half RoPE of the column pair (c, c + d/2) for 8 consecutive c = c0..c0+7 of one head
// vector x (bf16): o1 = x1 cos - x2 sin, o2 = x2 cos + x1 sin; cs = the position's (cos, sin)
// row.  Both 16-byte halves and the 64 bytes of cos/sin are read once.
__device__ __forceinline__ void rope_pair8(const __nv_bfloat16* __restrict__ x, int c0, int d,
                                           const float2* __restrict__ cs, bool enabled, uint4& o1, uint4& o2) {
  const uint4 r1 = *reinterpret_cast<const uint4*>(x + c0);
  const uint4 r2 = *reinterpret_cast<const uint4*>(x + c0 + d / 2);
  if (!enabled) {
    o1 = r1;
    o2 = r2;
    return;
  }
  const __nv_bfloat162* a = reinterpret_cast<const __nv_bfloat162*>(&r1);
  const __nv_bfloat162* b = reinterpret_cast<const __nv_bfloat162*>(&r2);
  const float4* t4 = reinterpret_cast<const float4*>(cs + c0);
  uint32_t w1[4], w2[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const float4 t = t4[i];  // (cos, sin) of columns c0+2i, c0+2i+1
    const float2 fa = __bfloat1622float2(a[i]), fb = __bfloat1622float2(b[i]);
    w1[i] = ptx::pack_bf16x2(fa.x * t.x - fb.x * t.y, fa.y * t.z - fb.y * t.w);
    w2[i] = ptx::pack_bf16x2(fb.x * t.x + fa.x * t.y, fb.y * t.z + fa.y * t.w);
  }
  o1 = make_uint4(w1[0], w1[1], w1[2], w1[3]);
  o2 = make_uint4(w2[0], w2[1], w2[2], w2[3]);
}

// a4: RoPE(q, k) at the plan's positions; write the q-tiles (GQA-packed rows = token x
// head-in-group, 128-byte swizzled [Dp/64][128][64]) and the suffix K/V pages.  Only real rows
// and columns are written: the buffers are zeroed at allocation and padding is never written.
__global__ void stage_kernel(const StageParams p) {
  const int d = p.head_dim;
  const int nqkv = (p.q_heads + 2 * p.kv_heads) * d;
  const int32_t* img = p.img;
  const int pairs = d / 16;  // 8-column chunk pairs (c, c + d/2) per head
  int blk = blockIdx.x;
  const int n_q_blocks = p.n_qtiles * p.kv_heads;
  if (blk < n_q_blocks) {
    const int gq = blk / p.kv_heads, kvh = blk % p.kv_heads;
    const int4 qt = *reinterpret_cast<const int4*>(img + p.off_qtiles + int64_t(gq) * 4);
    const int b = qt.x, t0 = qt.y, ntok = qt.z;
    const int tok_off = img[p.off_qinfo + int64_t(b) * 8];
    char* tile = reinterpret_cast<char*>(p.qp) + (int64_t(gq) * p.kv_heads + kvh) * (p.dpad / 64) * 16384;
    const int rows = ntok * p.group;
    for (int e = threadIdx.x; e < rows * pairs; e += blockDim.x) {
      const int r = e / pairs, pc = e % pairs;
      const int c0 = pc * 8, c1 = c0 + d / 2;
      const int m = tok_off + t0 + r / p.group;
      const int head = kvh * p.group + r % p.group;
      const int pos = min(img[p.off_pos + m], p.max_pos - 1);
      uint4 o1, o2;
      rope_pair8(p.qkv + int64_t(m) * nqkv + head * d, c0, d, p.rope + int64_t(pos) * (d / 2), p.rope_enabled, o1, o2);
      *reinterpret_cast<uint4*>(tile + (c0 / 64) * 16384 + ptx::swz128(r, (c0 % 64) / 8)) = o1;
      *reinterpret_cast<uint4*>(tile + (c1 / 64) * 16384 + ptx::swz128(r, (c1 % 64) / 8)) = o2;
    }
    return;
  }
  blk -= n_q_blocks;
  const int sp = blk / p.kv_heads, kvh = blk % p.kv_heads;
  const int4 si = *reinterpret_cast<const int4*>(img + p.off_spages + int64_t(sp) * 4);
  const int b = si.x, t0 = si.y, ntok = si.z, target = si.w;
  const int tok_off = img[p.off_qinfo + int64_t(b) * 8];
  char* page = target >= 0 ? p.pool + int64_t(target) * p.pool_page_bytes + p.pool_layer_off
                           : p.scratch + int64_t(-target - 1) * p.scratch_page_bytes + p.scratch_layer_off;
  for (int e = threadIdx.x; e < 2 * ntok * pairs; e += blockDim.x) {
    const int kv = e / (ntok * pairs);
    const int rem = e % (ntok * pairs);
    const int j = rem / pairs, pc = rem % pairs;
    const int c0 = pc * 8, c1 = c0 + d / 2;
    const int m = tok_off + t0 + j;
    const __nv_bfloat16* src = p.qkv + int64_t(m) * nqkv + (p.q_heads + kv * p.kv_heads + kvh) * d;
    const int pos = min(img[p.off_pos + m], p.max_pos - 1);
    uint4 o1, o2;
    rope_pair8(src, c0, d, p.rope + int64_t(pos) * (d / 2), kv == 0 && p.rope_enabled, o1, o2);
    char* blockp = page + (int64_t(kv) * p.kv_heads + kvh) * p.head_bytes;
    const uint32_t ch = uint32_t(p.dpad / 64);
    *reinterpret_cast<uint4*>(blockp + ptx::page_blk_off(j, c0, ch)) = o1;
    *reinterpret_cast<uint4*>(blockp + ptx::page_blk_off(j, c1, ch)) = o2;
  }
}

template <class T>
__global__ void gather_rows_kernel(const T* __restrict__ src, const int32_t* __restrict__ idx,
                                   T* __restrict__ dst, int cols) {
  const int r = blockIdx.x;
  const int64_t s = int64_t(idx[r]) * cols, o = int64_t(r) * cols;
  for (int c = threadIdx.x; c < cols; c += blockDim.x) dst[o + c] = src[s + c];
}

// a9: z_i = W_out[v_i] . hf, s = softmax over the N candidates, top-k
template <class TW, bool MULTI>
__global__ void score_kernel(const float* __restrict__ hidden, const TW* __restrict__ w,
                             const int32_t* __restrict__ labels, const int32_t* __restrict__ n_items,
                             int n_max, int H, float* __restrict__ scores, int k,
                             int32_t* __restrict__ topk, float* __restrict__ logits) {
  extern __shared__ float sh[];
  float* hf = sh;            // [H]
  float* z = sh + H;         // [n_max]
  __shared__ float red[32];
  __shared__ int redi[32];
  const int b = blockIdx.x;
  // n_items is device data: clamp to the row width so a bad count can never overrun z[n_max]
  const int n = max(0, min(n_items[b], n_max));
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (!MULTI)
    for (int c = threadIdx.x; c < H; c += blockDim.x) hf[c] = hidden[int64_t(b) * H + c];
  __syncthreads();
  for (int i = wid; i < n; i += nw) {
    const TW* row = w + int64_t(labels[int64_t(b) * n_max + i]) * H;
    float acc = 0.0f;
    if constexpr (MULTI) {  // one discriminant hidden state per item
      const float* hi = hidden + (int64_t(b) * n_max + i) * H;
      for (int c = lane; c < H; c += 32) acc = fmaf(float(row[c]), hi[c], acc);
    } else if constexpr (sizeof(TW) == 4) {  // fp32 correctness mode
      for (int c = lane; c < H; c += 32) acc = fmaf(row[c], hf[c], acc);
    } else {
      for (int c = lane * 8; c < H; c += 256) {
        uint4 raw = *reinterpret_cast<const uint4*>(row + c);
        const __nv_bfloat162* b2 = reinterpret_cast<const __nv_bfloat162*>(&raw);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          float2 f = __bfloat1622float2(b2[q]);
          acc += f.x * hf[c + 2 * q] + f.y * hf[c + 2 * q + 1];
        }
      }
    }
    acc = warp_sum(acc);
    if (lane == 0) z[i] = acc;
  }
  __syncthreads();
  if (logits)  // z_i as computed here, for parity checks of the GEMV itself
    for (int i = threadIdx.x; i < n_max; i += blockDim.x) logits[int64_t(b) * n_max + i] = i < n ? z[i] : 0.0f;
  // max
  float mx = -INFINITY;
  for (int i = threadIdx.x; i < n; i += blockDim.x) mx = fmaxf(mx, z[i]);
  mx = warp_max(mx);
  if (lane == 0) red[wid] = mx;
  __syncthreads();
  if (wid == 0) {
    float v = lane < nw ? red[lane] : -INFINITY;
    v = warp_max(v);
    if (lane == 0) red[0] = v;
  }
  __syncthreads();
  mx = red[0];
  __syncthreads();
  float sm = 0.0f;
  for (int i = threadIdx.x; i < n; i += blockDim.x) sm += __expf(z[i] - mx);
  sm = warp_sum(sm);
  if (lane == 0) red[wid] = sm;
  __syncthreads();
  if (wid == 0) {
    float v = lane < nw ? red[lane] : 0.0f;
    v = warp_sum(v);
    if (lane == 0) red[0] = v;
  }
  __syncthreads();
  const float inv = n > 0 ? 1.0f / red[0] : 0.0f;
  __syncthreads();
  for (int i = threadIdx.x; i < n_max; i += blockDim.x) {
    const float s = i < n ? __expf(z[i] - mx) * inv : 0.0f;
    scores[int64_t(b) * n_max + i] = s;
    if (i < n) z[i] = s;
  }
  __syncthreads();
  // top-k by repeated arg-max (ties -> lower index); taken entries set to -1
  for (int t = 0; t < k; ++t) {
    if (t >= n) {  // fewer candidates than k: the remaining ranks are empty (-1)
      if (threadIdx.x == 0) topk[int64_t(b) * k + t] = -1;
      continue;
    }
    float best = -2.0f;
    int bi = 0x7fffffff;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
      const float v = z[i];
      if (v > best || (v == best && i < bi)) { best = v; bi = i; }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const float ov = __shfl_xor_sync(0xffffffffu, best, o);
      const int oi = __shfl_xor_sync(0xffffffffu, bi, o);
      if (ov > best || (ov == best && oi < bi)) { best = ov; bi = oi; }
    }
    if (lane == 0) { red[wid] = best; redi[wid] = bi; }
    __syncthreads();
    if (threadIdx.x == 0) {
      float bb = red[0];
      int bbi = redi[0];
      for (int q = 1; q < nw; ++q)
        if (red[q] > bb || (red[q] == bb && redi[q] < bbi)) { bb = red[q]; bbi = redi[q]; }
      topk[int64_t(b) * k + t] = bbi;
      if (bbi < n) z[bbi] = -1.0f;
    }
    __syncthreads();
  }
}

// K/V [layers][n][kv_heads][d] (plain) <-> swizzled pages.  One block per (token, layer).
template <bool TO_PAGES>
__global__ void kv_pages_kernel(PageIO io, __nv_bfloat16* k, __nv_bfloat16* v,
                                const int32_t* __restrict__ pages, int n_tokens, int slot0,
                                int n_total) {
  const int t = blockIdx.x, l = blockIdx.y;
  const int d = io.head_dim;
  const int cpr = d / 8;  // 16-byte chunks of a head row
  const int slot = slot0 + t;
  char* page = io.arena + int64_t(pages[slot / kPageTokens]) * io.page_bytes + int64_t(l) * io.layer_bytes;
  const int j = slot % kPageTokens;
  for (int e = threadIdx.x; e < 2 * io.kv_heads * cpr; e += blockDim.x) {
    const int kv = e / (io.kv_heads * cpr);
    const int rem = e % (io.kv_heads * cpr);
    const int h = rem / cpr, cc = rem % cpr;
    const int c0 = cc * 8;
    __nv_bfloat16* plain = (kv == 0 ? k : v) + ((int64_t(l) * n_total + t) * io.kv_heads + h) * d + c0;
    char* pg = page + (int64_t(kv) * io.kv_heads + h) * io.head_bytes +
               ptx::page_blk_off(j, c0, uint32_t(io.head_bytes / 2048));
    if (TO_PAGES) *reinterpret_cast<uint4*>(pg) = *reinterpret_cast<const uint4*>(plain);
    else *reinterpret_cast<uint4*>(plain) = *reinterpret_cast<const uint4*>(pg);
  }
}

__global__ void __launch_bounds__(128) mask_kernel(int32_t* img, int64_t off_mdesc, int64_t off_qinfo,
                                                  int64_t off_kmeta, int64_t off_rseg, int64_t off_masks, int32_t qt) {
  const int m = blockIdx.x;
  const int4 d = reinterpret_cast<const int4*>(img + off_mdesc)[m];  // {b, q-tile, k-tile, 0}
  const int32_t* qinfo = img + off_qinfo + int64_t(d.x) * 8;
  const int tok_off = qinfo[0], S = qinfo[1], page_off = qinfo[4];
  __shared__ int2 keys[kKtile];  // (kseg, kord) of the k-tile's slots
  const int2* km = reinterpret_cast<const int2*>(img + off_kmeta) + (int64_t(page_off) + int64_t(d.z) * kKtilePages) * kPageTokens;
  for (int k = threadIdx.x; k < kKtile; k += blockDim.x) keys[k] = km[k];
  __syncthreads();
  for (int r = threadIdx.x; r <= qt; r += blockDim.x) {
    const int t = d.y * qt + r;
    const bool real = r < qt && t < S;
    const int32_t rseg = real ? img[off_rseg + tok_off + t] : -1;
    const int32_t rord = real ? t + 1 : kInvalidOrd - 1;
    uint32_t w[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      uint32_t bits = 0;
      for (int i = 0; i < 32; ++i) {
        const int2 k = keys[32 * c + i];
        bits |= uint32_t((k.y <= rord) && ((k.x == rseg) || ((k.x | rseg) < 0))) << i;
      }
      w[c] = bits;
    }
    reinterpret_cast<int4*>(img + off_masks)[int64_t(m) * (qt + 1) + r] = make_int4(int(w[0]), int(w[1]), int(w[2]), int(w[3]));
  }
}

__global__ void page_copy_kernel(const uint64_t* __restrict__ src, const int32_t* __restrict__ dst_pages,
                                 char* dst_arena, int64_t page_bytes) {
  const uint4* s = reinterpret_cast<const uint4*>(src[blockIdx.x]);
  uint4* d = reinterpret_cast<uint4*>(dst_arena + int64_t(dst_pages[blockIdx.x]) * page_bytes);
  const int64_t n = page_bytes / 16;
  for (int64_t i = threadIdx.x; i < n; i += blockDim.x) d[i] = s[i];
}

}  // namespace

void launch_masks(int32_t* img, int64_t off_mdesc, int64_t off_qinfo, int64_t off_kmeta, int64_t off_rseg,
                  int64_t off_masks, int32_t n_masks, int32_t qt, cudaStream_t s) {
  if (n_masks <= 0) return;
  mask_kernel<<<n_masks, 128, 0, s>>>(img, off_mdesc, off_qinfo, off_kmeta, off_rseg, off_masks, qt);
  count_launch();
}

void launch_embed(const __nv_bfloat16* E, const int32_t* tok, float* h, int M, int H, cudaStream_t s) {
  if (M <= 0) return;
  embed_kernel<<<M, 128, 0, s>>>(E, tok, h, M, H);
  count_launch();
}
void launch_embed_norm(const __nv_bfloat16* E, const int32_t* tok, float* h, const __nv_bfloat16* g,
                       __nv_bfloat16* xg, float* ss, int M, int H, cudaStream_t s) {
  if (M <= 0) return;
  embed_norm_kernel<<<(M + 7) / 8, 256, 0, s>>>(E, tok, h, g, xg, ss, M, H);
  count_launch();
}
void launch_rmsnorm_bf16(const float* x, const __nv_bfloat16* g, __nv_bfloat16* y, int M, int H,
                         float eps, cudaStream_t s) {
  if (M <= 0) return;
  const int grid = (M + 7) / 8;
  switch (H) {  // register-resident rows for the model widths in use
    case 512: rmsnorm_reg_kernel<4><<<grid, 256, 0, s>>>(x, g, y, M, eps); break;
    case 768: rmsnorm_reg_kernel<6><<<grid, 256, 0, s>>>(x, g, y, M, eps); break;
    case 896: rmsnorm_reg_kernel<7><<<grid, 256, 0, s>>>(x, g, y, M, eps); break;
    case 1536: rmsnorm_reg_kernel<12><<<grid, 256, 0, s>>>(x, g, y, M, eps); break;
    case 2048: rmsnorm_reg_kernel<16><<<grid, 256, 0, s>>>(x, g, y, M, eps); break;
    case 3584: rmsnorm_reg_kernel<28><<<grid, 256, 0, s>>>(x, g, y, M, eps); break;
    default: rmsnorm_kernel<false><<<grid, 256, 0, s>>>(x, g, y, M, H, eps);
  }
  count_launch();
}
void launch_rmsnorm_f32out(const float* x, const __nv_bfloat16* g, float* y, int M, int H, float eps,
                           cudaStream_t s) {
  if (M <= 0) return;
  rmsnorm_kernel<true><<<(M + 7) / 8, 256, 0, s>>>(x, g, y, M, H, eps);
  count_launch();
}
void launch_rope_table(float2* tab, int max_pos, int d, double theta, cudaStream_t s) {
  rope_table_kernel<<<1024, 256, 0, s>>>(tab, max_pos, d, theta);
  count_launch();
}
void launch_stage(const StageParams& p, cudaStream_t s) {
  const int blocks = (p.n_qtiles + p.n_spages) * p.kv_heads;
  if (blocks <= 0) return;
  stage_kernel<<<blocks, 256, 0, s>>>(p);
  count_launch();
}
void launch_gather_rows_bf16(const __nv_bfloat16* src, const int32_t* idx, __nv_bfloat16* dst, int n,
                             int cols, cudaStream_t s) {
  if (n <= 0) return;
  gather_rows_kernel<__nv_bfloat16><<<n, 256, 0, s>>>(src, idx, dst, cols);
  count_launch();
}
void launch_gather_rows_f32(const float* src, const int32_t* idx, float* dst, int n, int cols,
                            cudaStream_t s) {
  if (n <= 0) return;
  gather_rows_kernel<float><<<n, 256, 0, s>>>(src, idx, dst, cols);
  count_launch();
}
template <class TW, bool MULTI = false>
static void score_launch(const float* hidden, const TW* w_out, const int32_t* labels, const int32_t* n_items, int B,
                         int n_max, int H, float* scores, int k, int32_t* topk, float* logits, cudaStream_t s) {
  if (B <= 0) return;
  const size_t smem = sizeof(float) * (size_t(H) + size_t(n_max));
  set_smem_attr(score_kernel<TW, MULTI>, 64 * 1024);
  score_kernel<TW, MULTI><<<B, 256, smem, s>>>(hidden, w_out, labels, n_items, n_max, H, scores, k, topk, logits);
  count_launch();
}
void launch_score_multi(const float* hidden, const __nv_bfloat16* w_bf16, const float* w_f32, const int32_t* labels,
                        const int32_t* n_items, int B, int n_max, int H, float* scores, int k, int32_t* topk,
                        float* logits, cudaStream_t s) {
  if (w_f32) score_launch<float, true>(hidden, w_f32, labels, n_items, B, n_max, H, scores, k, topk, logits, s);
  else score_launch<__nv_bfloat16, true>(hidden, w_bf16, labels, n_items, B, n_max, H, scores, k, topk, logits, s);
}
void launch_score(const float* hidden, const __nv_bfloat16* w_out, const int32_t* labels,
                  const int32_t* n_items, int B, int n_max, int H, float* scores, int k,
                  int32_t* topk, float* logits, cudaStream_t s) {
  score_launch(hidden, w_out, labels, n_items, B, n_max, H, scores, k, topk, logits, s);
}
void launch_score_f32w(const float* hidden, const float* w_out, const int32_t* labels, const int32_t* n_items, int B,
                       int n_max, int H, float* scores, int k, int32_t* topk, float* logits, cudaStream_t s) {
  score_launch(hidden, w_out, labels, n_items, B, n_max, H, scores, k, topk, logits, s);
}
void launch_kv_scatter(const PageIO& io, const __nv_bfloat16* k, const __nv_bfloat16* v,
                       const int32_t* pages_dev, int n_tokens, int slot0, int n_total, cudaStream_t s) {
  if (n_tokens <= 0) return;
  dim3 grid(n_tokens, io.layers);
  kv_pages_kernel<true><<<grid, 128, 0, s>>>(io, const_cast<__nv_bfloat16*>(k), const_cast<__nv_bfloat16*>(v),
                                             pages_dev, n_tokens, slot0, n_total);
  count_launch();
}
void launch_kv_gather(const PageIO& io, __nv_bfloat16* k, __nv_bfloat16* v, const int32_t* pages_dev,
                      int n_tokens, cudaStream_t s) {
  if (n_tokens <= 0) return;
  dim3 grid(n_tokens, io.layers);
  kv_pages_kernel<false><<<grid, 128, 0, s>>>(io, k, v, pages_dev, n_tokens, 0, n_tokens);
  count_launch();
}
void launch_page_copy(const uint64_t* src_ptrs, const int32_t* dst_pages, char* dst_arena,
                      int64_t page_bytes, int n, cudaStream_t s) {
  if (n <= 0) return;
  page_copy_kernel<<<n, 512, 0, s>>>(src_ptrs, dst_pages, dst_arena, page_bytes);
  count_launch();
}

}  // namespace bat
