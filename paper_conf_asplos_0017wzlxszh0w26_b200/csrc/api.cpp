// C ABI of libbat (include/bat.h): model, pool, prefill driver, score, plan introspection,
// HRCS placement and the NVLink page pull.  Host code only; device work is in k_*.cu.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <mutex>
#include <numeric>
#include <string>
#include <vector>

#include "common.h"
#include "kernels.h"
#include "plan.h"
#include "pool.h"

struct bat_model_s;
struct bat_pool_s {
  bat::Pool pool;
};
struct bat_plan_s {
  bat::Plan plan;
  void* dev_img = nullptr;  // device copy of plan.img (bat_plan_build)
  int device = -1;
  bat_pool_s* pool = nullptr;              // the pool whose page ids the device image holds
  std::vector<bat::EntityKey> pinned;      // entries pinned (not evictable) while the plan lives
  std::vector<int32_t> dev_copy;           // host copy of the device image (bat_plan_export_device)
  int32_t slot = -1;                       // staging slot of a bat_plan_build_staged plan
  std::vector<uint64_t> pull_src;          // its cold-item pulls: peer page addresses ...
  std::vector<int32_t> pull_dst;           // ... -> local staging pages
  // CUDA graph of this plan's prefill (bat_prefill_plan, BAT_GRAPH != 0): captured on the second
  // call (the first sizes the workspace), replayed while the workspace buffers, the output
  // pointer and the model are those it was captured with
  cudaGraphExec_t gexec = nullptr;
  uint64_t warm_gen = 0, graph_gen = 0;
  bool warm = false;
  const void* graph_model = nullptr;
  float* graph_out = nullptr;
  int64_t graph_launches = 0;
  ~bat_plan_s() {
    if (gexec) cudaGraphExecDestroy(gexec);
    if (dev_img) cudaFree(dev_img);
  }
};

namespace bat {

static thread_local std::string g_err;
void set_error(const std::string& m) { g_err = m; }
const char* last_error() { return g_err.c_str(); }

#define CUDA_OK(expr)                                                                    \
  do {                                                                                   \
    cudaError_t e_ = (expr);                                                             \
    if (e_ != cudaSuccess)                                                               \
      ::bat::fail(BAT_E_CUDA, std::string(#expr) + ": " + cudaGetErrorString(e_));       \
  } while (0)

// ---------------------------------------------------------------- tensor-map creation
using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                   const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                   const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                   CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  });
  if (!fn) fail(BAT_E_CUDA, "cuTensorMapEncodeTiled unavailable");
  return fn;
}

// row-major [rows][cols] with leading dimension ld (elements); box = [128 bytes of cols][box_rows],
// 128-byte swizzle (bf16: 64 columns; fp32: 32 columns)
static CUtensorMap make_tmap(const void* ptr, int64_t rows, int64_t cols, int64_t ld, int box_rows,
                             bool f32 = false) {
  CUtensorMap m;
  const int esz = f32 ? 4 : 2;
  cuuint64_t dims[2] = {cuuint64_t(cols), cuuint64_t(rows)};
  cuuint64_t strides[1] = {cuuint64_t(ld * esz)};
  cuuint32_t box[2] = {cuuint32_t(128 / esz), cuuint32_t(box_rows)};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = encode_fn()(&m, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2,
                           const_cast<void*>(ptr), dims,
                           strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                           CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fail(BAT_E_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string(int(r)) + ")");
  return m;
}


// ------------------------------------------------------------------------ device buffer
// bumped whenever a workspace buffer or the RoPE table is (re)allocated: a captured prefill
// graph holds their addresses (bat_prefill_plan)
static std::atomic<uint64_t> g_buf_gen{1};

struct DevBuf {
  void* p = nullptr;
  size_t cap = 0;
  // zero: clear on (re)allocation — q-tiles and suffix pages rely on never-written padding
  // (head-dim padding columns, rows 126-127 of a q-tile) staying zero
  // (on `st`, the stream of the work that then writes into the buffer: ordered with it for any
  // stream kind — a legacy-default-stream memset would not be with a non-blocking stream)
  void ensure(size_t bytes, cudaStream_t st, bool zero = false) {
    if (bytes <= cap) return;
    ++g_buf_gen;
    if (p) {
      CUDA_OK(cudaStreamSynchronize(st));  // the old buffer may still be read by queued work
      cudaFree(p);
    }
    p = nullptr;
    cap = 0;
    size_t want = std::max(bytes, size_t(1) << 16);
    want = (want + (want >> 2) + 255) & ~size_t(255);
    CUDA_OK(cudaMalloc(&p, want));
    if (zero) CUDA_OK(cudaMemsetAsync(p, 0, want, st));
    cap = want;
  }
  ~DevBuf() {
    if (p) cudaFree(p);
  }
  template <class T>
  T* as() const { return static_cast<T*>(p); }
};

struct Workspace {
  DevBuf h, xn, qkv, qp, scratch, o, act, hc, xc, oc, actc, img, small, part_o, part_ml, gpart, ss;
  void* img_host = nullptr;
  size_t img_host_cap = 0;
  cudaEvent_t img_done = nullptr;
  ~Workspace() {
    if (img_host) cudaFreeHost(img_host);
    if (img_done) cudaEventDestroy(img_done);
  }
};

// CUDA-event timing of every launch of the prefill, grouped by kernel class
struct Profiler {
  bool on = false;
  struct Rec {
    cudaEvent_t a, b;
    int cls;
    double flops, bytes;
  };
  std::vector<Rec> recs;
  std::vector<cudaEvent_t> spare;
  double ms[BAT_K_N] = {0}, flops[BAT_K_N] = {0}, bytes[BAT_K_N] = {0};
  int64_t n[BAT_K_N] = {0};
  cudaEvent_t ev() {
    if (!spare.empty()) {
      cudaEvent_t e = spare.back();
      spare.pop_back();
      return e;
    }
    cudaEvent_t e;
    CUDA_OK(cudaEventCreate(&e));
    return e;
  }
  void begin(cudaStream_t st) {
    if (!on) return;
    Rec r{ev(), nullptr, 0, 0, 0};
    CUDA_OK(cudaEventRecord(r.a, st));
    recs.push_back(r);
  }
  void end(cudaStream_t st, int cls, double fl, double by) {
    if (!on) return;
    Rec& r = recs.back();
    r.b = ev();
    r.cls = cls;
    r.flops = fl;
    r.bytes = by;
    CUDA_OK(cudaEventRecord(r.b, st));
  }
  void collect() {
    for (Rec& r : recs) {
      CUDA_OK(cudaEventSynchronize(r.b));
      float t = 0;
      CUDA_OK(cudaEventElapsedTime(&t, r.a, r.b));
      ms[r.cls] += t;
      flops[r.cls] += r.flops;
      bytes[r.cls] += r.bytes;
      n[r.cls] += 1;
      spare.push_back(r.a);
      spare.push_back(r.b);
    }
    recs.clear();
  }
  void reset() {
    collect();
    for (int i = 0; i < BAT_K_N; ++i) ms[i] = flops[i] = bytes[i] = 0, n[i] = 0;
  }
  ~Profiler() {
    for (Rec& r : recs) {
      cudaEventDestroy(r.a);
      if (r.b) cudaEventDestroy(r.b);
    }
    for (cudaEvent_t e : spare) cudaEventDestroy(e);
  }
};

struct Model {
  Profiler prof;
  bat_model_cfg cfg{};
  int device = 0, num_sms = 148, dpad = 128;
  const __nv_bfloat16 *embed = nullptr, *lm_head = nullptr, *final_norm = nullptr;
  struct Layer {
    const __nv_bfloat16 *ln1, *wqkv, *bqkv, *wo, *ln2, *wgu, *wd;
    CUtensorMap t_qkv, t_o, t_gu, t_d;
  };
  std::vector<Layer> layers;
  std::vector<const void*> w;  // every weight pointer as passed (the fp32 mode reads these)
  bool f32 = false;
  float2* rope = nullptr;
  int max_pos = 0;
  Workspace ws;
  ~Model() {
    if (rope) cudaFree(rope);
  }
  int nqkv() const { return (cfg.q_heads + 2 * cfg.kv_heads) * cfg.head_dim; }
};

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (dev >= 0 && dev != prev) CUDA_OK(cudaSetDevice(dev));
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

static void ensure_rope(Model& m, int need_pos, cudaStream_t st) {
  if (need_pos <= m.max_pos) return;
  int np = std::max(32768, m.max_pos);
  while (np < need_pos) np *= 2;
  ++g_buf_gen;
  if (m.rope) {
    CUDA_OK(cudaStreamSynchronize(st));
    cudaFree(m.rope);
    m.rope = nullptr;
  }
  CUDA_OK(cudaMalloc(&m.rope, sizeof(float2) * size_t(np) * (m.cfg.head_dim / 2)));
  launch_rope_table(m.rope, np, m.cfg.head_dim, double(m.cfg.rope_theta), st);
  m.max_pos = np;
}

static PageIO page_io(const Pool& p) {
  PageIO io;
  io.arena = p.arena;
  io.page_bytes = p.geo.page_bytes;
  io.layer_bytes = p.geo.layer_bytes;
  io.head_bytes = p.geo.head_bytes;
  io.layers = p.geo.layers;
  io.kv_heads = p.geo.kv_heads;
  io.head_dim = p.geo.head_dim;
  return io;
}

static void check_compat(const Pool& p, const Model& m) {
  if (p.index_only) fail(BAT_E_STATE, "index-only pool cannot run device work");
  BAT_REQUIRE(p.cfg.layers == m.cfg.layers && p.cfg.kv_heads == m.cfg.kv_heads &&
                  p.cfg.head_dim == m.cfg.head_dim && p.cfg.dtype == m.cfg.dtype,
              "pool geometry / dtype does not match the model");
  BAT_REQUIRE(p.device == m.device, "pool and model are on different devices");
}

// Device-side part of a plan image: the visibility masks of its partial tiles.
static void build_masks(const Plan& plan, int32_t* dev_img, cudaStream_t st) {
  const PlanImage& im = plan.img;
  launch_masks(dev_img, im.off_mdesc, im.off_qinfo, im.off_kmeta, im.off_rseg, im.off_masks, im.n_masks, plan.qt, st);
}

// Workspace sizing + plan upload; returns the device image.
static const int32_t* prepare(Pool& pool, Model& m, Plan& plan, cudaStream_t st,
                              const int32_t* dev_img = nullptr) {
  const bat_model_cfg& c = m.cfg;
  Workspace& ws = m.ws;
  const int M = plan.M, B = static_cast<int>(plan.q.size());
  const int H = c.hidden, F = c.ffn, nq = c.q_heads * c.head_dim;
  const int64_t tile_bytes = int64_t(m.dpad / 64) * 16384;
  int max_pos = 0;
  for (auto& q : plan.q)
    for (int32_t ps : q.pos) max_pos = std::max(max_pos, ps);
  ensure_rope(m, max_pos + 1, st);
  const size_t es = m.f32 ? 4 : 2;  // activation element size
  ws.h.ensure(size_t(M) * H * 4, st);
  ws.xn.ensure(size_t(M) * std::max(H, nq) * es, st);
  ws.qkv.ensure(size_t(M) * m.nqkv() * es, st);
  if (m.f32) ws.qp.ensure(size_t(M) * nq * 4, st);
  else ws.qp.ensure(size_t(plan.n_qtiles_total) * c.kv_heads * tile_bytes, st, true);
  ws.scratch.ensure(size_t(std::max(plan.n_spages, 1)) * pool.geo.layer_bytes, st, true);
  ws.o.ensure(size_t(M) * nq * es, st);
  ws.act.ensure(size_t(M) * F * es, st);
  const size_t D = size_t(B) * plan.n_disc;  // discriminant rows
  ws.hc.ensure(D * H * 4, st);
  ws.xc.ensure(D * H * es, st);
  ws.oc.ensure(D * nq * es, st);
  ws.actc.ensure(D * F * es, st);
  const int64_t slots = std::max(plan.img.n_slots, plan.img.n_slots_last);
  if (slots > 0 && !m.f32) {  // split-KV partials (small batches)
    ws.part_o.ensure(size_t(slots) * 2 * 128 * m.dpad * 4, st);
    ws.part_ml.ensure(size_t(slots) * 2 * 128 * 8, st);
  }
  if (dev_img) return dev_img;
  const size_t img_bytes = plan.img.buf.size() * 4;
  ws.img.ensure(size_t(plan.img.total_ints) * 4, st);
  if (!ws.img_done) CUDA_OK(cudaEventCreateWithFlags(&ws.img_done, cudaEventDisableTiming));
  CUDA_OK(cudaEventSynchronize(ws.img_done));  // the previous upload finished reading the staging buffer
  if (ws.img_host_cap < img_bytes) {
    if (ws.img_host) cudaFreeHost(ws.img_host);
    ws.img_host_cap = img_bytes + img_bytes / 4 + 4096;
    CUDA_OK(cudaMallocHost(&ws.img_host, ws.img_host_cap));
  }
  std::memcpy(ws.img_host, plan.img.buf.data(), img_bytes);
  CUDA_OK(cudaMemcpyAsync(ws.img.p, ws.img_host, img_bytes, cudaMemcpyHostToDevice, st));
  CUDA_OK(cudaEventRecord(ws.img_done, st));
  build_masks(plan, ws.img.as<int32_t>(), st);
  return ws.img.as<int32_t>();
}

static AttnParams attn_params(const Pool& pool, const Model& m, const Plan& plan, const int32_t* I) {
  const bat_model_cfg& c = m.cfg;
  const PlanImage& im = plan.img;
  AttnParams ap{};
  ap.img = I;
  ap.off_qinfo = im.off_qinfo;
  ap.off_pages = im.off_pages;
  ap.off_kmeta = im.off_kmeta;
  ap.off_rseg = im.off_rseg;
  ap.off_work = im.off_work;
  ap.n_work = plan.n_work;
  ap.pool = pool.arena;
  ap.pool_page_bytes = pool.geo.page_bytes;
  ap.scratch = m.ws.scratch.as<char>();
  ap.scratch_page_bytes = pool.geo.layer_bytes;
  ap.scratch_layer_off = 0;
  ap.zero_page = pool.arena + int64_t(pool.zero_page) * pool.geo.page_bytes;
  ap.head_bytes = pool.geo.head_bytes;
  ap.kv_heads = c.kv_heads;
  ap.group = plan.group;
  ap.qt = plan.qt;
  ap.head_dim = c.head_dim;
  ap.ldo = c.q_heads * c.head_dim;
  ap.qp = m.ws.qp.as<__nv_bfloat16>();
  ap.out = m.ws.o.as<__nv_bfloat16>();
  ap.scale_log2 = float(1.4426950408889634 / std::sqrt(double(c.head_dim)));
  ap.off_masks = im.off_masks;
  ap.off_wslot = im.off_wslot;
  const bool split = std::max(im.n_slots, im.n_slots_last) > 0;
  ap.part_o = split ? m.ws.part_o.as<float>() : nullptr;
  ap.part_ml = split ? m.ws.part_ml.as<float>() : nullptr;
  return ap;
}

// a5 launch (persistent tcgen05 kernel, one CTA per SM) over the main (last = false) or the
// last-layer work list, then the split-KV combine of that list's split items (if any)
static void run_attention(const Pool&, const Model& m, const Plan& plan, AttnParams ap, bool last, cudaStream_t st) {
  const PlanImage& im = plan.img;
  ap.off_work = last ? im.off_work_last : im.off_work;
  ap.n_work = last ? plan.n_work_last : plan.n_work;
  ap.off_wslot = last ? im.off_wslot_last : im.off_wslot;
  launch_attention(m.dpad, ap, m.num_sms, st);
  if (ap.part_o) launch_attention_combine(m.dpad, ap, last ? im.off_sgrp_last : im.off_sgrp,
                                          last ? im.n_sgrp_last : im.n_sgrp, st);
}

static StageParams stage_params(const Pool& pool, const Model& m, const Plan& plan, const int32_t* I) {
  const bat_model_cfg& c = m.cfg;
  const PlanImage& im = plan.img;
  StageParams sp{};
  sp.qkv = m.ws.qkv.as<__nv_bfloat16>();
  sp.img = I;
  sp.off_pos = im.off_pos;
  sp.off_qinfo = im.off_qinfo;
  sp.off_qtiles = im.off_qtiles;
  sp.off_spages = im.off_spages;
  sp.n_qtiles = plan.n_qtiles_total;
  sp.n_spages = plan.n_spages;
  sp.rope = m.rope;
  sp.rope_enabled = 1;
  sp.max_pos = m.max_pos;
  sp.q_heads = c.q_heads;
  sp.kv_heads = c.kv_heads;
  sp.head_dim = c.head_dim;
  sp.dpad = m.dpad;
  sp.group = plan.group;
  sp.qt = plan.qt;
  sp.qp = m.ws.qp.as<__nv_bfloat16>();
  sp.pool = pool.arena;
  sp.pool_page_bytes = pool.geo.page_bytes;
  sp.scratch = m.ws.scratch.as<char>();
  sp.scratch_page_bytes = pool.geo.layer_bytes;
  sp.scratch_layer_off = 0;
  sp.head_bytes = pool.geo.head_bytes;
  sp.n_req = static_cast<int32_t>(plan.q.size());
  sp.off_rowreq = im.off_rowreq;
  return sp;
}

// FP32 SIMT correctness mode (k_f32.cu): the same steps in plain fp32, no last-layer trim (the
// discriminant rows are picked by the final norm), no kernel profiling.
static void run_plan_f32(Pool& pool, Model& m, Plan& plan, float* out_hidden, cudaStream_t st,
                         const int32_t* dev_img) {
  const bat_model_cfg& c = m.cfg;
  Workspace& ws = m.ws;
  const int M = plan.M, B = static_cast<int>(plan.q.size());
  const int H = c.hidden, F = c.ffn, nq = c.q_heads * c.head_dim, nqkv = m.nqkv();
  const int32_t* I = prepare(pool, m, plan, st, dev_img);
  const PlanImage& im = plan.img;
  auto W = [&](int i) { return static_cast<const float*>(m.w[i]); };
  auto WL = [&](int l, int j) { return W(BAT_W_N_GLOBAL + BAT_WL_N * l + j); };
  float *h = ws.h.as<float>(), *xn = ws.xn.as<float>(), *qkv = ws.qkv.as<float>(), *o = ws.o.as<float>(),
        *act = ws.act.as<float>();
  int max_S = 0;
  for (auto& q : plan.q) max_S = std::max(max_S, q.S);
  StageF32Params sp{};
  sp.qkv = qkv;
  sp.img = I;
  sp.off_pos = im.off_pos;
  sp.off_qinfo = im.off_qinfo;
  sp.off_spages = im.off_spages;
  sp.M = M;
  sp.n_spages = plan.n_spages;
  sp.rope = m.rope;
  sp.rope_enabled = 1;
  sp.max_pos = m.max_pos;
  sp.q_heads = c.q_heads;
  sp.kv_heads = c.kv_heads;
  sp.head_dim = c.head_dim;
  sp.qf = ws.qp.as<float>();
  sp.pool = pool.arena;
  sp.pool_page_bytes = pool.geo.page_bytes;
  sp.scratch = ws.scratch.as<char>();
  sp.scratch_page_bytes = pool.geo.layer_bytes;
  AttnF32Params ap{};
  ap.img = I;
  ap.off_qinfo = im.off_qinfo;
  ap.off_pages = im.off_pages;
  ap.off_kmeta = im.off_kmeta;
  ap.off_rseg = im.off_rseg;
  ap.pool = pool.arena;
  ap.pool_page_bytes = pool.geo.page_bytes;
  ap.scratch = ws.scratch.as<char>();
  ap.scratch_page_bytes = pool.geo.layer_bytes;
  ap.q_heads = c.q_heads;
  ap.kv_heads = c.kv_heads;
  ap.group = c.q_heads / c.kv_heads;
  ap.head_dim = c.head_dim;
  ap.qf = ws.qp.as<float>();
  ap.out = o;
  ap.scale = float(1.0 / std::sqrt(double(c.head_dim)));
  launch_embed_f32(W(BAT_W_EMBED), I + im.off_tok, h, M, H, st);
  for (int l = 0; l < c.layers; ++l) {
    launch_rmsnorm_f32(h, WL(l, BAT_WL_LN1), xn, nullptr, M, H, c.rms_eps, st);
    launch_gemm_f32(0, xn, WL(l, BAT_WL_WQKV), WL(l, BAT_WL_BQKV), qkv, M, nqkv, H, 0, st);
    sp.pool_layer_off = int64_t(l) * pool.geo.layer_bytes;
    launch_stage_f32(sp, st);
    if (l == c.layers - 1 && plan.entity_mode) break;
    ap.pool_layer_off = sp.pool_layer_off;
    launch_attention_f32(ap, B, max_S, st);
    launch_gemm_f32(1, o, WL(l, BAT_WL_WO), nullptr, h, M, H, nq, 0, st);
    launch_rmsnorm_f32(h, WL(l, BAT_WL_LN2), xn, nullptr, M, H, c.rms_eps, st);
    launch_gemm_f32(2, xn, WL(l, BAT_WL_WGU), nullptr, act, M, F, H, F, st);
    launch_gemm_f32(1, act, WL(l, BAT_WL_WD), nullptr, h, M, H, F, 0, st);
  }
  if (out_hidden && !plan.entity_mode)
    launch_rmsnorm_f32(h, W(BAT_W_FINAL_NORM), out_hidden, I + im.off_disc, B * plan.n_disc, H, c.rms_eps, st);
  CUDA_OK(cudaGetLastError());
}

// Run the L layers over a planned batch (SURVEY §3 call stack (3)).
static void run_plan(Pool& pool, Model& m, Plan& plan, float* out_hidden, cudaStream_t st,
                     const int32_t* dev_img = nullptr) {
  const bat_model_cfg& c = m.cfg;
  Workspace& ws = m.ws;
  const int M = plan.M, B = static_cast<int>(plan.q.size());
  const int H = c.hidden, F = c.ffn;
  const int nq = c.q_heads * c.head_dim;
  if (m.f32) return run_plan_f32(pool, m, plan, out_hidden, st, dev_img);
  const int32_t* I = prepare(pool, m, plan, st, dev_img);
  Profiler& pf = m.prof;
  const double d_ = c.head_dim, Hq_ = c.q_heads, Hkv_ = c.kv_heads;
  auto gemm_fb = [&](int Mr, int N, int K, int out_bytes) {
    return std::make_pair(2.0 * Mr * N * K, 2.0 * (double(Mr) * K + double(N) * K) + double(out_bytes) * Mr * N);
  };
  double live_all = 0, live_last = 0, kv_slots = 0;
  for (auto& q : plan.q) {
    live_all += double(q.n_live_pairs);
    live_last += double(q.n_live_pairs_last);
    kv_slots += double(q.n_pages) * kPageTokens;
  }
  const double attn_fl = 4.0 * d_ * Hq_ * live_all, attn_fl_last = 4.0 * d_ * Hq_ * live_last;
  const double attn_by = 2.0 * 2.0 * M * Hq_ * d_ + 2.0 * 2.0 * kv_slots * Hkv_ * d_;
  const PlanImage& im = plan.img;

  // tensor maps of this call's activations
  const CUtensorMap tA_xn = make_tmap(ws.xn.p, M, H, H, 128);
  const CUtensorMap tA_o = make_tmap(ws.o.p, M, nq, nq, 128);
  const CUtensorMap tA_act = make_tmap(ws.act.p, M, F, F, 128);
  const int Dr = B * plan.n_disc;  // discriminant rows (multi_disc: n_disc per request)
  const CUtensorMap tA_xc = make_tmap(ws.xc.p, Dr, H, H, 128);
  const CUtensorMap tA_oc = make_tmap(ws.oc.p, Dr, nq, nq, 128);
  const CUtensorMap tA_actc = make_tmap(ws.actc.p, Dr, F, F, 128);
  // outputs (epilogue TMA store / reduce-add, 32-row boxes)
  const CUtensorMap tC_qkv = make_tmap(ws.qkv.p, M, m.nqkv(), m.nqkv(), 32);
  const CUtensorMap tC_h = make_tmap(ws.h.p, M, H, H, 32, true);
  const CUtensorMap tC_act = make_tmap(ws.act.p, M, F, F, 32);
  const CUtensorMap tC_hc = make_tmap(ws.hc.p, Dr, H, H, 32, true);
  const CUtensorMap tC_actc = make_tmap(ws.actc.p, Dr, F, F, 32);
  AttnParams ap = attn_params(pool, m, plan, I);
  StageParams sp = stage_params(pool, m, plan, I);
  // a dense projection; split-K (deterministic fp32 partials + an ordered reduce) when its tile
  // grid would leave SMs idle — batch-1 requests, the last layer's discriminant rows
  auto gemm = [&](int epi, const CUtensorMap& tA, const CUtensorMap& tB, const CUtensorMap& tC, const GemmParams& gp) {
    int mpad = 0;
    const int ks = (epi == EPI_RESID_F32 || epi == EPI_BF16_BIAS) ? gemm_ksplit(epi, gp.M, gp.N, gp.K, m.num_sms, &mpad) : 1;
    if (ks <= 1) {
      launch_gemm(epi, tA, tB, tC, gp, m.num_sms, st);
      return;
    }
    ws.gpart.ensure(size_t(ks) * mpad * gp.N * 4, st);
    const CUtensorMap tP = make_tmap(ws.gpart.p, int64_t(ks) * mpad, gp.N, gp.N, 32, true);
    GemmParams pp = gp;
    pp.ksplit = ks;
    pp.mpad = mpad;
    launch_gemm(EPI_PART_F32, tA, tB, tP, pp, m.num_sms, st);
    launch_gemm_reduce(ws.gpart.as<float>(), ks, mpad, gp.M, gp.N, gp.out, gp.ldo,
                       epi == EPI_BF16_BIAS ? gp.bias : nullptr, epi == EPI_RESID_F32 ? 0 : 1, st);
  };

  // RMSNorm fused across the residual updates (GemmParams::norm_g / ss_in; large batches only: no
  // projection of a full-row layer on the split-K path).  Default (BAT_FUSED_NORM=d): the
  // attention-block norm (ln1) rides on the down GEMM's epilogue (long K: slack to absorb it) and
  // the embedding, the MLP norm (ln2) stays a kernel; =1: ln2 on the O GEMM too (short K: its
  // epilogue becomes the bottleneck, a net loss); =0: standalone norm kernels
  // (profiles/r2_gemm_epilogue.txt)
  const char* fuse_e = std::getenv("BAT_FUSED_NORM");  // read per call: tests A/B the paths
  const char fuse_mode = fuse_e ? fuse_e[0] : 'd';
  const bool fuse_env = fuse_mode == '1' || fuse_mode == 'd';
  const bool fuse_ok = fuse_env && (H % 32) == 0 &&
                         gemm_ksplit(EPI_BF16_BIAS, M, m.nqkv(), H, m.num_sms, nullptr) <= 1 &&
                         gemm_ksplit(EPI_RESID_F32, M, H, nq, m.num_sms, nullptr) <= 1 &&
                         gemm_ksplit(EPI_RESID_F32, M, H, F, m.num_sms, nullptr) <= 1;
  // a4 (RoPE + q-tile / page staging) fused into the QKV epilogue unless BAT_FUSED_STAGE=0 or the
  // QKV projection takes the split-K path (small batches: partial sums, then stage_kernel)
  const char* fst_e = std::getenv("BAT_FUSED_STAGE");
  const bool fuse_stage = !(fst_e && fst_e[0] == '0') && gemm_qkv_stage_fusable(c.head_dim) &&
                          gemm_ksplit(EPI_BF16_BIAS, M, m.nqkv(), H, m.num_sms, nullptr) <= 1;
  const int ss_parts_resid = (H + 255) / 256 * gemm_epi_col_splits();  // (N-tile, slice) partial sums
  const bool fuse_norm = fuse_ok && ss_parts_resid <= 32;                  // row_rstd loads <= 32 parts
  const bool fuse_norm2 = fuse_norm && fuse_mode == '1';                   // ln2 through the O GEMM too
  if (fuse_norm) ws.ss.ensure(size_t(ss_parts_resid) * M * 4, st);
  auto set_norm_out = [&](GemmParams& g, const __nv_bfloat16* gnext) {  // producer: h += .., xn, ss
    g.norm_g = gnext;
    g.xg_out = ws.xn.as<__nv_bfloat16>();
    g.ss_out = ws.ss.as<float>();
    g.norm_h = H;
  };
  auto set_norm_in = [&](GemmParams& g, int parts) {  // consumer: rows scaled by rsqrt(mean h^2 + eps)
    g.ss_in = ws.ss.as<float>();
    g.ss_parts = parts;
    g.norm_h = H;
    g.eps = c.rms_eps;
  };
  pf.begin(st);
  if (fuse_norm)
    launch_embed_norm(m.embed, I + im.off_tok, ws.h.as<float>(), m.layers[0].ln1, ws.xn.as<__nv_bfloat16>(),
                      ws.ss.as<float>(), M, H, st);
  else
    launch_embed(m.embed, I + im.off_tok, ws.h.as<float>(), M, H, st);
  pf.end(st, BAT_K_EMBED, 0, (fuse_norm ? 8.0 : 6.0) * M * H);
  for (int l = 0; l < c.layers; ++l) {
    const Model::Layer& Lw = m.layers[l];
    const bool last = (l == c.layers - 1);
    GemmParams gp{M, m.nqkv(), H, ws.qkv.p, m.nqkv(), Lw.bqkv, 0};
    if (fuse_norm) {
      set_norm_in(gp, l == 0 ? 1 : ss_parts_resid);
    } else {
      pf.begin(st);
      launch_rmsnorm_bf16(ws.h.as<float>(), Lw.ln1, ws.xn.as<__nv_bfloat16>(), M, H, c.rms_eps, st);
      pf.end(st, BAT_K_RMSNORM, 0, 6.0 * M * H);
    }
    auto fq = gemm_fb(M, m.nqkv(), H, 2);
    sp.pool_layer_off = int64_t(l) * pool.geo.layer_bytes;
    if (fuse_stage) {  // a4 in the QKV epilogue: q-tiles and suffix pages written directly
      gp.stage_on = 1;
      gp.stage = sp;
    }
    pf.begin(st);
    gemm(EPI_BF16_BIAS, tA_xn, Lw.t_qkv, tC_qkv, gp);
    pf.end(st, BAT_K_GEMM_QKV, fq.first, fq.second);
    if (!fuse_stage) {
      pf.begin(st);
      launch_stage(sp, st);
      pf.end(st, BAT_K_STAGE, 0, 4.0 * M * m.nqkv());
    }
    if (last && plan.entity_mode) break;  // entity prefill: only this layer's K/V are needed
    ap.pool_layer_off = int64_t(l) * pool.geo.layer_bytes;
    if (!last) {
      // debug (BAT_ATTN_ITEMS=file, BAT_ATTN_LAYER=l): per-work-item clock64 records of one layer
      static const char* items_file = std::getenv("BAT_ATTN_ITEMS");
      static const int items_layer = std::getenv("BAT_ATTN_LAYER") ? std::atoi(std::getenv("BAT_ATTN_LAYER")) : 1;
      long long* dbi = nullptr;
      if (items_file && l == items_layer) {
        CUDA_OK(cudaMalloc(&dbi, size_t(ap.n_work) * 6 * sizeof(long long)));
        CUDA_OK(cudaMemsetAsync(dbi, 0, size_t(ap.n_work) * 6 * sizeof(long long), st));
      }
      ap.dbg_items = dbi;
      pf.begin(st);
      run_attention(pool, m, plan, ap, false, st);
      pf.end(st, BAT_K_ATTN, attn_fl, attn_by);
      ap.dbg_items = nullptr;
      if (dbi) {
        std::vector<long long> h(size_t(ap.n_work) * 6);
        CUDA_OK(cudaMemcpyAsync(h.data(), dbi, h.size() * sizeof(long long), cudaMemcpyDeviceToHost, st));
        CUDA_OK(cudaStreamSynchronize(st));
        if (FILE* f = std::fopen(items_file, "w")) {
          for (int w = 0; w < ap.n_work; ++w) {
            for (int e = 0; e < 6; ++e) std::fprintf(f, "%lld ", h[size_t(w) * 6 + e]);
            std::fprintf(f, "\n");
          }
          std::fclose(f);
        }
        cudaFree(dbi);
      }
      GemmParams go{M, H, nq, ws.h.p, H, nullptr, 0};
      if (fuse_norm2) set_norm_out(go, Lw.ln2);
      auto fo = gemm_fb(M, H, nq, fuse_norm2 ? 10 : 8);
      pf.begin(st);
      gemm(EPI_RESID_F32, tA_o, Lw.t_o, tC_h, go);
      pf.end(st, BAT_K_GEMM_O, fo.first, fo.second);
      GemmParams gg{M, F, H, ws.act.p, F, nullptr, F};
      if (fuse_norm2) {
        set_norm_in(gg, ss_parts_resid);
      } else {
        pf.begin(st);
        launch_rmsnorm_bf16(ws.h.as<float>(), Lw.ln2, ws.xn.as<__nv_bfloat16>(), M, H, c.rms_eps, st);
        pf.end(st, BAT_K_RMSNORM, 0, 6.0 * M * H);
      }
      auto fg = gemm_fb(M, 2 * F, H, 1);
      pf.begin(st);
      launch_gemm(EPI_SWIGLU, tA_xn, Lw.t_gu, tC_act, gg, m.num_sms, st);
      pf.end(st, BAT_K_GEMM_GU, fg.first, fg.second);
      GemmParams gd{M, H, F, ws.h.p, H, nullptr, 0};
      // the next layer's RMSNorm rides on this residual update (its K/V are needed: not the last)
      if (fuse_norm) set_norm_out(gd, m.layers[l + 1].ln1);
      auto fd = gemm_fb(M, H, F, fuse_norm ? 10 : 8);
      pf.begin(st);
      gemm(EPI_RESID_F32, tA_act, Lw.t_d, tC_h, gd);
      pf.end(st, BAT_K_GEMM_DOWN, fd.first, fd.second);
    } else {
      // a8: after the last layer's K/V only the discriminant rows matter; with one
      // discriminant per item they are spread over the suffix: attend for every row
      pf.begin(st);
      run_attention(pool, m, plan, ap, !plan.multi_disc, st);
      pf.end(st, BAT_K_ATTN, plan.multi_disc ? attn_fl : attn_fl_last, attn_by);
      const int32_t* disc = I + im.off_disc;
      pf.begin(st);
      launch_gather_rows_bf16(ws.o.as<__nv_bfloat16>(), disc, ws.oc.as<__nv_bfloat16>(), Dr, nq, st);
      launch_gather_rows_f32(ws.h.as<float>(), disc, ws.hc.as<float>(), Dr, H, st);
      pf.end(st, BAT_K_OTHER, 0, 2.0 * Dr * (2.0 * nq + 4.0 * H));
      GemmParams go{Dr, H, nq, ws.hc.p, H, nullptr, 0};
      auto fo = gemm_fb(Dr, H, nq, 8);
      pf.begin(st);
      gemm(EPI_RESID_F32, tA_oc, Lw.t_o, tC_hc, go);
      pf.end(st, BAT_K_GEMM_O, fo.first, fo.second);
      pf.begin(st);
      launch_rmsnorm_bf16(ws.hc.as<float>(), Lw.ln2, ws.xc.as<__nv_bfloat16>(), Dr, H, c.rms_eps, st);
      pf.end(st, BAT_K_RMSNORM, 0, 6.0 * Dr * H);
      GemmParams gg{Dr, F, H, ws.actc.p, F, nullptr, F};
      auto fg = gemm_fb(Dr, 2 * F, H, 1);
      pf.begin(st);
      launch_gemm(EPI_SWIGLU, tA_xc, Lw.t_gu, tC_actc, gg, m.num_sms, st);
      pf.end(st, BAT_K_GEMM_GU, fg.first, fg.second);
      GemmParams gd{Dr, H, F, ws.hc.p, H, nullptr, 0};
      auto fd = gemm_fb(Dr, H, F, 8);
      pf.begin(st);
      gemm(EPI_RESID_F32, tA_actc, Lw.t_d, tC_hc, gd);
      pf.end(st, BAT_K_GEMM_DOWN, fd.first, fd.second);
      pf.begin(st);
      launch_rmsnorm_f32out(ws.hc.as<float>(), m.final_norm, out_hidden, Dr, H, c.rms_eps, st);
      pf.end(st, BAT_K_OTHER, 0, 8.0 * Dr * H);
    }
  }
  CUDA_OK(cudaGetLastError());
}

static int64_t key_kind_check(int32_t kind) {
  BAT_REQUIRE(kind == BAT_ENT_USER || kind == BAT_ENT_ITEM || kind == BAT_ENT_HEADER, "entity kind");
  return kind;
}

}  // namespace bat

using namespace bat;

struct bat_model_s {
  Model m;
};

extern "C" {

const char* bat_last_error(void) { return bat::last_error(); }
const char* bat_version(void) { return "bat-b200 0.1 (sm_100a)"; }
int64_t bat_kernel_launch_count(void) { return bat::launch_count(); }

bat_status bat_model_create(const bat_model_cfg* cfg, const void* const* weights, int32_t n_weights,
                            int32_t device, bat_model* out) {
  return guarded([&] {
    BAT_REQUIRE(cfg && weights && out, "null argument");
    const bat_model_cfg& c = *cfg;
    BAT_REQUIRE(c.dtype == BAT_BF16 || c.dtype == BAT_FP32, "dtype must be BAT_BF16 or BAT_FP32");
    BAT_REQUIRE(c.layers >= 1 && c.hidden >= 64 && c.hidden % 64 == 0, "hidden % 64 == 0");
    BAT_REQUIRE(c.head_dim == 16 || c.head_dim == 32 || c.head_dim == 64 || c.head_dim == 128,
                "head_dim in {16,32,64,128}");
    BAT_REQUIRE(c.kv_heads >= 1 && c.q_heads % c.kv_heads == 0 && c.q_heads / c.kv_heads <= 128,
                "q_heads % kv_heads == 0 and group <= 128");
    BAT_REQUIRE(c.ffn % 128 == 0, "ffn % 128 == 0");
    BAT_REQUIRE((c.q_heads * c.head_dim) % 64 == 0, "q_heads*head_dim % 64 == 0");
    BAT_REQUIRE(c.vocab >= 1, "vocab");
    BAT_REQUIRE(n_weights == BAT_W_N_GLOBAL + BAT_WL_N * c.layers, "n_weights == 3 + 7*layers");
    for (int i = 0; i < n_weights; ++i) BAT_REQUIRE(weights[i] != nullptr, "null weight pointer");
    DeviceGuard dg(device);
    auto mp = std::make_unique<bat_model_s>();
    Model& m = mp->m;
    m.cfg = c;
    m.device = device;
    m.dpad = head_dim_pad(c.head_dim);
    CUDA_OK(cudaDeviceGetAttribute(&m.num_sms, cudaDevAttrMultiProcessorCount, device));
    int major = 0;
    CUDA_OK(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, device));
    if (major != 10) fail(BAT_E_UNSUPPORTED, "libbat kernels are sm_100a (B200) only");
    m.w.assign(weights, weights + n_weights);
    m.f32 = c.dtype == BAT_FP32;
    auto W = [&](int i) { return static_cast<const __nv_bfloat16*>(weights[i]); };
    m.embed = W(BAT_W_EMBED);
    m.lm_head = W(BAT_W_LM_HEAD);
    m.final_norm = W(BAT_W_FINAL_NORM);
    const int H = c.hidden, nq = c.q_heads * c.head_dim, F = c.ffn;
    for (int l = 0; l < c.layers; ++l) {
      auto w = [&](int j) { return W(BAT_W_N_GLOBAL + BAT_WL_N * l + j); };
      Model::Layer L{};
      L.ln1 = w(BAT_WL_LN1);
      L.wqkv = w(BAT_WL_WQKV);
      L.bqkv = w(BAT_WL_BQKV);
      L.wo = w(BAT_WL_WO);
      L.ln2 = w(BAT_WL_LN2);
      L.wgu = w(BAT_WL_WGU);
      L.wd = w(BAT_WL_WD);
      if (!m.f32) {  // bf16 product path: TMA descriptors of the weights
        L.t_qkv = make_tmap(L.wqkv, m.nqkv(), H, H, 128);
        L.t_o = make_tmap(L.wo, H, nq, nq, 128);
        L.t_gu = make_tmap(L.wgu, 2 * int64_t(F), H, H, 128);
        L.t_d = make_tmap(L.wd, H, F, F, 128);
      }
      m.layers.push_back(L);
    }
    ensure_rope(m, 32768, 0);
    CUDA_OK(cudaStreamSynchronize(0));
    *out = mp.release();
  });
}

bat_status bat_model_destroy(bat_model m) {
  return guarded([&] {
    if (!m) return;
    DeviceGuard dg(m->m.device);
    cudaDeviceSynchronize();
    delete m;
  });
}

// ------------------------------------------------------------------------------- pool
bat_status bat_kv_pool_create(const bat_pool_cfg* cfg, bat_pool* out) {
  return guarded([&] {
    BAT_REQUIRE(cfg && out, "null argument");
    const bat_pool_cfg& c = *cfg;
    BAT_REQUIRE(c.page_tokens == kPageTokens, "page_tokens must be 16");
    BAT_REQUIRE(c.num_pages >= 1 && c.num_pages < (int64_t(1) << 30), "num_pages");
    BAT_REQUIRE(c.dtype == BAT_BF16 || c.dtype == BAT_FP32, "dtype must be BAT_BF16 or BAT_FP32");
    BAT_REQUIRE(c.layers >= 1 && c.kv_heads >= 1, "layers / kv_heads");
    BAT_REQUIRE(c.head_dim == 16 || c.head_dim == 32 || c.head_dim == 64 || c.head_dim == 128, "head_dim");
    auto pp = std::make_unique<bat_pool_s>();
    Pool& p = pp->pool;
    p.cfg = c;
    if (p.cfg.world < 1) p.cfg.world = 1;
    p.device = c.device;
    p.index_only = c.device < 0;
    p.geo.init(c.layers, c.kv_heads, c.head_dim, c.dtype == BAT_FP32);
    p.zero_page = static_cast<int32_t>(c.num_pages);
    p.free_pages.reserve(c.num_pages);
    for (int64_t i = c.num_pages - 1; i >= 0; --i) p.free_pages.push_back(static_cast<int32_t>(i));
    p.peer_arena.assign(p.cfg.world, nullptr);
    p.peer_ipc.assign(p.cfg.world, 0);
    if (!p.index_only) {
      DeviceGuard dg(c.device);
      const size_t bytes = size_t(c.num_pages + 1) * p.geo.page_bytes;
      cudaError_t e = cudaMalloc(&p.arena, bytes);
      if (e != cudaSuccess) fail(BAT_E_OOM, std::string("pool arena: ") + cudaGetErrorString(e));
      CUDA_OK(cudaMemset(p.arena, 0, bytes));  // padded columns / empty slots stay zero
    }
    *out = pp.release();
  });
}

bat_status bat_kv_pool_destroy(bat_pool p) {
  return guarded([&] {
    if (!p) return;
    if (p->pool.live_plans > 0) fail(BAT_E_STATE, "destroy the pool's plans (bat_plan_destroy) first");
    if (p->pool.arena) {
      DeviceGuard dg(p->pool.device);
      cudaDeviceSynchronize();
      for (size_t r = 0; r < p->pool.peer_arena.size(); ++r)
        if (p->pool.peer_arena[r] && p->pool.peer_ipc[r]) cudaIpcCloseMemHandle(p->pool.peer_arena[r]);
      if (p->pool.fetch_host) cudaFreeHost(p->pool.fetch_host);
      if (p->pool.fetch_done) cudaEventDestroy(static_cast<cudaEvent_t>(p->pool.fetch_done));
      for (auto& f : p->pool.pending) cudaEventDestroy(f.ev);
      for (cudaEvent_t e : p->pool.spare_events) cudaEventDestroy(e);
      cudaFree(p->pool.arena);
    }
    delete p;
  });
}

int64_t bat_kv_page_bytes(bat_pool p) { return p ? p->pool.geo.page_bytes : 0; }

bat_status bat_kv_pool_stats(bat_pool p, int64_t* free_pages, int64_t* used_pages, int64_t* n_entities) {
  return guarded([&] {
    BAT_REQUIRE(p, "null pool");
    if (free_pages) *free_pages = p->pool.n_free();
    if (used_pages) *used_pages = p->pool.cfg.num_pages - p->pool.n_free();
    if (n_entities) *n_entities = int64_t(p->pool.index.size());
  });
}

bat_status bat_kv_reserve(bat_pool p, int32_t kind, int64_t id, int32_t n_tokens) {
  return guarded([&] {
    BAT_REQUIRE(p, "null pool");
    key_kind_check(kind);
    BAT_REQUIRE(n_tokens >= 1, "n_tokens >= 1");
    Pool& P = p->pool;
    EntityKey k{kind, id};
    BAT_REQUIRE(P.index.find(k) == P.index.end(), "entry already exists");
    Entity e;
    e.n_tokens = n_tokens;
    if (!P.alloc_pages(ceil_div(n_tokens, kPageTokens), e.pages)) {
      P.release_pages(e.pages);
      fail(BAT_E_POOLFULL, "pool full");
    }
    P.index.emplace(k, std::move(e));
  });
}

bat_status bat_kv_evict(bat_pool p, int32_t kind, int64_t id) {
  return guarded([&] {
    BAT_REQUIRE(p, "null pool");
    Pool& P = p->pool;
    auto it = P.index.find(EntityKey{kind, id});
    if (it == P.index.end()) fail(BAT_E_NOTFOUND, "entry not found");
    if (it->second.pins > 0) fail(BAT_E_STATE, "entry is referenced by a live plan (bat_plan_build)");
    P.release_pages(it->second.pages);
    P.index.erase(it);
  });
}

bat_status bat_kv_lookup(bat_pool p, int32_t kind, int64_t id, int32_t* n_tokens, int32_t* pages_out,
                         int32_t pages_cap, int32_t* n_pages) {
  return guarded([&] {
    BAT_REQUIRE(p, "null pool");
    const Entity* e = p->pool.find(kind, id);
    if (!e) fail(BAT_E_NOTFOUND, "entry not found");
    if (n_tokens) *n_tokens = e->n_tokens;
    if (n_pages) *n_pages = int32_t(e->pages.size());
    if (pages_out) {
      BAT_REQUIRE(pages_cap >= int32_t(e->pages.size()), "pages_cap too small");
      std::copy(e->pages.begin(), e->pages.end(), pages_out);
    }
  });
}

bat_status bat_kv_append(bat_pool p, int32_t kind, int64_t id, const void* k, const void* v,
                         int32_t n_tokens, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && k && v, "null argument");
    key_kind_check(kind);
    BAT_REQUIRE(n_tokens >= 1, "n_tokens >= 1");
    Pool& P = p->pool;
    if (P.index_only) fail(BAT_E_STATE, "index-only pool");
    DeviceGuard dg(P.device);
    EntityKey key{kind, id};
    auto it = P.index.find(key);
    const bool exists = it != P.index.end();
    const int32_t old_n = exists ? it->second.n_tokens : 0;
    const int64_t need = ceil_div(old_n + n_tokens, kPageTokens) - (exists ? int64_t(it->second.pages.size()) : 0);
    std::vector<int32_t> fresh;
    if (!P.alloc_pages(need, fresh)) {
      P.release_pages(fresh);
      fail(BAT_E_POOLFULL, "pool full");
    }
    std::vector<int32_t> pages = exists ? it->second.pages : std::vector<int32_t>();
    pages.insert(pages.end(), fresh.begin(), fresh.end());
    int32_t* dpages = nullptr;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&dpages), pages.size() * 4, st);
    if (e != cudaSuccess) {
      P.release_pages(fresh);
      fail(BAT_E_CUDA, std::string("cudaMallocAsync: ") + cudaGetErrorString(e));
    }
    CUDA_OK(cudaMemcpyAsync(dpages, pages.data(), pages.size() * 4, cudaMemcpyHostToDevice, st));
    if (P.geo.f32)
      launch_kv_scatter_f32(page_io(P), static_cast<const float*>(k), static_cast<const float*>(v), dpages, n_tokens,
                            old_n, n_tokens, st);
    else
      launch_kv_scatter(page_io(P), static_cast<const __nv_bfloat16*>(k), static_cast<const __nv_bfloat16*>(v),
                        dpages, n_tokens, old_n, n_tokens, st);
    CUDA_OK(cudaFreeAsync(dpages, st));
    CUDA_OK(cudaStreamSynchronize(st));  // the host page list above is a stack temporary
    if (exists) {
      it->second.pages = std::move(pages);
      it->second.n_tokens = old_n + n_tokens;
    } else {
      Entity en;
      en.n_tokens = n_tokens;
      en.pages = std::move(pages);
      P.index.emplace(key, std::move(en));
    }
  });
}

bat_status bat_kv_read(bat_pool p, int32_t kind, int64_t id, void* k_out, void* v_out, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && k_out && v_out, "null argument");
    Pool& P = p->pool;
    if (P.index_only) fail(BAT_E_STATE, "index-only pool");
    const Entity* e = P.find(kind, id);
    if (!e) fail(BAT_E_NOTFOUND, "entry not found");
    DeviceGuard dg(P.device);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    int32_t* dpages = nullptr;
    CUDA_OK(cudaMallocAsync(reinterpret_cast<void**>(&dpages), e->pages.size() * 4, st));
    CUDA_OK(cudaMemcpyAsync(dpages, e->pages.data(), e->pages.size() * 4, cudaMemcpyHostToDevice, st));
    if (P.geo.f32)
      launch_kv_gather_f32(page_io(P), static_cast<float*>(k_out), static_cast<float*>(v_out), dpages, e->n_tokens,
                           st);
    else
      launch_kv_gather(page_io(P), static_cast<__nv_bfloat16*>(k_out), static_cast<__nv_bfloat16*>(v_out),
                       dpages, e->n_tokens, st);
    CUDA_OK(cudaFreeAsync(dpages, st));
    CUDA_OK(cudaStreamSynchronize(st));
  });
}

bat_status bat_kv_prefill_entities(bat_pool p, bat_model mdl, int32_t kind, int32_t n_entities,
                                   const int64_t* ids, const int32_t* tok_off, const int32_t* tokens,
                                   int32_t pos0, int32_t ctx_kind, int64_t ctx_id, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && mdl && ids && tok_off && tokens, "null argument");
    key_kind_check(kind);
    BAT_REQUIRE(n_entities >= 1 && pos0 >= 0, "n_entities / pos0");
    Pool& P = p->pool;
    Model& m = mdl->m;
    check_compat(P, m);
    DeviceGuard dg(P.device);
    std::vector<EntityKey> made;
    std::vector<std::vector<int32_t>> pages(n_entities);
    try {
      for (int e = 0; e < n_entities; ++e) {
        const int32_t n = tok_off[e + 1] - tok_off[e];
        BAT_REQUIRE(n >= 1, "entity with no tokens");
        for (int32_t j = 0; j < n; ++j)
          BAT_REQUIRE(tokens[tok_off[e] + j] >= 0 && tokens[tok_off[e] + j] < m.cfg.vocab, "token id out of range");
        EntityKey key{kind, ids[e]};
        BAT_REQUIRE(P.index.find(key) == P.index.end(), "entry already exists");
        Entity en;
        en.n_tokens = n;
        if (!P.alloc_pages(ceil_div(n, kPageTokens), en.pages)) {
          P.release_pages(en.pages);
          fail(BAT_E_POOLFULL, "pool full");
        }
        pages[e] = en.pages;
        P.index.emplace(key, std::move(en));
        made.push_back(key);
      }
      std::vector<PlanRequest> reqs(n_entities);
      for (int e = 0; e < n_entities; ++e) {
        reqs[e].ent_tok = tokens + tok_off[e];
        reqs[e].ent_n = tok_off[e + 1] - tok_off[e];
        reqs[e].ent_pos0 = pos0;
        reqs[e].ctx_kind = ctx_kind;
        reqs[e].ctx_id = ctx_id;
        reqs[e].ent_pages = &pages[e];
      }
      Plan plan;
      build_plan(P, m.cfg.q_heads / m.cfg.kv_heads, m.cfg.kv_heads, reqs, plan, true, attn_grid_slots(m.dpad, m.num_sms),
                 nullptr, attn_qtiles_per_item());
      run_plan(P, m, plan, nullptr, static_cast<cudaStream_t>(stream));
      CUDA_OK(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
    } catch (...) {
      for (auto& k : made) {
        auto it = P.index.find(k);
        if (it != P.index.end()) {
          P.release_pages(it->second.pages);
          P.index.erase(it);
        }
      }
      throw;
    }
  });
}

// -------------------------------------------------------------------------- prefill
static std::vector<PlanRequest> wrap(const bat_query* q, int32_t B) {
  std::vector<PlanRequest> r(B);
  for (int b = 0; b < B; ++b) r[b].q = &q[b];
  return r;
}

static void validate_tokens(const bat_query& q, int vocab) {
  auto chk = [&](const int32_t* t, int n) {
    for (int i = 0; i < n; ++i) BAT_REQUIRE(t[i] >= 0 && t[i] < vocab, "token id out of range");
  };
  chk(q.user_tok, q.n_user);
  chk(q.instr_tok, q.n_instr);
  chk(q.header_tok, q.n_header);
  if (q.n_items > 0 && q.item_off) chk(q.item_tok, q.item_off[q.n_items]);
}

bat_status bat_bipartite_prefill(bat_pool p, bat_model mdl, const bat_query* queries, int32_t B,
                                 float* out_hidden, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && mdl && queries && out_hidden, "null argument");
    BAT_REQUIRE(B >= 1, "B >= 1");
    Pool& P = p->pool;
    Model& m = mdl->m;
    check_compat(P, m);
    for (int b = 0; b < B; ++b) validate_tokens(queries[b], m.cfg.vocab);
    DeviceGuard dg(P.device);
    Plan plan;
    build_plan(P, m.cfg.q_heads / m.cfg.kv_heads, m.cfg.kv_heads, wrap(queries, B), plan, true, attn_grid_slots(m.dpad, m.num_sms),
               nullptr, attn_qtiles_per_item());
    run_plan(P, m, plan, out_hidden, static_cast<cudaStream_t>(stream));
  });
}

bat_status bat_score_multi(bat_model mdl, const float* hidden, const int32_t* labels, const int32_t* n_items,
                           int32_t B, int32_t n_max, float* scores, int32_t k, int32_t* topk, float* logits,
                           bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(mdl && hidden && labels && n_items && scores, "null argument");
    BAT_REQUIRE(B >= 1 && n_max >= 1 && n_max <= 4096, "B >= 1, 1 <= n_max <= 4096");
    BAT_REQUIRE(k >= 0 && (k == 0 || topk) && k <= n_max, "k / topk");
    Model& m = mdl->m;
    DeviceGuard dg(m.device);
    launch_score_multi(hidden, m.f32 ? nullptr : m.lm_head, m.f32 ? static_cast<const float*>(m.w[BAT_W_LM_HEAD]) : nullptr,
                       labels, n_items, B, n_max, m.cfg.hidden, scores, k, topk, logits,
                       static_cast<cudaStream_t>(stream));
    CUDA_OK(cudaGetLastError());
  });
}

bat_status bat_score(bat_model mdl, const float* hidden, const int32_t* labels, const int32_t* n_items,
                     int32_t B, int32_t n_max, float* scores, int32_t k, int32_t* topk, float* logits,
                     bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(mdl && hidden && labels && n_items && scores, "null argument");
    BAT_REQUIRE(B >= 1 && n_max >= 1 && n_max <= 4096, "B >= 1, 1 <= n_max <= 4096");
    BAT_REQUIRE(k >= 0 && (k == 0 || topk), "k / topk");
    BAT_REQUIRE(k <= n_max, "k <= n_max");
    Model& m = mdl->m;
    DeviceGuard dg(m.device);
    if (m.f32)
      launch_score_f32w(hidden, static_cast<const float*>(m.w[BAT_W_LM_HEAD]), labels, n_items, B, n_max,
                        m.cfg.hidden, scores, k, topk, logits, static_cast<cudaStream_t>(stream));
    else
      launch_score(hidden, m.lm_head, labels, n_items, B, n_max, m.cfg.hidden, scores, k, topk, logits,
                   static_cast<cudaStream_t>(stream));
    CUDA_OK(cudaGetLastError());
  });
}

// ---------------------------------------------------------------------- plan inspection
bat_status bat_plan_create(bat_pool p, int32_t group, const bat_query* queries, int32_t B, bat_plan* out) {
  return guarded([&] {
    BAT_REQUIRE(p && queries && out && B >= 1, "null argument");
    auto pl = std::make_unique<bat_plan_s>();
    build_plan(p->pool, group, 1, wrap(queries, B), pl->plan, false);
    *out = pl.release();
  });
}

bat_status bat_plan_destroy(bat_plan plan) {
  return guarded([&] {
    if (!plan) return;
    if (plan->pool) {
      Pool& P = plan->pool->pool;
      for (const EntityKey& k : plan->pinned) {
        auto it = P.index.find(k);
        if (it != P.index.end() && it->second.pins > 0) --it->second.pins;
      }
      --P.live_plans;
    }
    delete plan;
  });
}

bat_status bat_plan_query_info(bat_plan plan, int32_t b, int64_t info[13]) {
  return guarded([&] {
    BAT_REQUIRE(plan && info && b >= 0 && b < int32_t(plan->plan.q.size()), "argument");
    const QueryPlan& q = plan->plan.q[b];
    const int64_t v[13] = {q.S, q.P, q.n_pages, q.n_prefix_pages, q.n_qtiles, q.n_ktiles, q.token_off,
                           q.scratch0, q.n_live_pairs, plan->plan.qt, q.qtile0, q.page_off, q.n_live_pairs_last};
    std::copy(v, v + 13, info);
  });
}

bat_status bat_plan_export(bat_plan plan, int32_t b, int32_t field, int32_t* out, int64_t cap, int64_t* count) {
  return guarded([&] {
    BAT_REQUIRE(plan && b >= 0 && b < int32_t(plan->plan.q.size()), "argument");
    const QueryPlan& q = plan->plan.q[b];
    std::vector<int32_t> tiles;
    const std::vector<int32_t>* src = nullptr;
    switch (field) {
      case BAT_PF_TOKENS: src = &q.tokens; break;
      case BAT_PF_POS: src = &q.pos; break;
      case BAT_PF_SEG: src = &q.seg; break;
      case BAT_PF_PAGES: src = &q.pages; break;
      case BAT_PF_VALID: src = &q.valid; break;
      case BAT_PF_KSEG: src = &q.kseg; break;
      case BAT_PF_KORD: src = &q.kord; break;
      case BAT_PF_TILES:
        tiles.assign(q.tiles.begin(), q.tiles.end());
        src = &tiles;
        break;
      case BAT_PF_DISC: src = &q.disc; break;
      default: BAT_REQUIRE(false, "unknown field");
    }
    if (count) *count = int64_t(src->size());
    if (out) {
      BAT_REQUIRE(cap >= int64_t(src->size()), "cap too small");
      std::copy(src->begin(), src->end(), out);
    }
  });
}

// Decode the DEVICE copy of a bat_plan_build plan the way the attention kernel reads it: the
// work list (per KV head: q-tile pair, listed k-tiles, their per-q-tile state and the page ids
// the loader copies) and the partial-tile visibility masks mask_kernel wrote on the device.
bat_status bat_plan_export_device(bat_plan plan, int32_t b, int32_t field, void* out, int64_t cap, int64_t* count) {
  return guarded([&] {
    BAT_REQUIRE(plan && plan->dev_img, "plan built with bat_plan_build");
    const Plan& pl = plan->plan;
    BAT_REQUIRE(b >= 0 && b < int32_t(pl.q.size()), "request index");
    BAT_REQUIRE(field >= BAT_PFD_VIS && field <= BAT_PFD_STAGE, "field");
    const PlanImage& im = pl.img;
    if (plan->dev_copy.empty()) {
      DeviceGuard dg(plan->device);
      plan->dev_copy.resize(size_t(im.total_ints));
      CUDA_OK(cudaMemcpy(plan->dev_copy.data(), plan->dev_img, size_t(im.total_ints) * 4, cudaMemcpyDeviceToHost));
    }
    const std::vector<int32_t>& I = plan->dev_copy;
    const QueryPlan& q = pl.q[b];
    if (field == BAT_PFD_STAGE) {
      // the fused QKV epilogue's per-row lookups (k_gemm.cu Epilogue::stage_row), decoded from the
      // device image: row -> request (row map) -> q_info -> q-tile, suffix page (spages), slot
      std::vector<int32_t> st(size_t(q.S) * 3);
      const int32_t tok_off = I[size_t(im.off_qinfo + int64_t(b) * 8)];
      for (int32_t t = 0; t < q.S; ++t) {
        const int64_t row = int64_t(tok_off) + t;
        const int32_t rb = I[size_t(im.off_rowreq + row)];
        if (rb != b) fail(BAT_E_STATE, "row map names another request");
        const int32_t* qi = &I[size_t(im.off_qinfo + int64_t(rb) * 8)];
        const int32_t tt = int32_t(row - qi[0]);
        st[size_t(t) * 3 + 0] = qi[2] + tt / pl.qt;
        st[size_t(t) * 3 + 1] = I[size_t(im.off_spages + int64_t(qi[6] + tt / kPageTokens) * 4 + 3)];
        st[size_t(t) * 3 + 2] = tt % kPageTokens;
      }
      if (count) *count = int64_t(st.size());
      if (out) {
        BAT_REQUIRE(cap >= int64_t(st.size()), "cap too small");
        std::copy(st.begin(), st.end(), static_cast<int32_t*>(out));
      }
      return;
    }
    const int64_t n_cols = int64_t(q.n_ktiles) * kKtile;
    const bool last = field == BAT_PFD_VIS_LAST;
    const int64_t off_work = last ? im.off_work_last : im.off_work;
    const int32_t n_work = last ? pl.n_work_last : pl.n_work;
    // per KV head: decoded visibility [S][n_cols] and the loaded page ids [n_ktiles * 8]
    std::vector<std::vector<uint8_t>> vis(pl.kv_heads, std::vector<uint8_t>(size_t(q.S) * n_cols, 0));
    std::vector<std::vector<int32_t>> kp(pl.kv_heads, std::vector<int32_t>(size_t(q.n_ktiles) * kKtilePages, BAT_PFD_NOT_LOADED));
    std::vector<std::vector<uint8_t>> seen(pl.kv_heads, std::vector<uint8_t>(size_t(q.n_qtiles) * q.n_ktiles, 0));
    for (int32_t w = 0; w < n_work; ++w) {
      const int32_t* e = &I[size_t(off_work + int64_t(w) * 8)];
      if (e[5] == 0 || e[0] != b) continue;  // LPT padding / another request
      const int kvh = e[1];
      if (kvh < 0 || kvh >= pl.kv_heads) fail(BAT_E_STATE, "work item KV head out of range");
      for (int x = 0; x < e[5]; ++x) {
        const int32_t ktl = I[size_t(e[4] + x)];
        const int32_t j = ktl & 0xFFFFFF;
        if (j < 0 || j >= q.n_ktiles) fail(BAT_E_STATE, "listed k-tile out of range");
        for (int l = 0; l < kKtilePages; ++l) {
          const int32_t pg = I[size_t(e[6] + int64_t(x) * kKtilePages + l)];
          int32_t& slot = kp[kvh][size_t(j) * kKtilePages + l];
          if (slot != BAT_PFD_NOT_LOADED && slot != pg) fail(BAT_E_STATE, "k-tile loaded with two page lists");
          slot = pg;
        }
        for (int h = 0; h < 2; ++h) {
          const int qi = h == 0 ? e[2] : e[3];
          if (qi < 0) continue;
          const int st = (ktl >> (24 + 2 * h)) & 3;
          if (st == 0) continue;
          if (qi >= q.n_qtiles) fail(BAT_E_STATE, "q-tile out of range");
          uint8_t& sn = seen[kvh][size_t(qi) * q.n_ktiles + j];
          if (sn) fail(BAT_E_STATE, "(q-tile, k-tile) pair listed twice");
          sn = 1;
          const int32_t mid = I[size_t(e[7] + 2 * x + h)];
          if (st == 2 && (mid < 0 || mid >= im.n_masks)) fail(BAT_E_STATE, "partial tile without a mask");
          for (int r = 0; r < pl.qt; ++r) {
            const int t = qi * pl.qt + r;
            if (t >= q.S) break;
            uint8_t* row = &vis[kvh][size_t(t) * n_cols + int64_t(j) * kKtile];
            if (st == 1) {
              std::fill(row, row + kKtile, uint8_t(1));
            } else {
              const int32_t* mw = &I[size_t(im.off_masks + (int64_t(mid) * (pl.qt + 1) + r) * 4)];
              for (int k = 0; k < kKtile; ++k) row[k] = uint8_t((uint32_t(mw[k >> 5]) >> (k & 31)) & 1u);
            }
          }
        }
      }
    }
    for (int h = 1; h < pl.kv_heads; ++h)
      if (vis[h] != vis[0] || kp[h] != kp[0]) fail(BAT_E_STATE, "KV heads see different tile lists");
    const bool pages = field == BAT_PFD_KPAGES;
    const int64_t n = pages ? int64_t(kp[0].size()) : int64_t(vis[0].size());
    if (count) *count = n;
    if (out) {
      BAT_REQUIRE(cap >= n, "cap too small");
      if (pages) std::copy(kp[0].begin(), kp[0].end(), static_cast<int32_t*>(out));
      else std::copy(vis[0].begin(), vis[0].end(), static_cast<uint8_t*>(out));
    }
  });
}

// ------------------------------------------------------------------ HRCS (Algorithm 1)
bat_status bat_hrcs_rmax(double B, double t, double alpha, int32_t c, double tau_i, int32_t N, double* out) {
  return guarded([&] {
    BAT_REQUIRE(out && c >= 1 && tau_i > 0 && N >= 1, "argument");
    const double T_max = alpha * t;               // line 5
    const double S_item = tau_i;                  // line 6
    *out = T_max * B * double(N - 1) / (double(c) * S_item * double(N));  // line 7
  });
}

bat_status bat_hrcs_place(const double* freq, int64_t n, double r_max, int32_t world, int32_t* owner,
                          double* r_out) {
  return guarded([&] {
    BAT_REQUIRE(freq && owner && n >= 1 && world >= 1, "argument");
    double total = 0.0;
    for (int64_t i = 0; i < n; ++i) total += freq[i];
    BAT_REQUIRE(total > 0.0, "frequencies sum to zero");
    std::vector<int64_t> order(n);
    std::iota(order.begin(), order.end(), 0);
    std::stable_sort(order.begin(), order.end(), [&](int64_t a, int64_t b) { return freq[a] > freq[b]; });
    double cdf = 0.0, r = 1.0;
    for (int64_t i = 1; i <= n; ++i) {  // lines 9-16
      cdf += freq[order[i - 1]] / total;
      if (cdf >= 1.0 - r_max) {
        r = double(i) / double(n);
        break;
      }
    }
    const int64_t n_rep = static_cast<int64_t>(std::llround(r * double(n)));
    for (int64_t i = 0; i < n; ++i) {  // lines 17-18
      owner[order[i]] = i < n_rep ? -1 : static_cast<int32_t>((i - n_rep) % world);
    }
    if (r_out) *r_out = r;
  });
}

// Background placement update (P:312 Step 3, footnote P:322; R21): replicated area =
// top round(r n_new) by the new frequencies; cold items keep their owner; demoted and new cold
// items go to the rank owning the fewest cold items (ties: lowest rank), hottest first.
bat_status bat_hrcs_refresh(const int32_t* owner_old, int64_t n_old, const double* freq_new, int64_t n_new,
                            double r, int32_t world, int32_t* owner_new) {
  return guarded([&] {
    BAT_REQUIRE(freq_new && owner_new && (owner_old || n_old == 0) && n_new >= n_old && n_new >= 1 && world >= 1,
                "argument");
    BAT_REQUIRE(r >= 0.0 && r <= 1.0, "r in [0, 1]");
    std::vector<int64_t> order(n_new);
    std::iota(order.begin(), order.end(), 0);
    std::stable_sort(order.begin(), order.end(), [&](int64_t a, int64_t b) { return freq_new[a] > freq_new[b]; });
    const int64_t n_rep = static_cast<int64_t>(std::floor(r * double(n_new) + 0.5));  // round half up
    std::vector<uint8_t> rep(n_new, 0);
    for (int64_t k = 0; k < n_rep; ++k) rep[order[k]] = 1;
    std::vector<int64_t> load(world, 0);
    for (int64_t i = 0; i < n_old; ++i) {
      BAT_REQUIRE(owner_old[i] >= -1 && owner_old[i] < world, "owner_old out of range");
      if (!rep[i] && owner_old[i] >= 0) {
        owner_new[i] = owner_old[i];
        ++load[owner_old[i]];
      }
    }
    for (int64_t i : order) {
      if (rep[i]) {
        owner_new[i] = -1;
      } else if (i >= n_old || owner_old[i] < 0) {
        const int32_t k = static_cast<int32_t>(std::min_element(load.begin(), load.end()) - load.begin());
        owner_new[i] = k;
        ++load[k];
      }
    }
  });
}

// ------------------------------------------------------------- NVLink page pull (a10)
bat_status bat_pool_ipc_handle(bat_pool p, void* out64) {
  return guarded([&] {
    BAT_REQUIRE(p && out64, "null argument");
    Pool& P = p->pool;
    if (P.index_only) fail(BAT_E_STATE, "index-only pool");
    DeviceGuard dg(P.device);
    cudaIpcMemHandle_t h;
    CUDA_OK(cudaIpcGetMemHandle(&h, P.arena));
    static_assert(sizeof(h) == 64, "ipc handle size");
    std::memcpy(out64, &h, 64);
  });
}

bat_status bat_pool_attach_peer(bat_pool p, int32_t peer, const void* h64) {
  return guarded([&] {
    BAT_REQUIRE(p && h64, "null argument");
    Pool& P = p->pool;
    BAT_REQUIRE(peer >= 0 && peer < P.cfg.world && peer != P.cfg.rank, "peer rank");
    if (P.index_only) fail(BAT_E_STATE, "index-only pool");
    DeviceGuard dg(P.device);
    cudaIpcMemHandle_t h;
    std::memcpy(&h, h64, 64);
    void* ptr = nullptr;
    CUDA_OK(cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess));
    P.peer_arena[peer] = static_cast<char*>(ptr);
    P.peer_ipc[peer] = 1;
  });
}

bat_status bat_kv_register_remote(bat_pool p, int32_t kind, int64_t id, int32_t owner, const int32_t* pages,
                                  int32_t n_pages, int32_t n_tokens) {
  return guarded([&] {
    BAT_REQUIRE(p && pages && n_pages >= 1 && n_tokens >= 1, "argument");
    key_kind_check(kind);
    Pool& P = p->pool;
    BAT_REQUIRE(owner >= 0 && owner < P.cfg.world, "owner rank");
    BAT_REQUIRE(n_pages == ceil_div(n_tokens, kPageTokens), "n_pages == ceil(n_tokens/16)");
    RemoteEntity r;
    r.owner = owner;
    r.n_tokens = n_tokens;
    r.pages.assign(pages, pages + n_pages);
    P.remote[EntityKey{kind, id}] = std::move(r);
  });
}

bat_status bat_kv_lookup_remote(bat_pool p, int32_t kind, int64_t id, int32_t* owner, int32_t* n_tokens,
                                int32_t* pages_out, int32_t pages_cap, int32_t* n_pages) {
  return guarded([&] {
    BAT_REQUIRE(p, "null pool");
    auto it = p->pool.remote.find(EntityKey{kind, id});
    if (it == p->pool.remote.end()) fail(BAT_E_NOTFOUND, "remote entry not registered");
    const RemoteEntity& r = it->second;
    if (owner) *owner = r.owner;
    if (n_tokens) *n_tokens = r.n_tokens;
    if (n_pages) *n_pages = int32_t(r.pages.size());
    if (pages_out) {
      BAT_REQUIRE(pages_cap >= int32_t(r.pages.size()), "pages_cap too small");
      std::copy(r.pages.begin(), r.pages.end(), pages_out);
    }
  });
}

// Page pulls from peer-mapped arenas on the copy engines: one cudaMemcpyAsync per run of
// consecutive pages (no SMs taken from the kernels running beside it; the host-side enqueue is
// asynchronous); BAT_FETCH_SM=1 selects the round-1 SM copy kernel instead.
static void issue_page_pulls(Pool& P, const std::vector<uint64_t>& src, const std::vector<int32_t>& dst,
                             cudaStream_t st) {
  if (src.empty()) return;
  static const bool use_sm = std::getenv("BAT_FETCH_SM") && std::getenv("BAT_FETCH_SM")[0] == '1';
  const int64_t pb = P.geo.page_bytes;
  if (use_sm) {
    const size_t bytes = src.size() * 8 + dst.size() * 4;
    if (!P.fetch_done) {
      cudaEvent_t e;
      CUDA_OK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
      P.fetch_done = e;
    }
    CUDA_OK(cudaEventSynchronize(static_cast<cudaEvent_t>(P.fetch_done)));
    if (P.fetch_host_cap < bytes) {
      if (P.fetch_host) cudaFreeHost(P.fetch_host);
      P.fetch_host_cap = bytes * 2;
      CUDA_OK(cudaMallocHost(&P.fetch_host, P.fetch_host_cap));
    }
    std::memcpy(P.fetch_host, src.data(), src.size() * 8);
    std::memcpy(static_cast<char*>(P.fetch_host) + src.size() * 8, dst.data(), dst.size() * 4);
    void* buf = nullptr;
    CUDA_OK(cudaMallocAsync(&buf, bytes, st));
    CUDA_OK(cudaMemcpyAsync(buf, P.fetch_host, bytes, cudaMemcpyHostToDevice, st));
    CUDA_OK(cudaEventRecord(static_cast<cudaEvent_t>(P.fetch_done), st));
    launch_page_copy(static_cast<const uint64_t*>(buf), reinterpret_cast<const int32_t*>(static_cast<char*>(buf) + src.size() * 8),
                     P.arena, pb, int(src.size()), st);
    CUDA_OK(cudaFreeAsync(buf, st));
    return;
  }
  std::vector<void*> d, s;
  std::vector<size_t> n;
  for (size_t k = 0; k < src.size(); ++k) {
    char* dp = P.arena + int64_t(dst[k]) * pb;
    char* sp = reinterpret_cast<char*>(src[k]);
    if (!d.empty() && static_cast<char*>(d.back()) + n.back() == dp && static_cast<char*>(s.back()) + n.back() == sp) {
      n.back() += size_t(pb);
    } else {
      d.push_back(dp);
      s.push_back(sp);
      n.push_back(size_t(pb));
    }
  }
  for (size_t k = 0; k < d.size(); ++k) CUDA_OK(cudaMemcpyAsync(d[k], s[k], n[k], cudaMemcpyDefault, st));
}

bat_status bat_kv_fetch(bat_pool p, int32_t kind, const int64_t* ids, int32_t n, int32_t* n_fetched,
                        bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && (ids || n == 0), "null argument");
    Pool& P = p->pool;
    if (P.index_only) fail(BAT_E_STATE, "index-only pool");
    DeviceGuard dg(P.device);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    std::vector<uint64_t> src;
    std::vector<int32_t> dst;
    std::vector<EntityKey> made, bumped;
    int32_t fetched = 0;
    try {
      for (int32_t i = 0; i < n; ++i) {
        EntityKey key{kind, ids[i]};
        auto loc = P.index.find(key);
        if (loc != P.index.end()) {  // replicated / owned, or already pulled: one more holder
          if (loc->second.fetched) {
            ++loc->second.refs;
            bumped.push_back(key);
          }
          continue;
        }
        auto it = P.remote.find(key);
        if (it == P.remote.end()) fail(BAT_E_NOTFOUND, "entry neither local nor registered remote");
        const RemoteEntity& r = it->second;
        char* peer = P.peer_arena[r.owner];
        if (!peer) fail(BAT_E_STATE, "peer arena of rank " + std::to_string(r.owner) + " not attached");
        Entity en;
        en.n_tokens = r.n_tokens;
        en.fetched = true;
        en.refs = 1;
        // pages still pending a stream-ordered release are taken behind a wait on `st`
        if (!P.alloc_pages_on(int64_t(r.pages.size()), en.pages, st)) {
          P.release_pages(en.pages);
          fail(BAT_E_POOLFULL, "pool full while fetching");
        }
        for (size_t k = 0; k < r.pages.size(); ++k) {
          src.push_back(reinterpret_cast<uint64_t>(peer + int64_t(r.pages[k]) * P.geo.page_bytes));
          dst.push_back(en.pages[k]);
        }
        P.index.emplace(key, std::move(en));
        made.push_back(key);
        ++fetched;
      }
      issue_page_pulls(P, src, dst, st);
      CUDA_OK(cudaGetLastError());
    } catch (...) {
      for (auto& k : made) {
        auto it = P.index.find(k);
        if (it != P.index.end()) {
          P.release_pages(it->second.pages);
          P.index.erase(it);
        }
      }
      for (auto& k : bumped) {
        auto it = P.index.find(k);
        if (it != P.index.end()) --it->second.refs;
      }
      throw;
    }
    if (n_fetched) *n_fetched = fetched;
  });
}

bat_status bat_kv_replicate(bat_pool p, int32_t kind, const int64_t* ids, int32_t n, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && (ids || n == 0), "null argument");
    Pool& P = p->pool;
    for (int32_t i = 0; i < n; ++i) {
      auto it = P.index.find(EntityKey{kind, ids[i]});
      if (it != P.index.end() && it->second.fetched)
        fail(BAT_E_STATE, "entry is a pulled (reference-counted) copy; release it first");
    }
    int32_t nf = 0;
    const bat_status st = bat_kv_fetch(p, kind, ids, n, &nf, stream);
    if (st != BAT_OK) fail(st, last_error());
    for (int32_t i = 0; i < n; ++i) {  // the new copies become regular local (replicated) entries
      auto it = P.index.find(EntityKey{kind, ids[i]});
      if (it != P.index.end() && it->second.fetched) {
        it->second.fetched = false;
        it->second.refs = 0;
      }
    }
  });
}

bat_status bat_kv_release(bat_pool p, int32_t kind, const int64_t* ids, int32_t n, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && (ids || n == 0), "null argument");
    Pool& P = p->pool;
    if (P.index_only) fail(BAT_E_STATE, "index-only pool");
    DeviceGuard dg(P.device);
    // validate first (all-or-nothing)
    std::unordered_map<EntityKey, int32_t, EntityKeyHash> drops;
    for (int32_t i = 0; i < n; ++i) {
      EntityKey key{kind, ids[i]};
      auto it = P.index.find(key);
      if (it == P.index.end()) {
        if (P.remote.count(key)) fail(BAT_E_STATE, "remote entry released but not fetched");
        fail(BAT_E_NOTFOUND, "entry not found");
      }
      if (!it->second.fetched) continue;  // replicated / owned: not a pulled copy
      const int32_t d = ++drops[key];
      if (d > it->second.refs) fail(BAT_E_STATE, "more releases than fetches");
      if (d == it->second.refs && it->second.pins > 0) fail(BAT_E_STATE, "entry is referenced by a live plan");
    }
    std::vector<int32_t> freed;
    for (auto& kv : drops) {
      auto it = P.index.find(kv.first);
      it->second.refs -= kv.second;
      if (it->second.refs == 0) {
        freed.insert(freed.end(), it->second.pages.begin(), it->second.pages.end());
        P.index.erase(it);
      }
    }
    if (freed.empty()) return;
    cudaEvent_t ev;
    if (!P.spare_events.empty()) {
      ev = P.spare_events.back();
      P.spare_events.pop_back();
    } else {
      CUDA_OK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    }
    CUDA_OK(cudaEventRecord(ev, static_cast<cudaStream_t>(stream)));
    P.pending.push_back(Pool::PendingFree{ev, std::move(freed)});
  });
}

bat_status bat_kv_staging_reserve(bat_pool p, int32_t n_slots, int64_t pages_per_slot) {
  return guarded([&] {
    BAT_REQUIRE(p && n_slots >= 1 && n_slots <= 8 && pages_per_slot >= 1, "argument");
    Pool& P = p->pool;
    BAT_REQUIRE(P.staging.empty(), "staging already reserved");
    std::vector<std::vector<int32_t>> slots(n_slots);
    for (auto& sl : slots)
      if (!P.alloc_pages(pages_per_slot, sl)) {
        for (auto& x : slots) P.release_pages(x);
        fail(BAT_E_POOLFULL, "pool too small for the staging slots");
      }
    P.staging = std::move(slots);
  });
}

// ------------------------------------------------------------------------ test-only
bat_status bat_debug_gemm(int32_t epi, int32_t M, int32_t N, int32_t K, const void* A, const void* Bw,
                          int64_t b_rows, void* out, int32_t ldo, const void* bias, int32_t up_row0,
                          int32_t device, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(A && Bw && out && M >= 1 && N >= 1 && K >= 8 && K % 8 == 0, "argument");
    BAT_REQUIRE(epi >= 0 && epi <= 3, "epi");
    DeviceGuard dg(device);
    int sms = 148;
    CUDA_OK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
    const CUtensorMap ta = make_tmap(A, M, K, K, 128);
    const CUtensorMap tb = make_tmap(Bw, b_rows, K, K, 128);  // B is loaded in 128-row boxes
    const CUtensorMap tc = make_tmap(out, M, N, ldo, 32, epi == EPI_RESID_F32);
    GemmParams gp{M, N, K, out, ldo, static_cast<const __nv_bfloat16*>(bias), up_row0};
    launch_gemm(epi, ta, tb, tc, gp, sms, static_cast<cudaStream_t>(stream));
    CUDA_OK(cudaGetLastError());
  });
}

bat_status bat_debug_attention_layer(bat_pool p, bat_model mdl, const bat_query* queries, int32_t B,
                                     int32_t layer, const void* qkv, void* out_o, int32_t rope_enabled,
                                     bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && mdl && queries && qkv && out_o && B >= 1, "argument");
    Pool& P = p->pool;
    Model& m = mdl->m;
    check_compat(P, m);
    BAT_REQUIRE(layer >= 0 && layer < m.cfg.layers, "layer");
    if (m.f32) fail(BAT_E_UNSUPPORTED, "bat_debug_attention_layer tests the bf16 tensor-core kernel");
    DeviceGuard dg(P.device);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    Plan plan;
    build_plan(P, m.cfg.q_heads / m.cfg.kv_heads, m.cfg.kv_heads, wrap(queries, B), plan, true, attn_grid_slots(m.dpad, m.num_sms),
               nullptr, attn_qtiles_per_item());
    const int32_t* I = prepare(P, m, plan, st);
    StageParams sp = stage_params(P, m, plan, I);
    sp.qkv = static_cast<const __nv_bfloat16*>(qkv);
    sp.rope_enabled = rope_enabled;
    sp.pool_layer_off = int64_t(layer) * P.geo.layer_bytes;
    launch_stage(sp, st);
    AttnParams ap = attn_params(P, m, plan, I);
    ap.pool_layer_off = int64_t(layer) * P.geo.layer_bytes;
    ap.out = static_cast<__nv_bfloat16*>(out_o);
    const char* tl = std::getenv("BAT_ATTN_TIMELINE");  // debug: clock64 timeline of CTA 0
    long long* dbg = nullptr;
    if (tl) {
      CUDA_OK(cudaMalloc(&dbg, 24 * 64 * sizeof(long long)));
      CUDA_OK(cudaMemsetAsync(dbg, 0, 24 * 64 * sizeof(long long), st));
      ap.dbg = dbg;
    }
    const char* ti = std::getenv("BAT_ATTN_ITEMS");  // debug: per-work-item clock64 records
    long long* dbi = nullptr;
    if (ti) {
      CUDA_OK(cudaMalloc(&dbi, size_t(ap.n_work) * 6 * sizeof(long long)));
      CUDA_OK(cudaMemsetAsync(dbi, 0, size_t(ap.n_work) * 6 * sizeof(long long), st));
      ap.dbg_items = dbi;
    }
    run_attention(P, m, plan, ap, false, st);
    CUDA_OK(cudaGetLastError());
    CUDA_OK(cudaStreamSynchronize(st));
    if (dbg) {
      std::vector<long long> h(24 * 64);
      CUDA_OK(cudaMemcpy(h.data(), dbg, h.size() * sizeof(long long), cudaMemcpyDeviceToHost));
      FILE* f = std::fopen(tl, "w");
      if (f) {
        for (int e = 0; e < 24; ++e) {
          for (int x = 0; x < 64; ++x) std::fprintf(f, "%lld ", h[e * 64 + x]);
          std::fprintf(f, "\n");
        }
        std::fclose(f);
      }
      cudaFree(dbg);
    }
    if (dbi) {
      std::vector<long long> h(size_t(ap.n_work) * 6);
      CUDA_OK(cudaMemcpy(h.data(), dbi, h.size() * sizeof(long long), cudaMemcpyDeviceToHost));
      FILE* f = std::fopen(ti, "w");
      if (f) {
        for (int w = 0; w < ap.n_work; ++w) {
          for (int e = 0; e < 6; ++e) std::fprintf(f, "%lld ", h[size_t(w) * 6 + e]);
          std::fprintf(f, "\n");
        }
        std::fclose(f);
      }
      cudaFree(dbi);
    }
  });
}


// ------------------------------------------------------------------ planned execution
static void plan_build_impl(bat_pool p, bat_model mdl, const bat_query* queries, int32_t B, int32_t slot,
                            bat_stream_t stream, bat_plan* out) {
  BAT_REQUIRE(p && mdl && queries && out && B >= 1, "null argument");
  Pool& P = p->pool;
  Model& m = mdl->m;
  check_compat(P, m);
  for (int b = 0; b < B; ++b) validate_tokens(queries[b], m.cfg.vocab);
  DeviceGuard dg(P.device);
  auto pl = std::make_unique<bat_plan_s>();
  StagingCtx stg;
  if (slot >= 0) {
    BAT_REQUIRE(slot < int32_t(P.staging.size()), "staging slot (bat_kv_staging_reserve first)");
    stg.slot_pages = &P.staging[slot];
  }
  build_plan(P, m.cfg.q_heads / m.cfg.kv_heads, m.cfg.kv_heads, wrap(queries, B), pl->plan, true,
             attn_grid_slots(m.dpad, m.num_sms), slot >= 0 ? &stg : nullptr, attn_qtiles_per_item());
  pl->pull_src = std::move(stg.src);
  pl->pull_dst = std::move(stg.dst);
  pl->slot = slot;
  const size_t bytes = pl->plan.img.buf.size() * 4;
  CUDA_OK(cudaMalloc(&pl->dev_img, size_t(pl->plan.img.total_ints) * 4));
  CUDA_OK(cudaMemcpyAsync(pl->dev_img, pl->plan.img.buf.data(), bytes, cudaMemcpyHostToDevice,
                          static_cast<cudaStream_t>(stream)));
  build_masks(pl->plan, static_cast<int32_t*>(pl->dev_img), static_cast<cudaStream_t>(stream));
  CUDA_OK(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
  pl->device = P.device;
  // the device image bakes in page ids: pin every referenced entry until bat_plan_destroy
  for (const QueryPlan& q : pl->plan.q)
    for (const EntityKey& k : q.refs) {
      auto it = P.index.find(k);
      if (it != P.index.end()) {
        ++it->second.pins;
        pl->pinned.push_back(k);
      }
    }
  pl->pool = p;
  ++P.live_plans;
  *out = pl.release();
}

bat_status bat_plan_build(bat_pool p, bat_model mdl, const bat_query* queries, int32_t B, bat_stream_t stream,
                          bat_plan* out) {
  return guarded([&] { plan_build_impl(p, mdl, queries, B, -1, stream, out); });
}

bat_status bat_plan_build_staged(bat_pool p, bat_model mdl, const bat_query* queries, int32_t B, int32_t slot,
                                 bat_stream_t stream, bat_plan* out) {
  return guarded([&] { plan_build_impl(p, mdl, queries, B, slot, stream, out); });
}

bat_status bat_plan_work_info(bat_plan plan, int64_t out[6]) {
  return guarded([&] {
    BAT_REQUIRE(plan && out, "null argument");
    const Plan& pl = plan->plan;
    const int64_t v[6] = {pl.n_work, pl.n_work_last, pl.img.n_sgrp, pl.img.n_slots, pl.img.n_sgrp_last,
                          pl.img.n_slots_last};
    std::copy(v, v + 6, out);
  });
}

bat_status bat_plan_bytes(bat_plan plan, int64_t* host_bytes, int64_t* device_bytes) {
  return guarded([&] {
    BAT_REQUIRE(plan, "null plan");
    if (host_bytes) *host_bytes = int64_t(plan->plan.img.buf.size()) * 4;
    if (device_bytes) *device_bytes = plan->plan.img.total_ints * 4;
  });
}

bat_status bat_plan_fetch(bat_pool p, bat_plan plan, int64_t* n_pages, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && plan, "null argument");
    if (plan->pool != p) fail(BAT_E_STATE, "plan was built for another pool");
    Pool& P = p->pool;
    DeviceGuard dg(P.device);
    issue_page_pulls(P, plan->pull_src, plan->pull_dst, static_cast<cudaStream_t>(stream));
    CUDA_OK(cudaGetLastError());
    if (n_pages) *n_pages = int64_t(plan->pull_dst.size());
  });
}

bat_status bat_prefill_plan(bat_pool p, bat_model mdl, bat_plan plan, float* out_hidden, bat_stream_t stream) {
  return guarded([&] {
    BAT_REQUIRE(p && mdl && plan && out_hidden, "null argument");
    BAT_REQUIRE(plan->dev_img, "plan was not built with bat_plan_build");
    Pool& P = p->pool;
    Model& m = mdl->m;
    check_compat(P, m);
    BAT_REQUIRE(!plan->plan.entity_mode && plan->plan.kv_heads == m.cfg.kv_heads, "plan / model mismatch");
    if (plan->pool != p) fail(BAT_E_STATE, "plan was built for another pool");
    DeviceGuard dg(P.device);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const int32_t* img = static_cast<const int32_t*>(plan->dev_img);
    // CUDA graph replay of the ~12 launches per layer (launch-bound at small batches); not on the
    // legacy default stream (not capturable) nor while kernel profiling records events
    const char* gv = std::getenv("BAT_GRAPH");  // opt-in: measured neutral (batch-1 5.038 vs 5.038 ms)
    const bool use_graph = gv && std::atoi(gv) != 0;
    if (!use_graph || st == nullptr || m.prof.on) {
      run_plan(P, m, plan->plan, out_hidden, st, img);
      return;
    }
    const uint64_t gen = g_buf_gen.load();
    if (plan->gexec && plan->graph_gen == gen && plan->graph_out == out_hidden && plan->graph_model == &m) {
      CUDA_OK(cudaGraphLaunch(plan->gexec, st));
      count_launch(int(plan->graph_launches));
      return;
    }
    if (plan->gexec) {
      CUDA_OK(cudaGraphExecDestroy(plan->gexec));
      plan->gexec = nullptr;
    }
    if (!plan->warm || plan->warm_gen != gen) {  // size the workspace first: nothing may allocate during capture
      run_plan(P, m, plan->plan, out_hidden, st, img);
      plan->warm = true;
      plan->warm_gen = g_buf_gen.load();
      return;
    }
    const int64_t n0 = launch_count();
    CUDA_OK(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
    cudaGraph_t g = nullptr;
    try {
      run_plan(P, m, plan->plan, out_hidden, st, img);
    } catch (...) {
      cudaStreamEndCapture(st, &g);
      if (g) cudaGraphDestroy(g);
      throw;
    }
    CUDA_OK(cudaStreamEndCapture(st, &g));
    const cudaError_t ie = cudaGraphInstantiate(&plan->gexec, g, 0);
    cudaGraphDestroy(g);
    CUDA_OK(ie);
    plan->graph_gen = g_buf_gen.load();
    if (plan->graph_gen != gen) fail(BAT_E_CUDA, "workspace reallocated during graph capture");
    plan->graph_out = out_hidden;
    plan->graph_model = &m;
    plan->graph_launches = launch_count() - n0;
    CUDA_OK(cudaGraphLaunch(plan->gexec, st));
  });
}

// ----------------------------------------------------------------------- profiling
bat_status bat_profile_enable(bat_model mdl, int32_t on) {
  return guarded([&] {
    BAT_REQUIRE(mdl, "null model");
    mdl->m.prof.on = on != 0;
  });
}

bat_status bat_profile_read(bat_model mdl, int32_t cls, double* total_ms, int64_t* launches, double* flops,
                            double* bytes) {
  return guarded([&] {
    BAT_REQUIRE(mdl && cls >= 0 && cls < BAT_K_N, "argument");
    DeviceGuard dg(mdl->m.device);
    Profiler& pf = mdl->m.prof;
    pf.collect();
    if (total_ms) *total_ms = pf.ms[cls];
    if (launches) *launches = pf.n[cls];
    if (flops) *flops = pf.flops[cls];
    if (bytes) *bytes = pf.bytes[cls];
  });
}

bat_status bat_profile_reset(bat_model mdl) {
  return guarded([&] {
    BAT_REQUIRE(mdl, "null model");
    DeviceGuard dg(mdl->m.device);
    mdl->m.prof.reset();
  });
}

bat_status bat_debug_attach_peer_pool(bat_pool p, int32_t peer, bat_pool other) {
  return guarded([&] {
    BAT_REQUIRE(p && other, "null argument");
    Pool& P = p->pool;
    BAT_REQUIRE(peer >= 0 && peer < P.cfg.world && peer != P.cfg.rank, "peer rank");
    BAT_REQUIRE(other->pool.geo.page_bytes == P.geo.page_bytes, "page geometry differs");
    P.peer_arena[peer] = other->pool.arena;
  });
}
}  // extern "C"
