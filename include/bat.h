/*
 * bat.h — C ABI of the B200-native Bipartite Attention (BAT) prefill library (libbat.so).
 *
 * `P:n` cites /root/reference/PAPER.md line n (BAT: Efficient Generative Recommender Serving
 * with Bipartite Attention, ASPLOS '26).
 *
 * What the library computes: a ranking request is a user
 * profile U, N candidate items I_1..I_N and instruction tokens Instr.  Per request one
 * side is a reused prefix KV cache: the user (User-as-prefix, UP, order [U, I_1..I_N, Instr],
 * P:249) or every item independently (Item-as-prefix, IP, order [I_1..I_N, U, Instr]).
 * The other tokens (the suffix) run through L transformer layers; at every layer they attend
 * to [prefix KV ; suffix KV] under the bipartite mask — different items never see
 * each other, all items start at the same position id (|U| in UP, 0 or after header tokens in
 * IP), everything else causal (Fig. 1).  The discriminant (last) token's hidden
 * state is projected on the N item-identifier logits, softmaxed and ranked.
 *
 * Conventions (every call):
 *   - Return BAT_OK (0) or a negative bat_status; bat_last_error() returns a thread-local
 *     message for the last failure.  No C++ exception crosses the ABI.
 *   - "device" pointers are CUDA device pointers on the object's device; "host" pointers are
 *     ordinary host memory, read during the call and not retained.
 *   - Device work is enqueued on `stream` (a cudaStream_t; NULL = the legacy default stream)
 *     and is asynchronous unless stated; host arrays are copied before the call returns.
 *   - Objects are not thread-safe: calls on one pool/model must be externally serialised.
 *   - Layouts are row-major with the last index contiguous.
 */
#ifndef BAT_H_
#define BAT_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define BAT_API __attribute__((visibility("default")))
#else
#define BAT_API
#endif

typedef void* bat_stream_t; /* cudaStream_t */

typedef enum {
  BAT_OK = 0,
  BAT_E_INVAL = -1,       /* bad argument / shape / unsupported value */
  BAT_E_OOM = -2,         /* device or host allocation failed */
  BAT_E_CUDA = -3,        /* a CUDA runtime/driver call failed (message has the CUDA error) */
  BAT_E_NOTFOUND = -4,    /* a required prefix entity is not in the pool */
  BAT_E_POOLFULL = -5,    /* not enough free pages; the pool is left unchanged */
  BAT_E_UNSUPPORTED = -6, /* valid request this build does not implement */
  BAT_E_STATE = -7        /* object in the wrong state (e.g. index-only pool used for compute) */
} bat_status;

/* BAT_BF16: the product path (tcgen05 tensor-core GEMMs and attention, bf16 operands, fp32
 * accumulation and residual).  BAT_FP32: SIMT correctness mode — the same plan (positions,
 * segments, page tables, key metadata) through plain fp32 CUDA-core kernels, weights / KV pages /
 * activations in fp32; matches the fp64 oracle within 1e-5 abs/rel (north_star).  Not a fast
 * path.  A pool and a model used together must have the same dtype. */
typedef enum { BAT_BF16 = 0, BAT_FP32 = 1 } bat_dtype;

/* Cache entries at user / item granularity; HEADER = the optional IP notation
 * tokens ("Candidate items:"), cached once as its own entry. */
typedef enum { BAT_ENT_USER = 0, BAT_ENT_ITEM = 1, BAT_ENT_HEADER = 2 } bat_entity;

/* Prefix side of a request. */
typedef enum { BAT_ORDER_UP = 0, BAT_ORDER_IP = 1 } bat_order;

BAT_API const char* bat_last_error(void);
BAT_API const char* bat_version(void);
/* Number of device kernels this library launched since load (all devices). */
BAT_API int64_t bat_kernel_launch_count(void);

/* ------------------------------------------------------------------------------------------
 * Model (Qwen2-shaped GR ranking model, Table 2)
 * ---------------------------------------------------------------------------------------- */
typedef struct {
  int32_t layers, hidden, q_heads, kv_heads, head_dim, ffn, vocab;
  float rope_theta; /* rotate-half RoPE base */
  float rms_eps;    /* RMSNorm epsilon */
  int32_t dtype;    /* bat_dtype of weights / activations / KV (BAT_BF16 is the product path) */
} bat_model_cfg;

/* Index of each weight in the pointer array passed to bat_model_create (3 + 7*layers device
 * pointers, all of dtype cfg.dtype):
 *   [0] embed      [vocab][hidden]          E, h^(0)_t = E[x_t]
 *   [1] lm_head    [vocab][hidden]          W_out, z = W_out h_T; may alias embed (tied)
 *   [2] final_norm [hidden]                 RMSNorm gain applied to h_T
 *   per layer l, at 3 + 7*l + j:
 *   j=0 ln1  [hidden]                       pre-attention RMSNorm gain
 *   j=1 wqkv [(q_heads+2*kv_heads)*head_dim][hidden]   rows: all q heads, then k, then v
 *   j=2 bqkv [(q_heads+2*kv_heads)*head_dim]          q/k/v bias
 *   j=3 wo   [hidden][q_heads*head_dim]
 *   j=4 ln2  [hidden]                       pre-MLP RMSNorm gain
 *   j=5 wgu  [2*ffn][hidden]                rows: gate (ffn), then up (ffn); SwiGLU
 *   j=6 wd   [hidden][ffn]
 * The model BORROWS these pointers: the caller keeps them alive and unchanged until
 * bat_model_destroy.  Supported: head_dim in {16, 32, 64, 128}, q_heads % kv_heads == 0,
 * q_heads/kv_heads <= 128, hidden % 64 == 0, ffn % 128 == 0, BAT_BF16 or BAT_FP32 (weights
 * then fp32). */
enum { BAT_W_EMBED = 0, BAT_W_LM_HEAD = 1, BAT_W_FINAL_NORM = 2, BAT_W_N_GLOBAL = 3 };
enum { BAT_WL_LN1 = 0, BAT_WL_WQKV = 1, BAT_WL_BQKV = 2, BAT_WL_WO = 3, BAT_WL_LN2 = 4,
       BAT_WL_WGU = 5, BAT_WL_WD = 6, BAT_WL_N = 7 };

typedef struct bat_model_s* bat_model;
BAT_API bat_status bat_model_create(const bat_model_cfg* cfg, const void* const* weights,
                            int32_t n_weights, int32_t device, bat_model* out);
BAT_API bat_status bat_model_destroy(bat_model m);

/* ------------------------------------------------------------------------------------------
 * Disaggregated paged KV pool: one page arena per GPU; entries at user/item
 * granularity, each entry a list of fixed-size pages of page_tokens (16) tokens, each page
 * holding all layers of its tokens.  Byte size per token = 2*kv_heads*head_dim*layers*2
 * (Table 2: 28672 B for Qwen2-1.5B).  The in-HBM page layout is the tensor-core
 * operand layout and is private; read entries back with bat_kv_read.
 * ---------------------------------------------------------------------------------------- */
typedef struct {
  int32_t device;      /* CUDA device ordinal; -1 = index-only pool (no arena; planning tests) */
  int32_t page_tokens; /* must be 16 */
  int64_t num_pages;   /* arena capacity in pages */
  int32_t dtype;       /* bat_dtype; must match the model's */
  int32_t layers, kv_heads, head_dim;
  int32_t rank, world; /* data-parallel rank / size for the HRCS item placement */
} bat_pool_cfg;

typedef struct bat_pool_s* bat_pool;
BAT_API bat_status bat_kv_pool_create(const bat_pool_cfg* cfg, bat_pool* out); /* OWNS its arena */
BAT_API bat_status bat_kv_pool_destroy(bat_pool p);
/* bytes of one page (all layers) */
BAT_API int64_t bat_kv_page_bytes(bat_pool p);
BAT_API bat_status bat_kv_pool_stats(bat_pool p, int64_t* free_pages, int64_t* used_pages,
                             int64_t* n_entities);

/* Append n_tokens of prefix KV to entry (kind, id), creating it if absent (the background
 * cache write of P:209/P:294 and the offline item precompute of P:312).  k, v: device
 * [layers][n_tokens][kv_heads][head_dim] in the pool dtype, post-RoPE keys.  All-or-nothing:
 * BAT_E_POOLFULL leaves the pool unchanged. */
BAT_API bat_status bat_kv_append(bat_pool p, int32_t kind, int64_t id, const void* k, const void* v,
                         int32_t n_tokens, bat_stream_t stream);
/* Reserve pages for a new entry without writing data (index-only pools, and the entity
 * prefill below).  BAT_E_INVAL if the entry exists. */
BAT_API bat_status bat_kv_reserve(bat_pool p, int32_t kind, int64_t id, int32_t n_tokens);
/* Drop an entry and free its pages (BAT_E_STATE if a live bat_plan_build plan references it).
 * The caller must not evict an entry that queued device work still reads. */
BAT_API bat_status bat_kv_evict(bat_pool p, int32_t kind, int64_t id);
/* Host query of an entry: its token count and page ids (pages_out may be NULL). */
BAT_API bat_status bat_kv_lookup(bat_pool p, int32_t kind, int64_t id, int32_t* n_tokens,
                         int32_t* pages_out, int32_t pages_cap, int32_t* n_pages);
/* Copy an entry back out in the plain layout of bat_kv_append (device k_out, v_out). */
BAT_API bat_status bat_kv_read(bat_pool p, int32_t kind, int64_t id, void* k_out, void* v_out,
                       bat_stream_t stream);

/* Prefix-miss path: compute the KV of n_entities new entries with the
 * model — each entry's tokens run alone through the L layers, causally, at positions
 * pos0, pos0+1, ... (UP user: pos0 = 0; IP item: pos0 = header length), attending first to
 * the optional context entry (ctx_kind, ctx_id; pass ctx_kind = -1 for none; the IP header)
 * — and store them as entries (kind, ids[e]).  tokens: host, entry e's tokens are
 * tokens[tok_off[e] .. tok_off[e+1]).  The entries must not exist. */
BAT_API bat_status bat_kv_prefill_entities(bat_pool p, bat_model m, int32_t kind, int32_t n_entities,
                                   const int64_t* ids, const int32_t* tok_off,
                                   const int32_t* tokens, int32_t pos0, int32_t ctx_kind,
                                   int64_t ctx_id, bat_stream_t stream);

/* ------------------------------------------------------------------------------------------
 * Bipartite prefill (the hot path)
 * ---------------------------------------------------------------------------------------- */
typedef struct {
  int32_t order;      /* bat_order: prefix side chosen for this request */
  int32_t use_cache;  /* 1: prefix served from the pool; 0: recompute every token (RE) */
  int64_t user_id;
  const int32_t* user_tok; int32_t n_user;          /* host */
  int32_t n_items;                                  /* N >= 1 */
  const int64_t* item_id;                           /* host [N] */
  const int32_t* item_off;                          /* host [N+1]: item i = item_tok[off[i]..off[i+1]) */
  const int32_t* item_tok;                          /* host */
  const int32_t* instr_tok; int32_t n_instr;        /* host; n_instr >= 1 (discriminant) */
  int64_t header_id;                                /* IP notation tokens, may be 0-length */
  const int32_t* header_tok; int32_t n_header;      /* host */
  int32_t multi_disc; /* 1: one discriminant token per item — the last token of every
                         item, whose hidden state has attended to U and its own item; requires
                         order UP (the items must be computed) and the same value for the whole
                         batch.  0: the last sequence token is the discriminant. */
  int32_t pic_tail;   /* IP only: selective recompute (PIC, P:265 / P:476; R25).  k > 0:
                         the last min(k, |I_i|) tokens of every item are recomputed after U (they
                         attend to the header, their item's cached head, U and their earlier tail
                         tokens), at positions h + m + |U| + j; the instruction tokens then start
                         at h + m + |U| + m.  Each item serves only its head from the cache (the
                         first |I_i| - k rows of the same entry).  0 = plain IP. */
} bat_query;

/* Run the L layers for B requests (data-parallel batch): every request's suffix
 * tokens are computed and attend to its cached prefix entries (BAT_E_NOTFOUND if one is
 * missing and use_cache = 1).  Writes the final-RMSNormed discriminant hidden state of every
 * request to out_hidden (device fp32 [B][hidden]).  Positions follow P:257 with the readings
 * of DESIGN.md §2 (tokens after the item set continue from the longest item).  With
 * multi_disc out_hidden is device fp32 [B][n_max][hidden], n_max = the batch's largest
 * n_items: row (b, i) is the final-RMSNormed hidden state of item i's last token (rows
 * i >= n_items[b] repeat the request's last token); the last layer then runs on every row. */
BAT_API bat_status bat_bipartite_prefill(bat_pool p, bat_model m, const bat_query* queries, int32_t B,
                                 float* out_hidden, bat_stream_t stream);

/* z[b][i] = W_out[labels[b][i]] . hidden[b] (the logit of item i's identifier token),
 * s[b][i] = softmax_i z[b][i] over i < n_items[b]; topk[b][0..k) = candidate indices by
 * descending s (ties -> lower index).
 * hidden: device fp32 [B][hidden]; labels: device int32 [B][n_max] (identifier token v_i,
 * P:177); n_items: device int32 [B] (values are clamped to [0, n_max]); scores: device fp32
 * [B][n_max] (entries >= n_items[b] set to 0); topk: device int32 [B][k] or NULL when k = 0
 * (ranks >= n_items[b] are -1); logits: device fp32 [B][n_max] receiving z (entries >= n_items[b]
 * set to 0) or NULL.  Requires 1 <= n_max <= 4096 and k <= n_max. */
BAT_API bat_status bat_score(bat_model m, const float* hidden, const int32_t* labels,
                     const int32_t* n_items, int32_t B, int32_t n_max, float* scores,
                     int32_t k, int32_t* topk, float* logits, bat_stream_t stream);
/* Multi-discriminant scoring: z[b][i] = W_out[labels[b][i]] . hidden[b][i],
 * s[b][i] = softmax_i z[b][i], with hidden device fp32 [B][n_max][hidden]
 * (bat_bipartite_prefill with multi_disc); the other arguments as bat_score. */
BAT_API bat_status bat_score_multi(bat_model m, const float* hidden, const int32_t* labels,
                                   const int32_t* n_items, int32_t B, int32_t n_max, float* scores,
                                   int32_t k, int32_t* topk, float* logits, bat_stream_t stream);

/* ------------------------------------------------------------------------------------------
 * Planned execution: build (host) + upload (device, async on `stream`) the plan of a batch
 * once, then run it any number of times — the same computation as bat_bipartite_prefill
 * without the per-call planning and H2D upload.  The plan PINS every pool entry it reads:
 * bat_kv_evict / bat_kv_release of a pinned entry fail with BAT_E_STATE until bat_plan_destroy,
 * and bat_kv_pool_destroy fails while the pool has live plans.  bat_prefill_plan returns
 * BAT_E_STATE for a plan built on another pool.
 * CUDA graphs (opt-in: BAT_GRAPH=1 in the environment; measured neutral on a B200, where the
 * batch-1 prefill is GPU-bound): on a non-default stream (and with kernel profiling off) bat_prefill_plan runs a
 * plan's first call eagerly (sizing the model's workspace), captures its second call into a CUDA
 * graph and replays that graph on later calls with the same out_hidden, as long as no workspace
 * buffer was reallocated since (a larger plan run in between forces one eager call and a new
 * capture).  Results are bit-identical to eager runs.  The legacy default stream (stream = NULL)
 * always runs eagerly.
 * ---------------------------------------------------------------------------------------- */
typedef struct bat_plan_s* bat_plan;
BAT_API bat_status bat_plan_build(bat_pool p, bat_model m, const bat_query* queries, int32_t B,
                                  bat_stream_t stream, bat_plan* out);
BAT_API bat_status bat_prefill_plan(bat_pool p, bat_model m, bat_plan plan, float* out_hidden,
                                    bat_stream_t stream);

/* ------------------------------------------------------------------------------------------
 * Kernel timing (CUDA events recorded on the launch stream around every kernel of the
 * prefill, grouped by class).  bat_profile_read synchronises on the recorded events.
 * ---------------------------------------------------------------------------------------- */
enum { BAT_K_EMBED = 0, BAT_K_RMSNORM = 1, BAT_K_GEMM_QKV = 2, BAT_K_STAGE = 3, BAT_K_ATTN = 4,
       BAT_K_GEMM_O = 5, BAT_K_GEMM_GU = 6, BAT_K_GEMM_DOWN = 7, BAT_K_OTHER = 8, BAT_K_N = 9 };
BAT_API bat_status bat_profile_enable(bat_model m, int32_t on);
/* Accumulated since the last reset: total ms, launches, algorithmic FLOPs (GEMMs 2MNK;
 * attention 4 * head_dim * q_heads * visible pairs) and algorithmic bytes of class cls. */
BAT_API bat_status bat_profile_read(bat_model m, int32_t cls, double* total_ms, int64_t* launches,
                                    double* flops, double* bytes);
BAT_API bat_status bat_profile_reset(bat_model m);

/* ------------------------------------------------------------------------------------------
 * Plan introspection (host only; bit-exact checks against the oracle's plan)
 * ---------------------------------------------------------------------------------------- */
/* group = q_heads / kv_heads of the model the plan is for (GQA packing of q-tiles). */
BAT_API bat_status bat_plan_create(bat_pool p, int32_t group, const bat_query* queries, int32_t B,
                           bat_plan* out);
BAT_API bat_status bat_plan_destroy(bat_plan plan);
/* info[0..12] of request b: S (suffix tokens), P (prefix tokens), n_pages (incl. suffix
 * pages, excl. padding), n_prefix_pages, n_qtiles, n_ktiles, token_off, scratch_page0,
 * n_live_pairs (visible (query,key) pairs, per head per layer), qtile_tokens,
 * first_qtile (global), page_off (global), n_live_pairs of the last q-tile's rows. */
BAT_API bat_status bat_plan_query_info(bat_plan plan, int32_t b, int64_t info[13]);
enum {
  BAT_PF_TOKENS = 0,  /* int32 [S]  suffix token ids in prompt order */
  BAT_PF_POS = 1,     /* int32 [S]  position ids */
  BAT_PF_SEG = 2,     /* int32 [S]  -1 user, -2 instr, -3 header, i >= 0 item i */
  BAT_PF_PAGES = 3,   /* int32 [n_pages] pool page id >= 0, or -(s+1) for scratch page s */
  BAT_PF_VALID = 4,   /* int32 [n_pages] valid slots per page */
  BAT_PF_KSEG = 5,    /* int32 [16*n_pages] key segment (-1 for empty slots) */
  BAT_PF_KORD = 6,    /* int32 [16*n_pages] 0 prefix key, suffix index+1, INT32_MAX empty */
  BAT_PF_TILES = 7,   /* int32 [n_qtiles][n_ktiles] 0 skip / 1 full / 2 partial */
  BAT_PF_DISC = 8     /* int32 [1] or, multi_disc, [n_items]: suffix rows of the discriminants */
};
/* Copy field `field` of request b into out (cap elements); *count = its length. */
BAT_API bat_status bat_plan_export(bat_plan plan, int32_t b, int32_t field, int32_t* out, int64_t cap,
                           int64_t* count);

/* The DEVICE side of a bat_plan_build plan, read back and decoded exactly as the attention kernel
 * consumes it (block-skip work list, per-q-tile tile states, the loader's page ids and the
 * partial-tile visibility bits computed on the device), for bit-exact checks of the indexing the
 * kernel sees (north_star "page-table and indexing results must match bit-exact").  Fields:
 *   BAT_PFD_VIS       uint8 [S][n_ktiles*128]: 1 iff suffix row t attends key slot k in the
 *                     all-row work list (state 1 = every slot, state 2 = the mask bits, unlisted
 *                     or state-0 tiles = 0); layers 1..L-1 use it
 *   BAT_PFD_VIS_LAST  the same for the last layer's list (only the last q-tile, P:173 trim)
 *   BAT_PFD_KPAGES    int32 [n_ktiles*8]: page id each k-tile's loader copies (pool page >= 0,
 *                     -(s+1) suffix scratch page s, INT32_MIN the all-zero pad page), or
 *                     BAT_PFD_NOT_LOADED for a tile no work item lists (skipped)
 *   BAT_PFD_STAGE     int32 [S][3]: where the fused QKV epilogue (a4) stores suffix row t, from the
 *                     device row map: {global q-tile, suffix page id (as KPAGES), slot in the page}
 * BAT_E_STATE if the device image is inconsistent: KV heads with different lists, a (q-tile,
 * k-tile) pair listed twice, a partial tile without a mask, out-of-range indices. */
enum { BAT_PFD_VIS = 0, BAT_PFD_VIS_LAST = 1, BAT_PFD_KPAGES = 2, BAT_PFD_STAGE = 3 };
#define BAT_PFD_NOT_LOADED (-2147483647)
BAT_API bat_status bat_plan_export_device(bat_plan plan, int32_t b, int32_t field, void* out, int64_t cap,
                                          int64_t* count);

/* ------------------------------------------------------------------------------------------
 * Multi-GPU: hot-replicated / cold-sharded item placement (Algorithm 1)
 * ---------------------------------------------------------------------------------------- */
/* Algorithm 1 line 7 verbatim: R_max = alpha*t*B*(N-1) / (c*S_item*N), t = measured prefill
 * time (s) of one request (replaces PrefillTime, line 4), B tokens/s, S_item = tau_i. */
BAT_API bat_status bat_hrcs_rmax(double B, double t, double alpha, int32_t c, double tau_i,
                         int32_t N, double* r_max_out);
/* Lines 8-18: sort freq descending (ties: lower index first), replicate the first r*n items
 * where r = i/n at the first i with CDF >= 1 - R_max (r = 1 if never reached); the rest are
 * round-robin by hotness rank.  owner_out[i] = -1 replicated, else the owning rank. */
BAT_API bat_status bat_hrcs_place(const double* freq, int64_t n_items, double r_max, int32_t world,
                          int32_t* owner_out, double* r_out);

/* ------------------------------------------------------------------------------------------
 * Prompt scheduler + cache meta service for user prefixes (P:288-294
 * scheduler / meta service, P:366-381 prefix selection, P:405 hotness upkeep, P:441 hit rate).
 * Host-only bookkeeping: it decides each request's prefix side and the user-cache actions; the
 * caller applies them to a pool (bat_kv_evict the evicted users, bat_kv_prefill_entities the
 * admitted user, then bat_bipartite_prefill with the decided order).
 *   policy BAT_SCHED_HOTNESS: UP iff tau_u >= tau_i and (u is cached, or its pages fit
 *     in free space, or evicting cached users of lower sliding-window frequency f_p < f_u in
 *     ascending (f_p, last access, id) order frees enough pages); else IP.
 *   BAT_SCHED_GREEDY: UP iff tau_u >= tau_i, admitting with LRU replacement.
 *   BAT_SCHED_UP / BAT_SCHED_IP / BAT_SCHED_RE: the fixed baselines of P:441 (UP admits with LRU).
 * f_u(t) = the user's requests in (t - window, t], this one included.  A user entry
 * occupies ceil(tau_u / 16) pages.  Requests must arrive with non-decreasing t
 * (BAT_E_INVAL otherwise).  Readings: DESIGN.md R15-R19.
 * ---------------------------------------------------------------------------------------- */
typedef enum { BAT_SCHED_HOTNESS = 0, BAT_SCHED_GREEDY = 1, BAT_SCHED_UP = 2, BAT_SCHED_IP = 3,
               BAT_SCHED_RE = 4 } bat_sched_policy;
typedef struct {
  int32_t policy;         /* bat_sched_policy */
  int64_t capacity_pages; /* pages of the pool set aside for user prefixes */
  double window;          /* sliding-window length W (same unit as the request times) */
} bat_sched_cfg;
typedef struct {
  int32_t order;    /* BAT_ORDER_UP, BAT_ORDER_IP, or -1 (RE: full recompute, no cache) */
  int32_t user_hit; /* UP served from the cached user prefix */
  int32_t admit;    /* UP miss: the user's prefix must be computed and cached (after evictions) */
  int32_t n_evict;  /* users to evict first, written to evict_ids */
  int32_t freq;     /* f_u(t) of the request's user */
} bat_sched_decision;
typedef struct bat_sched_s* bat_sched;
BAT_API bat_status bat_sched_create(const bat_sched_cfg* cfg, bat_sched* out);
BAT_API bat_status bat_sched_destroy(bat_sched s);
/* Decide one request (user_id, tau_u user tokens, tau_i item tokens) arriving at time t and
 * update the user-cache index.  evict_ids: host array of evict_cap entries (BAT_E_INVAL if the
 * evictions do not fit; the state is then unchanged). */
BAT_API bat_status bat_sched_decide(bat_sched s, double t, int64_t user_id, int32_t tau_u, int32_t tau_i,
                                    bat_sched_decision* out, int64_t* evict_ids, int32_t evict_cap);
/* Totals so far: [0] prompt tokens, [1] reused prefix tokens (P:441 hit rate = [1]/[0]),
 * [2] UP hits, [3] UP requests, [4] IP requests, [5] cached users, [6] used pages. */
BAT_API bat_status bat_sched_stats(bat_sched s, int64_t out[7]);
/* Whether user_id's prefix is cached. */
BAT_API int32_t bat_sched_is_cached(bat_sched s, int64_t user_id);

/* Background placement update (P:312 Step 3: "replace the KV cache item according to ad hoc
 * hotness in a background process ... update these items in the replicate area"; footnote P:322:
 * new items "by a similar background compute and update strategy"; reading DESIGN.md R21).
 * owner_old[0..n_old): the current placement (-1 replicated, else the owning rank); freq_new
 * [0..n_new): new access frequencies, ids >= n_old are new items.  owner_new[0..n_new): the
 * replicated area keeps floor(r * n_new + 1/2) items — the top ones by freq_new (descending, lower id
 * first, Algorithm 1 line 8) — cold items keep their owner, and items leaving the replicated
 * area or new cold items go to the rank owning the fewest cold items (ties: lowest rank),
 * hottest first.  Moves follow from the diff: promoted items are pulled by every other rank
 * (bat_kv_replicate), demoted ones dropped (bat_kv_evict) by every rank but the new owner, new
 * items computed (bat_kv_prefill_entities) by their owner, or by every rank if replicated. */
BAT_API bat_status bat_hrcs_refresh(const int32_t* owner_old, int64_t n_old, const double* freq_new, int64_t n_new,
                                    double r, int32_t world, int32_t* owner_new);

/* CUDA-IPC export of the pool arena (64-byte handle) and import of a peer's arena. */
BAT_API bat_status bat_pool_ipc_handle(bat_pool p, void* handle_out64);
BAT_API bat_status bat_pool_attach_peer(bat_pool p, int32_t peer_rank, const void* handle64);
/* Record that entry (kind, id) lives on peer `owner` in its pages owner_pages[0..n_pages). */
BAT_API bat_status bat_kv_register_remote(bat_pool p, int32_t kind, int64_t id, int32_t owner,
                                  const int32_t* owner_pages, int32_t n_pages,
                                  int32_t n_tokens);
/* Host query of a registered remote entry: owner rank, token count, owner page ids. */
BAT_API bat_status bat_kv_lookup_remote(bat_pool p, int32_t kind, int64_t id, int32_t* owner,
                                        int32_t* n_tokens, int32_t* pages_out, int32_t pages_cap,
                                        int32_t* n_pages);
/* Pull the listed remote (cold-sharded) entries from their owners' arenas over NVLink into local
 * pages, making them resolvable by bat_bipartite_prefill.  The copies are enqueued on
 * `stream` — meant to be a dedicated copy stream, so the pull overlaps compute on another stream
 * (order the compute after it with an event) — as copy-engine memcpys, one per run of
 * consecutive pages (no SMs taken from the kernels).
 * Pulled copies are reference counted: an id already pulled gets one more reference, replicated /
 * owned (local) ids are skipped; *n_fetched = entries copied by this call.  Pages a previous
 * bat_kv_release gave back are reused behind a stream wait on their release event.  The owners
 * must not evict the entries while the copy runs.  BAT_E_NOTFOUND for an id neither local nor
 * registered remote; all-or-nothing. */
BAT_API bat_status bat_kv_fetch(bat_pool p, int32_t kind, const int64_t* ids, int32_t n,
                        int32_t* n_fetched, bat_stream_t stream);
/* Pull the listed remote entries as REGULAR local entries (a replicated-area refresh): as
 * bat_kv_fetch on `stream`, but the copies are not reference counted (bat_kv_evict drops them);
 * local ids are skipped; BAT_E_STATE for an id currently held as a pulled (counted) copy. */
BAT_API bat_status bat_kv_replicate(bat_pool p, int32_t kind, const int64_t* ids, int32_t n, bat_stream_t stream);
/* Drop one reference per listed pulled entry (ids as passed to bat_kv_fetch; local ids are
 * skipped).  An entry whose last reference goes is removed and its pages are freed IN STREAM
 * ORDER: they become reusable once the work enqueued on `stream` so far (the batches reading them)
 * has completed — no host synchronisation.  BAT_E_STATE for more releases than fetches or an entry
 * a live plan pins; all-or-nothing. */
BAT_API bat_status bat_kv_release(bat_pool p, int32_t kind, const int64_t* ids, int32_t n, bat_stream_t stream);

/* Double-buffered staging for pre-built plans ("fetched ... overlapped with compute"):
 * reserve n_slots (<= 8) slots of pages_per_slot pages each.  bat_plan_build_staged maps every
 * cold (registered remote) prefix item of its batch to pages of one slot (deduplicated within
 * the batch) and records the pulls; bat_plan_fetch enqueues them on a stream.  Pipelining batch
 * k+1's pull (slot (k+1) % 2) under batch k's compute (slot k % 2) is the caller's event
 * ordering: the pull into a slot must wait for the compute of the batch that last read it. */
BAT_API bat_status bat_kv_staging_reserve(bat_pool p, int32_t n_slots, int64_t pages_per_slot);
BAT_API bat_status bat_plan_build_staged(bat_pool p, bat_model m, const bat_query* queries, int32_t B,
                                         int32_t slot, bat_stream_t stream, bat_plan* out);
/* Bytes of a plan's image: *host_bytes uploaded from the host per call (bat_bipartite_prefill
 * uploads this much for the same batch), *device_bytes its device footprint incl. the masks. */
BAT_API bat_status bat_plan_bytes(bat_plan plan, int64_t* host_bytes, int64_t* device_bytes);
/* Attention work-list shape of a plan (host): out[0] work items of layers 1..L-1 (CTA-sized units
 * the persistent kernel balances over the SMs), out[1] of the last layer, out[2] / out[3] split-KV
 * groups / partial slots of the main list, out[4] / out[5] of the last-layer list.  A list with
 * fewer items than SMs has its long items split into k-tile chunks on separate CTAs (log-sum-exp
 * combine); BAT_SPLITKV=0 disables it. */
BAT_API bat_status bat_plan_work_info(bat_plan plan, int64_t out[6]);
/* Enqueue a staged plan's cold-item pulls on `stream` (copy engines); *n_pages = pages pulled. */
BAT_API bat_status bat_plan_fetch(bat_pool p, bat_plan plan, int64_t* n_pages, bat_stream_t stream);

/* ------------------------------------------------------------------------------------------
 * Test-only entry points (kernel-level parity tests; not part of the serving path)
 * ---------------------------------------------------------------------------------------- */
/* One tcgen05 GEMM: epi 0 out = A B^T (bf16), 1 out = A B^T + bias (bf16), 2 out += A B^T
 * (fp32 out), 3 out = silu(A Bg^T) * (A Bu^T) with Bg = B rows [0,N), Bu = rows [up_row0,..).
 * A: device bf16 [M][K]; B: device bf16 [rows][K]; out leading dimension ldo (elements). */
BAT_API bat_status bat_debug_gemm(int32_t epi, int32_t M, int32_t N, int32_t K, const void* A,
                                  const void* Bw, int64_t b_rows, void* out, int32_t ldo,
                                  const void* bias, int32_t up_row0, int32_t device,
                                  bat_stream_t stream);
/* Layer `layer` of the bipartite attention alone: plan the requests, apply RoPE (if
 * rope_enabled) to the given qkv rows (device bf16 [M][(q_heads+2 kv_heads) head_dim], rows
 * in plan order) and stage them, attend over the pool's prefix pages at that layer and the
 * staged suffix, write O (device bf16 [M][q_heads*head_dim]). */
/* Attach another in-process pool's arena as peer `peer_rank` (single-GPU tests of the
 * NVLink page pull; multi-process code uses bat_pool_ipc_handle / bat_pool_attach_peer). */
BAT_API bat_status bat_debug_attach_peer_pool(bat_pool p, int32_t peer_rank, bat_pool other);
BAT_API bat_status bat_debug_attention_layer(bat_pool p, bat_model m, const bat_query* queries,
                                             int32_t B, int32_t layer, const void* qkv,
                                             void* out_o, int32_t rope_enabled,
                                             bat_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* BAT_H_ */
