// Host planner: per request, the suffix tokens in prompt order, their
// bipartite positions and segments, the key-slot list (prefix entries'
// pages, then the suffix's own pages), key metadata, and the block-skip tile states
// of every (packed q-tile, 128-key k-tile) pair; plus the flat device image the kernels read.
#pragma once

#include <cstdint>
#include <vector>

#include "common.h"
#include "pool.h"

namespace bat {

struct QueryPlan {
  int32_t S = 0, P = 0;
  int32_t n_pages = 0, n_prefix_pages = 0, n_qtiles = 0, n_ktiles = 0;
  int32_t token_off = 0, scratch0 = 0, qtile0 = 0, page_off = 0;
  int64_t n_live_pairs = 0;       // visible (row, key) pairs per head per layer
  int64_t n_live_pairs_last = 0;  // ... of the rows in the last q-tile (last-layer trim)
  std::vector<int32_t> tokens, pos, seg;  // [S]
  std::vector<int32_t> pages, valid;      // [n_pages]
  std::vector<int32_t> kseg, kord;        // [16 * n_pages]
  std::vector<uint8_t> tiles;             // [n_qtiles * n_ktiles]: 0 skip, 1 full, 2 partial
  std::vector<int32_t> disc;              // suffix rows of the discriminant(s): [1] or, multi, [n_items]
  std::vector<EntityKey> refs;            // prefix entries whose pages the plan reads
};

// One request description, independent of the C struct (entity prefill builds these too).
struct PlanRequest {
  const bat_query* q = nullptr;  // a ranking request, or
  // an entity-prefill pseudo request: tokens at pos0.., causal, optional context entry,
  // suffix pages = the new entry's own pool pages
  const int32_t* ent_tok = nullptr;
  int32_t ent_n = 0, ent_pos0 = 0;
  int32_t ctx_kind = -1;
  int64_t ctx_id = 0;
  const std::vector<int32_t>* ent_pages = nullptr;
};

// Flat int32 image uploaded once per call; offsets (in int32 units) into it.
struct PlanImage {
  std::vector<int32_t> buf;
  int64_t off_tok = 0, off_pos = 0, off_rseg = 0;   // [M]
  int64_t off_rowreq = 0;                           // [M] request index of every suffix row
  int64_t off_qinfo = 0;                            // [B][8]
  int64_t off_pages = 0;                            // [n_pages_padded_total]
  int64_t off_kmeta = 0;                            // [16 * n_pages_padded_total][2]
  int64_t off_qtiles = 0;                           // [n_qtiles_total][4] {b, t0, ntok, 0}
  int64_t off_spages = 0;                           // [n_spages][4] {b, t0, ntok, target}
  int64_t off_work = 0, off_work_last = 0;          // [W][8] {b, kvh, q0, q1|-1, kt_off, kt_n, tp_off, km_off}
  // split-KV (small batches): per work item its partial-result slot (-1: writes O directly);
  // per split group {b, kvh, q0, q1, first slot, parts} for the combine kernel
  int64_t off_wslot = 0, off_wslot_last = 0;        // [W]
  int64_t off_sgrp = 0, off_sgrp_last = 0;          // [groups][6]
  int32_t n_sgrp = 0, n_sgrp_last = 0, n_slots = 0, n_slots_last = 0;
  int64_t off_ktl = 0;                              // kt list: ktile | state0 << 24 | state1 << 26
  int64_t off_disc = 0;                             // [B][n_disc] global discriminant rows
  // Visibility masks of the partial (state 2) (q-tile, k-tile) pairs, shared by all KV heads and
  // layers: mask m = (b, q-tile, k-tile) from off_mdesc [n_masks][4]; per listed tile of a work
  // item, km_off + 2 x + q holds q-tile q's mask id (-1: not partial).  The masks themselves,
  // [n_masks][qt + 1 rows][4 x 32 bits] (row qt: the padding rows' mask), are computed on the
  // device into [off_masks, total_ints) beyond the uploaded host part (launch_masks).
  int64_t off_mdesc = 0, off_masks = 0, total_ints = 0;
  int32_t n_masks = 0;
};

struct Plan {
  int32_t group = 1, qt = 128, kv_heads = 1;
  std::vector<QueryPlan> q;
  int32_t M = 0, n_qtiles_total = 0, n_spages = 0, n_pages_padded = 0;
  int32_t n_work = 0, n_work_last = 0;
  bool entity_mode = false;
  bool multi_disc = false;  // one discriminant per item: off_disc holds [B][n_disc]
  int32_t n_disc = 1;       // discriminant rows per request in the image (multi: max n_items)
  PlanImage img;
};

// Build the plan of a batch.  Pool supplies the entry -> pages index.  Throws bat::Error.
// grid > 0: order the attention work lists for a persistent grid of that many CTAs (LPT
// balance; empty items pad the rounds).
// stg != nullptr: prefix items that are not local but registered remote are mapped to pages of
// the staging slot (deduplicated per plan) and their pulls recorded in *stg.
// qtiles_per_item: 2 = attention work items are q-tile PAIRS sharing every K/V tile (the v1/v2
// kernels), 1 = single q-tiles with their own exact k-tile lists (the v3 kernel).
void build_plan(const Pool& pool, int32_t group, int32_t kv_heads,
                const std::vector<PlanRequest>& reqs, Plan& plan, bool build_image, int32_t grid = 0,
                StagingCtx* stg = nullptr, int32_t qtiles_per_item = 2);

}  // namespace bat
