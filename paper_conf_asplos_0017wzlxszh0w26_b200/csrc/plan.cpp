// Host planner: see plan.h.  The visibility rule (DESIGN.md §2 R4-R6):
//   key k is visible to suffix row t  iff  kord[k] <= rord[t]  and
//   (kseg[k] == rseg[t]  or  kseg[k] < 0  or  rseg[t] < 0)
// with kord = 0 for a prefix key (every prefix token precedes every suffix token), the suffix
// index + 1 for a suffix key, INT32_MAX for an empty slot; rord[t] = t + 1.
#include "plan.h"

#include <algorithm>
#include <cstdlib>
#include <numeric>
#include <unordered_map>

namespace bat {
namespace {

struct PrefixEnt {
  int32_t kind;
  int64_t id;
  int32_t seg;
  int32_t expect_n;  // tokens the request carries for it (-1: unchecked)
  int32_t use_n = -1;  // tokens served from the entry (PIC: an item's head); -1: all
};

// A cold item of a staged plan: pages of the staging slot, the pull recorded once per plan.
const Entity* staged_entity(const Pool& pool, const PrefixEnt& e, StagingCtx* stg) {
  if (!stg) return nullptr;
  const EntityKey key{e.kind, e.id};
  auto a = stg->assigned.find(key);
  if (a != stg->assigned.end()) return &a->second;
  auto r = pool.remote.find(key);
  if (r == pool.remote.end()) return nullptr;
  const RemoteEntity& re = r->second;
  const char* peer = pool.peer_arena[re.owner];
  if (!peer) fail(BAT_E_STATE, "peer arena of rank " + std::to_string(re.owner) + " not attached");
  if (stg->used + re.pages.size() > stg->slot_pages->size())
    fail(BAT_E_POOLFULL, "staging slot too small for the batch's cold items");
  Entity en;
  en.n_tokens = re.n_tokens;
  en.fetched = true;
  for (size_t k = 0; k < re.pages.size(); ++k) {
    const int32_t dst = (*stg->slot_pages)[stg->used++];
    en.pages.push_back(dst);
    stg->src.push_back(reinterpret_cast<uint64_t>(peer + int64_t(re.pages[k]) * pool.geo.page_bytes));
    stg->dst.push_back(dst);
  }
  return &stg->assigned.emplace(key, std::move(en)).first->second;
}

void add_prefix_pages(const Pool& pool, const PrefixEnt& e, QueryPlan& qp, StagingCtx* stg) {
  const Entity* ent = pool.find(e.kind, e.id);
  const bool staged = !ent && (ent = staged_entity(pool, e, stg)) != nullptr;
  if (!ent) {
    fail(BAT_E_NOTFOUND, "prefix entry (kind " + std::to_string(e.kind) + ", id " +
                             std::to_string(e.id) + ") is not in the pool");
  }
  if (e.expect_n >= 0 && ent->n_tokens != e.expect_n) {
    fail(BAT_E_INVAL, "prefix entry (kind " + std::to_string(e.kind) + ", id " +
                          std::to_string(e.id) + ") holds " + std::to_string(ent->n_tokens) +
                          " tokens but the request has " + std::to_string(e.expect_n));
  }
  const int32_t use = e.use_n >= 0 ? std::min(e.use_n, ent->n_tokens) : ent->n_tokens;
  if (use == 0) return;  // PIC: the whole item is recomputed
  if (!staged) qp.refs.push_back(EntityKey{e.kind, e.id});
  const size_t n_pages = static_cast<size_t>(ceil_div(use, kPageTokens));
  for (size_t pi = 0; pi < n_pages; ++pi) {
    int32_t nv = std::min<int32_t>(kPageTokens, use - static_cast<int32_t>(pi) * kPageTokens);
    qp.pages.push_back(ent->pages[pi]);
    qp.valid.push_back(nv);
    for (int j = 0; j < kPageTokens; ++j) {
      qp.kseg.push_back(j < nv ? e.seg : -1);
      qp.kord.push_back(j < nv ? 0 : kInvalidOrd);
    }
  }
  qp.P += use;
}

// Suffix tokens / positions / segments of a ranking request (readings R2, R3).
void build_request(const Pool& pool, const bat_query& q, QueryPlan& qp, StagingCtx* stg) {
  BAT_REQUIRE(q.order == BAT_ORDER_UP || q.order == BAT_ORDER_IP, "order must be UP or IP");
  BAT_REQUIRE(q.n_items >= 1, "n_items >= 1");
  BAT_REQUIRE(q.n_instr >= 1, "n_instr >= 1 (the discriminant is the last token, P:173)");
  BAT_REQUIRE(q.n_user >= 0 && q.n_header >= 0, "negative length");
  BAT_REQUIRE(q.n_header == 0 || q.order == BAT_ORDER_IP, "header tokens are IP-only (P:257)");
  BAT_REQUIRE(q.pic_tail >= 0, "pic_tail >= 0");
  BAT_REQUIRE(q.pic_tail == 0 || q.order == BAT_ORDER_IP, "pic_tail (selective recompute) is IP-only");
  BAT_REQUIRE(q.pic_tail == 0 || !q.multi_disc, "pic_tail and multi_disc do not combine");
  BAT_REQUIRE(q.item_off && q.item_id, "item arrays");
  BAT_REQUIRE(q.n_user == 0 || q.user_tok, "user_tok");
  BAT_REQUIRE(q.instr_tok, "instr_tok");
  BAT_REQUIRE(q.n_header == 0 || q.header_tok, "header_tok");
  BAT_REQUIRE(q.item_off[0] == 0, "item_off[0] == 0");
  int32_t m = 0;
  for (int i = 0; i < q.n_items; ++i) {
    int32_t n = q.item_off[i + 1] - q.item_off[i];
    BAT_REQUIRE(n >= 1, "every item has >= 1 token");
    m = std::max(m, n);
  }
  const int32_t nu = q.n_user, nx = q.n_instr, h = q.n_header;
  auto put = [&](const int32_t* t, int32_t n, int32_t seg, int32_t pos0) {
    for (int32_t j = 0; j < n; ++j) {
      qp.tokens.push_back(t[j]);
      qp.seg.push_back(seg);
      qp.pos.push_back(pos0 + j);
    }
  };
  auto put_items = [&](int32_t start) {
    for (int i = 0; i < q.n_items; ++i)
      put(q.item_tok + q.item_off[i], q.item_off[i + 1] - q.item_off[i], i, start);
  };
  if (q.order == BAT_ORDER_UP) {
    if (q.use_cache) {
      add_prefix_pages(pool, PrefixEnt{BAT_ENT_USER, q.user_id, SEG_USER, nu}, qp, stg);
    } else {
      put(q.user_tok, nu, SEG_USER, 0);
    }
    put_items(nu);
    put(q.instr_tok, nx, SEG_INSTR, nu + m);
  } else {
    // PIC (reading R25): item i keeps its first n_i - k_i tokens in the prefix, its last k_i
    // tokens are recomputed after U at positions h + m + |U| + j
    auto tail = [&](int i) { return std::min(q.pic_tail, q.item_off[i + 1] - q.item_off[i]); };
    int32_t any_tail = 0;
    for (int i = 0; i < q.n_items; ++i) any_tail += tail(i);
    if (q.use_cache) {
      if (h > 0) add_prefix_pages(pool, PrefixEnt{BAT_ENT_HEADER, q.header_id, SEG_HEADER, h}, qp, stg);
      for (int i = 0; i < q.n_items; ++i) {
        const int32_t n = q.item_off[i + 1] - q.item_off[i];
        PrefixEnt pe{BAT_ENT_ITEM, q.item_id[i], i, n};
        pe.use_n = n - tail(i);
        add_prefix_pages(pool, pe, qp, stg);
      }
    } else {
      put(q.header_tok, h, SEG_HEADER, 0);
      for (int i = 0; i < q.n_items; ++i)
        put(q.item_tok + q.item_off[i], q.item_off[i + 1] - q.item_off[i] - tail(i), i, h);
    }
    put(q.user_tok, nu, SEG_USER, h + m);
    for (int i = 0; i < q.n_items; ++i) {
      const int32_t n = q.item_off[i + 1] - q.item_off[i], k = tail(i);
      put(q.item_tok + q.item_off[i] + (n - k), k, i, h + m + nu + (n - k));
    }
    put(q.instr_tok, nx, SEG_INSTR, h + m + nu + (any_tail > 0 ? m : 0));
  }
  qp.n_prefix_pages = static_cast<int32_t>(qp.pages.size());
  qp.S = static_cast<int32_t>(qp.tokens.size());
}

void build_entity(const Pool& pool, const PlanRequest& r, QueryPlan& qp) {
  if (r.ctx_kind >= 0) add_prefix_pages(pool, PrefixEnt{r.ctx_kind, r.ctx_id, SEG_HEADER, -1}, qp, nullptr);
  for (int32_t j = 0; j < r.ent_n; ++j) {
    qp.tokens.push_back(r.ent_tok[j]);
    qp.seg.push_back(SEG_USER);  // one entity alone: plain causal attention
    qp.pos.push_back(r.ent_pos0 + j);
  }
  qp.n_prefix_pages = static_cast<int32_t>(qp.pages.size());
  qp.S = r.ent_n;
}

// Exact block-skip states by per-tile summaries (matches the oracle's pair enumeration).
void classify_tiles(QueryPlan& qp, int32_t qt) {
  const int32_t n_slots = qp.n_pages * kPageTokens;
  qp.n_ktiles = static_cast<int32_t>(ceil_div(n_slots, kKtile));
  qp.n_qtiles = static_cast<int32_t>(ceil_div(qp.S, qt));
  constexpr int32_t INF = kInvalidOrd;
  struct KT {
    int32_t min_all = INF, max_all = -1, min_nonitem = INF;
    bool all_valid = true;
    std::vector<std::pair<int32_t, int32_t>> item_min;  // (item, min kord), item ascending
  };
  std::vector<KT> kts(qp.n_ktiles);
  for (int32_t j = 0; j < qp.n_ktiles; ++j) {
    KT& k = kts[j];
    for (int32_t s = j * kKtile; s < (j + 1) * kKtile; ++s) {
      if (s >= n_slots || qp.kord[s] == kInvalidOrd) {
        k.all_valid = false;
        continue;
      }
      int32_t o = qp.kord[s], g = qp.kseg[s];
      k.min_all = std::min(k.min_all, o);
      k.max_all = std::max(k.max_all, o);
      if (g < 0) {
        k.min_nonitem = std::min(k.min_nonitem, o);
      } else {
        auto it = std::lower_bound(k.item_min.begin(), k.item_min.end(), std::make_pair(g, INT32_MIN));
        if (it != k.item_min.end() && it->first == g) it->second = std::min(it->second, o);
        else k.item_min.insert(it, {g, o});
      }
    }
  }
  qp.tiles.assign(static_cast<size_t>(qp.n_qtiles) * qp.n_ktiles, 0);
  std::vector<std::pair<int32_t, int32_t>> row_items;  // (item, max rord)
  for (int32_t i = 0; i < qp.n_qtiles; ++i) {
    const int32_t r0 = i * qt, r1 = std::min(qp.S, (i + 1) * qt);
    const int32_t rmin = r0 + 1;
    int32_t rn_max = -1;
    row_items.clear();
    for (int32_t t = r0; t < r1; ++t) {
      int32_t g = qp.seg[t];
      if (g < 0) {
        rn_max = std::max(rn_max, t + 1);
      } else {
        if (!row_items.empty() && row_items.back().first == g) row_items.back().second = t + 1;
        else {
          auto it = std::find_if(row_items.begin(), row_items.end(), [&](auto& p) { return p.first == g; });
          if (it == row_items.end()) row_items.push_back({g, t + 1});
          else it->second = std::max(it->second, t + 1);
        }
      }
    }
    for (int32_t j = 0; j < qp.n_ktiles; ++j) {
      const KT& k = kts[j];
      bool any = rn_max >= 0 && k.min_all <= rn_max;
      for (size_t a = 0; !any && a < row_items.size(); ++a) {
        int32_t mm = k.min_nonitem;
        auto it = std::lower_bound(k.item_min.begin(), k.item_min.end(),
                                   std::make_pair(row_items[a].first, INT32_MIN));
        if (it != k.item_min.end() && it->first == row_items[a].first) mm = std::min(mm, it->second);
        any = mm <= row_items[a].second;
      }
      uint8_t st = 0;
      if (any) {
        bool excl_free = row_items.empty() || k.item_min.empty() ||
                         (row_items.size() == 1 && k.item_min.size() == 1 &&
                          row_items[0].first == k.item_min[0].first);
        bool full = k.all_valid && k.max_all <= rmin && excl_free;
        st = full ? 1 : 2;
      }
      qp.tiles[static_cast<size_t>(i) * qp.n_ktiles + j] = st;
    }
  }
  // visible pairs per head per layer, O(S + slots): count per row
  int64_t pre_nonitem = 0;
  std::unordered_map<int32_t, int64_t> pre_item;
  for (int32_t s = 0; s < qp.n_prefix_pages * kPageTokens; ++s) {
    if (qp.kord[s] == kInvalidOrd) continue;
    if (qp.kseg[s] < 0) ++pre_nonitem;
    else ++pre_item[qp.kseg[s]];
  }
  const int64_t pre_total = qp.P;
  int64_t sfx_nonitem = 0, live = 0, live_last = 0;
  std::unordered_map<int32_t, int64_t> sfx_item;
  const int32_t last_tile0 = (qp.n_qtiles - 1) * qt;
  for (int32_t t = 0; t < qp.S; ++t) {
    int32_t g = qp.seg[t];
    if (g < 0) ++sfx_nonitem;
    else ++sfx_item[g];
    int64_t row;
    if (g < 0) {
      row = pre_total + (t + 1);
    } else {
      auto pi = pre_item.find(g);
      row = pre_nonitem + (pi == pre_item.end() ? 0 : pi->second) + sfx_nonitem + sfx_item[g];
    }
    live += row;
    if (t >= last_tile0) live_last += row;
  }
  qp.n_live_pairs = live;
  qp.n_live_pairs_last = live_last;
}

}  // namespace

void build_plan(const Pool& pool, int32_t group, int32_t kv_heads,
                const std::vector<PlanRequest>& reqs, Plan& plan, bool build_image, int32_t grid,
                StagingCtx* stg, int32_t qtiles_per_item) {
  BAT_REQUIRE(group >= 1 && group <= kQtileRows, "group in [1,128]");
  plan.group = group;
  plan.kv_heads = kv_heads;
  plan.qt = kQtileRows / group;
  plan.q.assign(reqs.size(), QueryPlan{});
  plan.multi_disc = !reqs.empty() && reqs[0].q && reqs[0].q->multi_disc;
  plan.n_disc = 1;
  for (const PlanRequest& r : reqs) {
    BAT_REQUIRE(bool(r.q && r.q->multi_disc) == plan.multi_disc, "multi_disc must be the same for the whole batch");
    if (plan.multi_disc) {
      BAT_REQUIRE(r.q->order == BAT_ORDER_UP, "multi_disc requires User-as-prefix (the items must be computed, P:259)");
      plan.n_disc = std::max(plan.n_disc, r.q->n_items);
    }
  }
  int32_t tok = 0, sp = 0, qt0 = 0, pg = 0;
  for (size_t b = 0; b < reqs.size(); ++b) {
    QueryPlan& qp = plan.q[b];
    const PlanRequest& r = reqs[b];
    if (r.q) {
      build_request(pool, *r.q, qp, stg);
    } else {
      build_entity(pool, r, qp);
      plan.entity_mode = true;
    }
    BAT_REQUIRE(qp.S >= 1, "request with no suffix tokens");
    if (plan.multi_disc) {  // the last suffix token of every item
      qp.disc.assign(r.q->n_items, -1);
      for (int32_t t = 0; t < qp.S; ++t)
        if (qp.seg[t] >= 0) qp.disc[qp.seg[t]] = t;
      for (int32_t d : qp.disc) BAT_REQUIRE(d >= 0, "multi_disc: an item is not in the suffix");
    } else {
      qp.disc.assign(1, qp.S - 1);
    }
    // the suffix's own pages follow the prefix pages (reading: virtual key order)
    const int32_t n_sfx = static_cast<int32_t>(ceil_div(qp.S, kPageTokens));
    if (r.ent_pages) BAT_REQUIRE(static_cast<int32_t>(r.ent_pages->size()) == n_sfx, "entity pages");
    for (int32_t s = 0; s < n_sfx; ++s) {
      int32_t nv = std::min(kPageTokens, qp.S - s * kPageTokens);
      qp.pages.push_back(r.ent_pages ? (*r.ent_pages)[s] : -(sp + s) - 1);
      qp.valid.push_back(nv);
      for (int j = 0; j < kPageTokens; ++j) {
        int32_t t = s * kPageTokens + j;
        qp.kseg.push_back(j < nv ? qp.seg[t] : -1);
        qp.kord.push_back(j < nv ? t + 1 : kInvalidOrd);
      }
    }
    qp.n_pages = static_cast<int32_t>(qp.pages.size());
    classify_tiles(qp, plan.qt);
    qp.token_off = tok;
    qp.scratch0 = sp;
    qp.qtile0 = qt0;
    qp.page_off = pg;
    tok += qp.S;
    sp += n_sfx;
    qt0 += qp.n_qtiles;
    pg += qp.n_ktiles * kKtilePages;
  }
  plan.M = tok;
  plan.n_spages = sp;
  plan.n_qtiles_total = qt0;
  plan.n_pages_padded = pg;
  if (!build_image) return;

  // ---- flat device image --------------------------------------------------------------
  const int32_t B = static_cast<int32_t>(plan.q.size());
  PlanImage& im = plan.img;
  std::vector<int32_t>& v = im.buf;
  v.clear();
  auto reserve_at = [&](int64_t n) {
    int64_t o = static_cast<int64_t>(v.size());
    o = (o + 3) & ~int64_t(3);  // 16-byte alignment of every array
    v.resize(o + n, 0);
    return o;
  };
  im.off_tok = reserve_at(plan.M);
  im.off_pos = reserve_at(plan.M);
  im.off_rseg = reserve_at(plan.M);
  im.off_rowreq = reserve_at(plan.M);
  im.off_qinfo = reserve_at(int64_t(B) * 8);
  im.off_pages = reserve_at(plan.n_pages_padded);
  im.off_kmeta = reserve_at(int64_t(plan.n_pages_padded) * kPageTokens * 2);
  im.off_qtiles = reserve_at(int64_t(plan.n_qtiles_total) * 4);
  im.off_spages = reserve_at(int64_t(plan.n_spages) * 4);
  im.off_disc = reserve_at(int64_t(B) * plan.n_disc);
  for (int32_t b = 0; b < B; ++b) {
    const QueryPlan& qp = plan.q[b];
    for (int32_t t = 0; t < qp.S; ++t) {
      v[im.off_tok + qp.token_off + t] = qp.tokens[t];
      v[im.off_pos + qp.token_off + t] = qp.pos[t];
      v[im.off_rseg + qp.token_off + t] = qp.seg[t];
      v[im.off_rowreq + qp.token_off + t] = b;
    }
    int32_t* qi = &v[im.off_qinfo + int64_t(b) * 8];
    qi[0] = qp.token_off; qi[1] = qp.S; qi[2] = qp.qtile0; qi[3] = qp.n_qtiles;
    qi[4] = qp.page_off; qi[5] = qp.n_ktiles; qi[6] = qp.scratch0; qi[7] = qp.token_off + qp.S - 1;
    for (int32_t p = 0; p < qp.n_ktiles * kKtilePages; ++p) {
      bool real = p < qp.n_pages;
      v[im.off_pages + qp.page_off + p] = real ? qp.pages[p] : kZeroPage;
      for (int j = 0; j < kPageTokens; ++j) {
        int64_t s = int64_t(p) * kPageTokens + j;
        int64_t o = im.off_kmeta + (int64_t(qp.page_off) * kPageTokens + s) * 2;
        v[o] = real ? qp.kseg[s] : -1;
        v[o + 1] = real ? qp.kord[s] : kInvalidOrd;
      }
    }
    for (int32_t i = 0; i < qp.n_qtiles; ++i) {
      int32_t* e = &v[im.off_qtiles + int64_t(qp.qtile0 + i) * 4];
      e[0] = b; e[1] = i * plan.qt; e[2] = std::min(plan.qt, qp.S - i * plan.qt); e[3] = 0;
    }
    const int32_t n_sfx = static_cast<int32_t>(ceil_div(qp.S, kPageTokens));
    for (int32_t s = 0; s < n_sfx; ++s) {
      int32_t* e = &v[im.off_spages + int64_t(qp.scratch0 + s) * 4];
      e[0] = b; e[1] = s * kPageTokens; e[2] = std::min(kPageTokens, qp.S - s * kPageTokens);
      e[3] = qp.pages[qp.n_prefix_pages + s];
    }
    for (int32_t i = 0; i < plan.n_disc; ++i)  // padding rows repeat the last token
      v[im.off_disc + int64_t(b) * plan.n_disc + i] = qp.token_off + (i < int32_t(qp.disc.size()) ? qp.disc[i] : qp.S - 1);
  }
  // work items: (b, kvh, q-tile pair) sharing every K/V tile, with the union of the two
  // q-tiles' live k-tiles and a state per q-tile; longest first (LPT over the SMs)
  struct W { int32_t b, kvh, q0, q1, n; std::vector<int32_t> kt; int32_t slot = -1; };
  std::unordered_map<int64_t, int32_t> mask_id;  // (b, q-tile, k-tile) -> mask
  std::vector<int32_t> mdesc;
  auto mask_of = [&](int32_t b, int32_t qi, int32_t j) {
    const int64_t key = (int64_t(b) << 40) | (int64_t(qi) << 20) | int64_t(j);
    auto it = mask_id.find(key);
    if (it != mask_id.end()) return it->second;
    const int32_t id = static_cast<int32_t>(mdesc.size() / 4);
    mask_id.emplace(key, id);
    mdesc.insert(mdesc.end(), {b, qi, j, 0});
    return id;
  };
  // split-KV: when a list has fewer items than the persistent grid, a long item's k-tile list is
  // cut into contiguous chunks (>= kSplitMin tiles) run by different CTAs; each chunk writes its
  // O / l and (m, l) to a partial slot and a combine kernel merges them (log-sum-exp weights)
  static const bool split_on = !(std::getenv("BAT_SPLITKV") && std::getenv("BAT_SPLITKV")[0] == '0');
  constexpr int32_t kSplitMin = 2;
  auto make_work = [&](bool last_only, int64_t& off_work, int32_t& n_work, int64_t& off_wslot, int64_t& off_sgrp,
                       int32_t& n_sgrp, int32_t& n_slots) {
    std::vector<W> ws;
    for (int32_t b = 0; b < B; ++b) {
      const QueryPlan& qp = plan.q[b];
      std::vector<std::pair<int32_t, int32_t>> pairs;
      if (last_only) pairs.push_back({qp.n_qtiles - 1, -1});
      else
        for (int32_t i = 0; i < qp.n_qtiles; i += qtiles_per_item)
          pairs.push_back({i, (qtiles_per_item == 2 && i + 1 < qp.n_qtiles) ? i + 1 : -1});
      for (auto& pr : pairs) {
        std::vector<int32_t> kt;
        for (int32_t j = 0; j < qp.n_ktiles; ++j) {
          uint8_t s0 = qp.tiles[static_cast<size_t>(pr.first) * qp.n_ktiles + j];
          uint8_t s1 = pr.second >= 0 ? qp.tiles[static_cast<size_t>(pr.second) * qp.n_ktiles + j] : 0;
          if (s0 || s1) kt.push_back(j | (int32_t(s0) << 24) | (int32_t(s1) << 26));
        }
        if (kt.empty()) continue;  // cannot happen for real rows (each row sees itself)
        for (int32_t h = 0; h < kv_heads; ++h) ws.push_back(W{b, h, pr.first, pr.second, int32_t(kt.size()), kt});
      }
    }
    std::vector<int32_t> groups;  // [g][6]
    n_slots = 0;
    if (split_on && grid > 0 && !ws.empty() && static_cast<int32_t>(ws.size()) < grid) {
      const int32_t want = static_cast<int32_t>(ceil_div(grid, static_cast<int64_t>(ws.size())));
      std::vector<W> out;
      for (W& w : ws) {
        const int32_t c = std::min(want, w.n / kSplitMin);
        if (c <= 1) {
          out.push_back(std::move(w));
          continue;
        }
        groups.insert(groups.end(), {w.b, w.kvh, w.q0, w.q1, n_slots, c});
        for (int32_t k = 0; k < c; ++k) {
          const int32_t t0 = k * w.n / c, t1 = (k + 1) * w.n / c;
          W part{w.b, w.kvh, w.q0, w.q1, t1 - t0, std::vector<int32_t>(w.kt.begin() + t0, w.kt.begin() + t1), n_slots++};
          out.push_back(std::move(part));
        }
      }
      ws.swap(out);
    }
    // cost of an item in k-tile-pair units: its tiles, with a fixed prologue / epilogue share
    // (BAT_LPT_SINGLE, BAT_LPT_ITEM: experiment knobs for the per-tile weight of single-q-tile
    // items and the fixed per-item cost, in quarter k-tile-pair units.  A single-q-tile item
    // costs about as much per tile as a pair — the attention kernel is bound by each q-tile's
    // S -> softmax -> P.V chain, not by tensor work — so both weigh 4; measured in-step
    // 593.5 (3/8) vs 597.4 (4/8) vs 598.0 (4/4) vs 593.0 (4/16) TFLOP/s)
    static const int64_t w1 = std::getenv("BAT_LPT_SINGLE") ? std::atoi(std::getenv("BAT_LPT_SINGLE")) : 4;
    static const int64_t wi = std::getenv("BAT_LPT_ITEM") ? std::atoi(std::getenv("BAT_LPT_ITEM")) : 8;
    auto cost = [](const W& a) { return int64_t(a.n) * (a.q1 >= 0 ? 4 : w1) + wi; };
    std::stable_sort(ws.begin(), ws.end(), [&](const W& a, const W& c) { return cost(a) > cost(c); });
    if (grid > 0 && static_cast<int32_t>(ws.size()) > grid) {
      // LPT over the persistent grid: CTA c runs items c, c + grid, c + 2 grid, ... of the list,
      // so place every CTA's greedily balanced share at those positions (empty items pad)
      std::vector<std::vector<int32_t>> per(grid);
      std::vector<std::pair<int64_t, int32_t>> heap;  // (load, cta), min-heap
      for (int32_t c = 0; c < grid; ++c) heap.push_back({0, c});
      auto gt = [](const std::pair<int64_t, int32_t>& a, const std::pair<int64_t, int32_t>& b) { return a > b; };
      std::make_heap(heap.begin(), heap.end(), gt);
      for (int32_t i = 0; i < static_cast<int32_t>(ws.size()); ++i) {
        std::pop_heap(heap.begin(), heap.end(), gt);
        heap.back().first += cost(ws[i]);
        per[heap.back().second].push_back(i);
        std::push_heap(heap.begin(), heap.end(), gt);
      }
      size_t rounds = 0;
      for (auto& l : per) rounds = std::max(rounds, l.size());
      std::vector<W> out;
      out.reserve(rounds * grid);
      for (size_t r = 0; r < rounds; ++r)
        for (int32_t c = 0; c < grid; ++c)
          out.push_back(r < per[c].size() ? ws[per[c][r]] : W{0, 0, -1, -1, 0, {}, -1});
      ws.swap(out);
    }
    n_work = static_cast<int32_t>(ws.size());
    off_work = reserve_at(int64_t(n_work) * 8);
    off_wslot = reserve_at(std::max<int64_t>(1, n_work));
    for (int32_t w = 0; w < n_work; ++w) v[off_wslot + w] = ws[w].slot;
    n_sgrp = static_cast<int32_t>(groups.size() / 6);
    off_sgrp = reserve_at(std::max<int64_t>(1, int64_t(groups.size())));
    std::copy(groups.begin(), groups.end(), v.begin() + off_sgrp);
    int64_t total_kt = 0;
    for (auto& w : ws) total_kt += w.n;
    int64_t off_kt = reserve_at(total_kt);
    // the page ids of every listed k-tile, in list order (8 per tile): the attention loader
    // reads them at addresses known in advance instead of chasing kt list -> page table
    int64_t off_tp = reserve_at(total_kt * kKtilePages);
    int64_t off_km = reserve_at(total_kt * 2);
    int64_t cur = 0;
    for (int32_t w = 0; w < n_work; ++w) {
      int32_t* e = &v[off_work + int64_t(w) * 8];
      e[0] = ws[w].b; e[1] = ws[w].kvh; e[2] = ws[w].q0; e[3] = ws[w].q1;
      e[4] = static_cast<int32_t>(off_kt + cur); e[5] = ws[w].n;
      e[6] = static_cast<int32_t>(off_tp + cur * kKtilePages); e[7] = static_cast<int32_t>(off_km + cur * 2);
      const int32_t page_off = plan.q[ws[w].b].page_off;
      for (int32_t x : ws[w].kt) {
        const int32_t j = x & 0xFFFFFF;
        v[off_km + cur * 2] = ((x >> 24) & 3) == 2 ? mask_of(ws[w].b, ws[w].q0, j) : -1;
        v[off_km + cur * 2 + 1] = ((x >> 26) & 3) == 2 ? mask_of(ws[w].b, ws[w].q1, j) : -1;
        for (int l = 0; l < kKtilePages; ++l)
          v[off_tp + cur * kKtilePages + l] = v[im.off_pages + page_off + int64_t(j) * kKtilePages + l];
        v[off_kt + cur++] = x;
      }
    }
  };
  make_work(false, im.off_work, plan.n_work, im.off_wslot, im.off_sgrp, im.n_sgrp, im.n_slots);
  make_work(true, im.off_work_last, plan.n_work_last, im.off_wslot_last, im.off_sgrp_last, im.n_sgrp_last,
            im.n_slots_last);
  im.n_masks = static_cast<int32_t>(mdesc.size() / 4);
  im.off_mdesc = reserve_at(std::max<int64_t>(1, int64_t(mdesc.size())));
  std::copy(mdesc.begin(), mdesc.end(), v.begin() + im.off_mdesc);
  reserve_at(0);  // align the end of the host part
  im.off_masks = static_cast<int64_t>(v.size());
  im.total_ints = im.off_masks + int64_t(im.n_masks) * (plan.qt + 1) * 4;
}

}  // namespace bat
