// Prompt scheduler + user-prefix cache meta service: the prefix-selection
// policies of PAPER.md P:366 (cache-agnostic greedy) and P:377 (hotness-aware), the sliding-window
// user frequency f_u of P:373 kept up to date on every access, and the page-granular
// user-cache index they act on.  Host-only: decisions and cache actions, which the
// caller applies to a pool.  Readings (R15-R19) are listed in include/bat.h.
#include <algorithm>
#include <cmath>
#include <deque>
#include <memory>
#include <unordered_map>
#include <vector>

#include "common.h"

namespace bat {
namespace {

struct UserState {
  std::deque<double> times;  // access times inside the current window
  double last = -INFINITY;   // last access
  int64_t pages = 0;         // > 0 iff cached
};

struct Sched {
  bat_sched_cfg cfg{};
  std::unordered_map<int64_t, UserState> users;
  std::vector<int64_t> cached;  // ids of cached users
  int64_t used = 0;
  double now = -INFINITY;
  int64_t tot[5] = {0, 0, 0, 0, 0};  // tokens, reused, hits, up, ip

  // f_u(t): accesses in (t - W, t]; older ones can never re-enter a later window
  int32_t freq(UserState& u, double t) {
    while (!u.times.empty() && u.times.front() <= t - cfg.window) u.times.pop_front();
    return static_cast<int32_t>(u.times.size());
  }
};

int64_t pages_of(int32_t tau_u) { return (int64_t(tau_u) + kPageTokens - 1) / kPageTokens; }

}  // namespace
}  // namespace bat

using namespace bat;

struct bat_sched_s {
  Sched s;
};

extern "C" {

bat_status bat_sched_create(const bat_sched_cfg* cfg, bat_sched* out) {
  return guarded([&] {
    BAT_REQUIRE(cfg && out, "null argument");
    BAT_REQUIRE(cfg->policy >= BAT_SCHED_HOTNESS && cfg->policy <= BAT_SCHED_RE, "policy");
    BAT_REQUIRE(cfg->capacity_pages >= 0 && cfg->window > 0.0, "capacity_pages >= 0, window > 0");
    auto p = std::make_unique<bat_sched_s>();
    p->s.cfg = *cfg;
    *out = p.release();
  });
}

bat_status bat_sched_destroy(bat_sched s) {
  return guarded([&] { delete s; });
}

bat_status bat_sched_decide(bat_sched sp, double t, int64_t user_id, int32_t tau_u, int32_t tau_i,
                            bat_sched_decision* out, int64_t* evict_ids, int32_t evict_cap) {
  return guarded([&] {
    BAT_REQUIRE(sp && out, "null argument");
    BAT_REQUIRE(tau_u >= 0 && tau_i >= 0, "token counts");
    Sched& S = sp->s;
    BAT_REQUIRE(t >= S.now, "request times must be non-decreasing");
    const int policy = S.cfg.policy;
    UserState& U = S.users[user_id];
    const int32_t f_u = S.freq(U, t) + 1;  // this request included
    std::vector<int64_t> evict;
    int32_t order = BAT_ORDER_IP, hit = 0, admit = 0;
    if (policy == BAT_SCHED_RE) {
      order = -1;
    } else if (policy == BAT_SCHED_IP || ((policy == BAT_SCHED_HOTNESS || policy == BAT_SCHED_GREEDY) && tau_u < tau_i)) {
      order = BAT_ORDER_IP;
    } else if (U.pages > 0) {
      order = BAT_ORDER_UP;
      hit = 1;
    } else {
      const int64_t need = pages_of(tau_u);
      const int64_t cap = S.cfg.capacity_pages;
      if (need > cap) {
        order = (policy == BAT_SCHED_UP) ? BAT_ORDER_UP : BAT_ORDER_IP;  // UP-only: served, not cached
      } else if (policy == BAT_SCHED_HOTNESS) {
        if (cap - S.used >= need) {
          order = BAT_ORDER_UP;
        } else {
          struct C { int32_t f; double last; int64_t id; int64_t pages; };
          std::vector<C> cand;
          cand.reserve(S.cached.size());
          for (int64_t id : S.cached) {
            UserState& P = S.users[id];
            cand.push_back(C{S.freq(P, t), P.last, id, P.pages});
          }
          std::sort(cand.begin(), cand.end(), [](const C& a, const C& b) {
            if (a.f != b.f) return a.f < b.f;
            if (a.last != b.last) return a.last < b.last;
            return a.id < b.id;
          });
          int64_t free = cap - S.used;
          for (const C& c : cand) {
            if (free >= need || c.f >= f_u) break;
            evict.push_back(c.id);
            free += c.pages;
          }
          if (free >= need) order = BAT_ORDER_UP;
          else evict.clear();
        }
      } else {  // greedy / UP-only: LRU replacement
        std::vector<std::pair<double, int64_t>> cand;
        for (int64_t id : S.cached) cand.push_back({S.users[id].last, id});
        std::sort(cand.begin(), cand.end());
        int64_t free = cap - S.used;
        for (auto& c : cand) {
          if (free >= need) break;
          evict.push_back(c.second);
          free += S.users[c.second].pages;
        }
        order = BAT_ORDER_UP;
      }
      if (order == BAT_ORDER_UP && need <= cap) admit = 1;
    }
    BAT_REQUIRE(int64_t(evict.size()) <= int64_t(evict_cap) && (evict.empty() || evict_ids), "evict_cap too small");
    // ---- commit
    S.now = t;
    U.times.push_back(t);
    U.last = t;
    for (size_t i = 0; i < evict.size(); ++i) {
      UserState& P = S.users[evict[i]];
      S.used -= P.pages;
      P.pages = 0;
      evict_ids[i] = evict[i];
    }
    if (!evict.empty())
      S.cached.erase(std::remove_if(S.cached.begin(), S.cached.end(),
                                    [&](int64_t id) { return S.users[id].pages == 0; }),
                     S.cached.end());
    if (admit) {
      U.pages = pages_of(tau_u);
      S.used += U.pages;
      S.cached.push_back(user_id);
    }
    S.tot[0] += int64_t(tau_u) + tau_i;
    if (order == BAT_ORDER_UP) {
      S.tot[3] += 1;
      if (hit) {
        S.tot[2] += 1;
        S.tot[1] += tau_u;
      }
    } else if (order == BAT_ORDER_IP) {
      S.tot[4] += 1;
      S.tot[1] += tau_i;
    }
    out->order = order;
    out->user_hit = hit;
    out->admit = admit;
    out->n_evict = static_cast<int32_t>(evict.size());
    out->freq = f_u;
  });
}

bat_status bat_sched_stats(bat_sched sp, int64_t out[7]) {
  return guarded([&] {
    BAT_REQUIRE(sp && out, "null argument");
    for (int i = 0; i < 5; ++i) out[i] = sp->s.tot[i];
    out[5] = int64_t(sp->s.cached.size());
    out[6] = sp->s.used;
  });
}

int32_t bat_sched_is_cached(bat_sched sp, int64_t user_id) {
  if (!sp) return 0;
  auto it = sp->s.users.find(user_id);
  return (it != sp->s.users.end() && it->second.pages > 0) ? 1 : 0;
}

}  // extern "C"
