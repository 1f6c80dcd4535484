"""Prefix selection rules (TEST INFRASTRUCTURE ONLY).

Cache-agnostic greedy rule: "compares the number of user tokens and item tokens and
selects the one with more tokens as the prefix" (ties -> user, matching P:377's >=).
Hotness-aware rule, P:377:
    prefix(r) = user  if tau_u(r) >= tau_i(r) and f_u(r) > min_{p in C_u} f_p
                item  otherwise
with min over an empty C_u = -inf (reading R14).
"""
from __future__ import annotations

from typing import Iterable


def cache_agnostic(tau_u: int, tau_i: int) -> str:
    return "UP" if tau_u >= tau_i else "IP"


def hotness_aware(tau_u: int, tau_i: int, f_u: float, cached_freqs: Iterable[float]) -> str:
    freqs = list(cached_freqs)
    lowest = min(freqs) if freqs else float("-inf")
    return "UP" if (tau_u >= tau_i and f_u > lowest) else "IP"


def window_similarity(f_now: float, f_prev: float) -> float:
    """1 - |f(t) - f(t - delta)| / (f(t) + f(t - delta))."""
    return 1.0 - abs(f_now - f_prev) / (f_now + f_prev)


# ---------------------------------------------------------------------------------------------
# Plain reference simulation of the prompt scheduler + user-prefix cache (
# P:366-381 rules, P:405 meta-service hotness, P:441 hit-rate definition).  Readings (DESIGN.md
# R15-R19):
#   * f_u(t) = number of the user's requests with timestamp in (t - W, t], the current one
#     included (a sliding window; it "decays" as the window slides);
#   * a user whose prefix is cached is served User-as-prefix (a hit) whenever tau_u >= tau_i —
#     the P:377 comparison is against the OTHER cached users (min over C_u \ {u});
#   * admission: free pages first; otherwise evict cached users in ascending
#     (f_p, last access, id) order while f_p < f_u, and admit only if that frees enough pages
#     (else the request falls back to Item-as-prefix and nothing is evicted);
#   * the cache-agnostic greedy policy and the UP-only baseline admit every UP user
#     with LRU replacement ("using LRU replacement"); IP-only and RE never cache users;
#   * a user entry occupies ceil(tau_u / 16) pages (P:298 paged entries);
#   * hit rate = reused prefix tokens / all prompt tokens; IP reuses the item tokens
#     (the item pool holds every candidate, §8(e)), a UP hit reuses the user tokens.
# ---------------------------------------------------------------------------------------------
POLICIES = ("hotness", "greedy", "up", "ip", "re")


def _pages(tau_u: int) -> int:
    return -(-int(tau_u) // 16)


def simulate(trace, policy: str, capacity_pages: int, window: float):
    """trace: iterable of (time, user_id, tau_u, tau_i), times non-decreasing.
    Returns (decisions, totals): decisions[k] = (order, hit, evicted_user_ids) with order in
    {"UP", "IP", "RE"}; totals = dict(tokens, reused, hits, up, ip)."""
    assert policy in POLICIES
    history = {}     # user -> list of access times (all; the window is applied on read)
    cached = {}      # user -> pages
    last = {}        # user -> last access time (LRU / tie break)
    used = 0
    out = []
    tot = dict(tokens=0, reused=0, hits=0, up=0, ip=0)

    def freq(u, t):
        return sum(1 for s in history.get(u, ()) if t - window < s <= t)

    for (t, u, tau_u, tau_i) in trace:
        history.setdefault(u, []).append(t)
        tot["tokens"] += tau_u + tau_i
        evicted = []
        if policy == "re":
            order, hit = "RE", False
        elif policy == "ip" or (policy in ("hotness", "greedy") and tau_u < tau_i):
            order, hit = "IP", False
        elif u in cached:
            order, hit = "UP", True
        else:
            need = _pages(tau_u)
            if need > capacity_pages:  # can never be cached: UP-only serves it uncached
                order, hit = ("IP" if policy in ("hotness", "greedy") else "UP"), False
                need = None
            elif policy == "hotness":
                f_u = freq(u, t)
                if capacity_pages - used >= need:
                    order = "UP"
                else:
                    cand = sorted(cached, key=lambda p: (freq(p, t), last[p], p))
                    free, chosen = capacity_pages - used, []
                    for p in cand:
                        if free >= need or freq(p, t) >= f_u:
                            break
                        chosen.append(p)
                        free += cached[p]
                    if free >= need:
                        order, evicted = "UP", chosen
                    else:
                        order = "IP"
                hit = False
            else:  # greedy / up: admit with LRU replacement
                cand = sorted(cached, key=lambda p: (last[p], p))
                free, chosen = capacity_pages - used, []
                for p in cand:
                    if free >= need:
                        break
                    chosen.append(p)
                    free += cached[p]
                order, hit, evicted = "UP", False, chosen
            if order == "UP" and need is not None:
                for p in evicted:
                    used -= cached.pop(p)
                cached[u] = need
                used += need
        last[u] = t
        if order == "UP":
            tot["up"] += 1
            if hit:
                tot["hits"] += 1
                tot["reused"] += tau_u
        elif order == "IP":
            tot["ip"] += 1
            tot["reused"] += tau_i
        out.append((order, hit, list(evicted)))
    return out, tot
