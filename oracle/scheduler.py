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
