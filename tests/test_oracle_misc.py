"""Pins for oracle/score.py, oracle/sizes.py, oracle/hrcs.py, oracle/scheduler.py."""
import math

import numpy as np
import pytest

from oracle import hrcs, scheduler, sizes
from oracle.score import score, softmax, topk


# ----------------------------------------------------------------- score
def test_softmax_closed_form():
    s = softmax(np.log([1.0, 2.0, 3.0]))          # exp(z_i) = 1, 2, 3 -> s = i / 6
    np.testing.assert_allclose(s, [1 / 6, 2 / 6, 3 / 6], rtol=1e-15)


def test_softmax_shift_invariance_and_extremes():
    z = np.array([1000.0, 1000.0, -1000.0])       # max subtraction keeps this finite
    np.testing.assert_allclose(softmax(z), [0.5, 0.5, 0.0], atol=1e-300)


def test_score_uses_identifier_rows():
    rows = np.array([[1.0, 0.0], [0.0, 2.0], [1.0, 1.0]])
    hf = np.array([0.5, 0.25])
    z, s, top = score(rows, hf, k=2)
    np.testing.assert_allclose(z, [0.5, 0.5, 0.75])
    assert list(top) == [2, 0]                    # tie between 0 and 1 -> lower index first


def test_topk_tie_rule():
    assert list(topk(np.array([0.2, 0.3, 0.3, 0.2]), 4)) == [1, 2, 0, 3]


# ------------------------------------------------------------------ sizes (Table 2)
@pytest.mark.parametrize("kv,d,L,expected", [(2, 128, 28, 28672), (4, 128, 28, 57344), (8, 64, 16, 32768)])
def test_table2_bytes_per_token(kv, d, L, expected):
    assert sizes.kv_bytes_per_token(kv, d, L) == expected


def test_kv_size_examples():
    # a 1000-token Qwen2-1.5B user occupies ~29 MB; 10^8 such users ~2.9 PB
    user = sizes.prefix_bytes(1000, 2, 128, 28)
    assert round(user / 1e6) == 29
    assert round(1e8 * round(user / 1e6) * 1e6 / 1e15, 1) == 2.9
    # P:273 / P:427: 1M (10M) items x 10 tokens ~ 287 GB (2.87 TB)
    assert round(sizes.prefix_bytes(10 * 10 ** 6, 2, 128, 28) / 1e9) == 287
    assert round(sizes.prefix_bytes(10 * 10 ** 7, 2, 128, 28) / 1e12, 2) == 2.87
    # one 16-token page of all 28 layers: 16 x 28672 B
    assert sizes.page_bytes(16, 2, 128, 28) == 458752


# ---------------------------------------------------------------- HRCS (Algorithm 1)
def test_rmax_paper_formula_by_hand():
    # alpha*t = 0.2 s; 0.2 * 100 tok/s * 3 / (10 * 5 * 4) = 0.3
    assert math.isclose(hrcs.rmax_paper(B=100, t=2, alpha=0.1, c=10, tau_i=5, N=4), 0.3)
    assert hrcs.rmax_paper(B=100, t=2, alpha=0.1, c=10, tau_i=5, N=1) == 0.0


def test_replication_ratio_hand_cases():
    F = [0.5, 0.3, 0.1, 0.1]
    assert hrcs.replication_ratio(F, 0.25) == 2 / 4     # CDF .5, .8 >= .75
    assert hrcs.replication_ratio(F, 1.0) == 1 / 4      # R_max >= 1 -> first item
    assert hrcs.replication_ratio(F, 5.0) == 1 / 4
    assert hrcs.replication_ratio(F, 0.0) == 1.0        # nothing may cross the network
    assert hrcs.replication_ratio([1, 3, 2, 4], 0.35) == 2 / 4   # unnormalised, unsorted input


def test_place_round_robin_by_hotness():
    F = [0.05, 0.4, 0.05, 0.3, 0.1, 0.1]
    rep, owner = hrcs.place(F, 2 / 6, 2)
    assert rep == [1, 3]
    assert owner == {4: 0, 5: 1, 0: 0, 2: 1}                      # ties -> lower id first


def test_compute_replication_ratio_end_to_end():
    r = hrcs.compute_replication_ratio(B=100, F=[0.5, 0.3, 0.1, 0.1], tau_u=1000, tau_i=5,
                                       alpha=0.1, c=10, N=4, t=2)
    assert r == 2 / 4                                   # R_max = 0.3 -> CDF .8 >= .7 at i = 2


# ----------------------------------------------------------- scheduler
def test_cache_agnostic_rule():
    assert scheduler.cache_agnostic(4096, 3200) == "UP"
    assert scheduler.cache_agnostic(512, 3200) == "IP"
    assert scheduler.cache_agnostic(3200, 3200) == "UP"


def test_hotness_aware_rule():
    assert scheduler.hotness_aware(4096, 3200, 5.0, [1.0, 7.0]) == "UP"
    assert scheduler.hotness_aware(4096, 3200, 0.5, [1.0, 7.0]) == "IP"
    assert scheduler.hotness_aware(512, 3200, 99.0, [1.0]) == "IP"
    assert scheduler.hotness_aware(4096, 3200, 0.0, []) == "UP"        # empty C_u


def test_window_similarity():
    assert scheduler.window_similarity(3, 3) == 1.0
    assert scheduler.window_similarity(3, 1) == 0.5


# ------------------------------------------------- scheduler simulation (NEXT-2)
def test_simulation_hand_trace():
    """Pinned by hand (see tests/test_sched.py::test_scheduler_hand_trace for the arithmetic)."""
    tr = [(0.0, 1, 4000, 1600), (1.0, 2, 5000, 1600), (2.0, 1, 4000, 1600), (3.0, 3, 6000, 1600),
          (3.5, 4, 500, 1600), (4.0, 3, 6000, 1600)]
    d, tot = scheduler.simulate(tr, "hotness", 700, 10.0)
    assert [x[0] for x in d] == ["UP", "UP", "UP", "IP", "IP", "UP"]
    assert d[5][2] == [2] and d[2][1] is True
    d, tot = scheduler.simulate(tr, "greedy", 700, 10.0)  # LRU evicts u2 (last access 1.0) for u3
    assert [x[0] for x in d] == ["UP", "UP", "UP", "UP", "IP", "UP"] and d[3][2] == [2]
    assert tot["hits"] == 2 and tot["reused"] == 4000 + 1600 + 6000


def test_simulation_degenerate_policies_are_closed_forms():
    import synth
    tr = synth.request_trace(3, 500, 50)
    tokens = sum(a + b for _, _, a, b in tr)
    _, t_re = scheduler.simulate(tr, "re", 1000, 5.0)
    assert t_re["reused"] == 0 and t_re["tokens"] == tokens
    _, t_ip = scheduler.simulate(tr, "ip", 1000, 5.0)
    assert t_ip["reused"] == sum(b for *_, b in tr) and t_ip["ip"] == len(tr)
    # unbounded cache: UP-only hits every repeat visit of a user, misses each first visit
    _, t_up = scheduler.simulate(tr, "up", 10 ** 9, 5.0)
    first = len({u for _, u, _, _ in tr})
    assert t_up["hits"] == len(tr) - first
    # zero capacity: hotness never admits, so it is IP for every request
    _, t_h = scheduler.simulate(tr, "hotness", 0, 5.0)
    assert t_h["ip"] == len(tr) and t_h["hits"] == 0


# ------------------------------------------------ placement refresh (footnote P:322; R21)
def test_refresh_hand_case():
    """5 placed items, 1 new; r = 1/3 of 6 -> 2 replicated.  New order: 1 (.5), 2 (.2), 0 (.1),
    5 (.1, new), 3, 4 (.05).  Replicated {1, 2}; 3 and 4 keep owners 0 / 1 (loads 1, 1); demoted
    item 0 -> rank 0 (tie -> lower rank), new item 5 -> rank 1."""
    assert hrcs.refresh([-1, 0, 1, 0, 1], [0.1, 0.5, 0.2, 0.05, 0.05, 0.1], 1 / 3, 2) == [0, -1, -1, 0, 1, 1]


@pytest.mark.parametrize("seed", range(6))
def test_refresh_invariants(seed):
    """The replicated area is exactly Algorithm 1's top-r set under the new frequencies (the
    same set place() picks); items cold before and after never move; every rank's cold load
    differs by at most the imbalance it already had (new assignments go to the least loaded)."""
    rng = np.random.default_rng(seed)
    n_old, n_new, N = int(rng.integers(10, 200)), 0, int(rng.integers(1, 6))
    n_new = n_old + int(rng.integers(0, 30))
    F_old = rng.pareto(1.1, size=n_old) + 1e-3
    r = float(rng.uniform(0, 0.5))
    rep, own = hrcs.place(F_old, r, N)
    owner_old = [-1 if i in set(rep) else own[i] for i in range(n_old)]
    F_new = rng.pareto(1.1, size=n_new) + 1e-3
    owner_new = hrcs.refresh(owner_old, F_new, r, N)
    rep_new, _ = hrcs.place(F_new, r, N)
    assert {i for i in range(n_new) if owner_new[i] < 0} == set(rep_new)
    for i in range(n_old):
        if owner_old[i] >= 0 and owner_new[i] >= 0:
            assert owner_new[i] == owner_old[i]
    loads = [sum(1 for o in owner_new if o == k) for k in range(N)]
    kept = [sum(1 for i in range(n_old) if owner_old[i] == k and owner_new[i] == k) for k in range(N)]
    assert max(loads) - min(loads) <= max(1, max(kept) - min(kept))


def test_refresh_without_change_is_identity():
    """Same frequencies, same r, no new items: the placement of Algorithm 1 is a fixed point."""
    F = np.arange(50, 0, -1, dtype=float)
    rep, own = hrcs.place(F, 0.2, 3)
    owner = [-1 if i in set(rep) else own[i] for i in range(50)]
    assert hrcs.refresh(owner, F, 0.2, 3) == owner
